# round-2 iteration on one B200: GPU parity (not slow) + short benches, optional launch list
set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt 2>&1
timeout ${PYT:-900} python -m pytest tests -m "gpu and not slow" -x -q ${PYARGS:-} 2>&1 | tail -25 > gpurun_out/pytest_gpu.log
for c in ${CFGS:-C2 C3}; do timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/qb_$c.json 2> gpurun_out/qb_$c.err; done
if [ -n "$LAUNCH" ]; then
  for c in $LAUNCH; do timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launch_$c.csv python bench.py --config $c --steps 2 --warmup 1 --profile > /dev/null 2>&1; done
fi
cat gpurun_out/pytest_gpu.log
python scripts/bsum.py gpurun_out/qb_*.json
