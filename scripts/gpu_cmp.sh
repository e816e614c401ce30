set -x
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -15 > gpurun_out/pytest_gpu.log
for c in ${CFGS:-C2 C3}; do
  timeout 300 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/qb_$c.json 2> gpurun_out/qb_$c.err
  timeout 300 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 0 --step3-rows > gpurun_out/qbr_$c.json 2> gpurun_out/qbr_$c.err
done
cat gpurun_out/pytest_gpu.log | tail -3
python scripts/bsum.py gpurun_out/qb_*.json gpurun_out/qbr_*.json
