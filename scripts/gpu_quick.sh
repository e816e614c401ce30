# quick GPU iteration: parity tests + short benches (no cpu baseline / e2e)
set -x
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -15 > gpurun_out/pytest_gpu.log
for c in ${CFGS:-C2 C3 C4}; do timeout 300 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/qb_$c.json 2> gpurun_out/qb_$c.err; done
cat gpurun_out/pytest_gpu.log
python scripts/bsum.py gpurun_out/qb_*.json
