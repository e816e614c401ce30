# re-establish state: gpu parity tests, default bench line, quick benches on C2..C4
set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -15 > gpurun_out/pytest_gpu.log
timeout 600 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
for c in ${CFGS:-C2 C3 C4}; do timeout 300 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/qb_$c.json 2> gpurun_out/qb_$c.err; done
cat gpurun_out/pytest_gpu.log
cat gpurun_out/bench_default.json
python scripts/bsum.py gpurun_out/qb_*.json
