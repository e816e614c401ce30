set -x
mkdir -p gpurun_out
for c in ${CFGS:-C2 C3 C4}; do timeout 300 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/qb_$c.json 2> gpurun_out/qb_$c.err; done
python scripts/bsum.py gpurun_out/qb_*.json
