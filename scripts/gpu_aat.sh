mkdir -p gpurun_out
for c in C1 C4 C2; do timeout 600 python bench.py --config $c --aat --steps 5 --warmup 3 --e2e-steps 1 > gpurun_out/aat_$c.json 2> gpurun_out/aat_$c.err; done
python scripts/bsum.py gpurun_out/aat_*.json
