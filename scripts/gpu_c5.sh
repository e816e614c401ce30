set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=memory.total,memory.used --format=csv
( time timeout 1200 python bench.py --config C5 --steps 3 --warmup 3 --e2e-steps 1 > gpurun_out/b_C5.json ) 2> gpurun_out/b_C5.err
timeout 300 python bench.py --config C2 --steps 5 --warmup 3 --row-blocks 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/b_C2_rb3.json 2> gpurun_out/b_C2_rb3.err
python scripts/bsum.py gpurun_out/b_C5.json gpurun_out/b_C2_rb3.json
