set -x
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -4 > gpurun_out/pytest_gpu.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/launches_it_C4.csv python bench.py --config C4 --profile --steps 1 --warmup 0 > /dev/null 2>&1
CFG=C4 KREGEX="k_row_big|k_s2_light|k_s3_small" COUNT=3 TAG=c4 bash scripts/gpu_srcprof.sh
cat gpurun_out/pytest_gpu.log
python profiles/summarize.py launches gpurun_out/launches_it_C4.csv > gpurun_out/launches_it_C4.md
