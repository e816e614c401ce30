# round profile: default bench line, launch lists (C2, C3, C4), --set full of the top kernels
# (C2, C3), fp32/fp16 quick benches.  TAG names the files.
set -x
mkdir -p gpurun_out
TAG=${TAG:-r}
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -4 > gpurun_out/pytest_gpu_${TAG}.log
timeout 900 python bench.py > gpurun_out/bench_${TAG}.json 2> gpurun_out/bench_${TAG}.err
for c in C2 C3 C4; do
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/launches_${TAG}_$c.csv python bench.py --config $c --profile --steps 1 --warmup 1 > /dev/null 2>&1
done
timeout 900 ncu --set full --clock-control none --import-source on -k "regex:k_s3|k_s2|k_row_merge" -s 0 -c 5 \
  -o gpurun_out/prof_${TAG}_C2 python bench.py --config C2 --profile --steps 1 --warmup 0 > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k "regex:k_s3" -s 0 -c 3 \
  -o gpurun_out/prof_${TAG}_C3 python bench.py --config C3 --profile --steps 1 --warmup 0 > /dev/null 2>&1
for d in f32 f16; do for c in C2 C3; do
timeout 300 python bench.py --config $c --dtype $d --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/qb_${TAG}_${d}_$c.json 2>/dev/null
done; done
for c in C2 C3 C4; do python profiles/summarize.py launches gpurun_out/launches_${TAG}_$c.csv > gpurun_out/launches_${TAG}_$c.md 2>&1; done
python profiles/summarize.py full gpurun_out/prof_${TAG}_C2.ncu-rep gpurun_out/prof_${TAG}_C3.ncu-rep > gpurun_out/full_${TAG}.md 2>&1
cat gpurun_out/pytest_gpu_${TAG}.log gpurun_out/bench_${TAG}.json
ls gpurun_out
