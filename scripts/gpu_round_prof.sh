# round profile: launch lists (C2, C3, C4) + --set full of the top kernels (C2, C3)
set -x
mkdir -p gpurun_out
for c in C2 C3 C4; do
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/launches_${TAG}_$c.csv python bench.py --config $c --profile --steps 1 --warmup 1 > /dev/null 2>&1
done
timeout 900 ncu --set full --clock-control none --import-source on -k "regex:k_s3|k_s2|k_row_small" -s 3 -c 3 \
  -o gpurun_out/prof_${TAG}_C2 python bench.py --config C2 --profile --steps 1 --warmup 1 > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k "regex:k_s3" -s 1 -c 1 \
  -o gpurun_out/prof_${TAG}_C3 python bench.py --config C3 --profile --steps 1 --warmup 1 > /dev/null 2>&1
ls gpurun_out
