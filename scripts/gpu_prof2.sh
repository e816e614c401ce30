# source-level ncu of step-2 and step-1 kernels on C2, plus launch lists of C3/C4 for the current build
set -x
mkdir -p gpurun_out
TAG=${TAG:-p2}
timeout 900 ncu --set full --clock-control none --import-source on -k "regex:k_s2$|k_row_merge|k_s2_light" -s 0 -c 3 \
  -o gpurun_out/prof_${TAG}_C2 python bench.py --config C2 --profile --steps 1 --warmup 0 > gpurun_out/prof_${TAG}_C2.log 2>&1
for k in k_s2 k_row_merge k_s2_light; do
ncu -i gpurun_out/prof_${TAG}_C2.ncu-rep --page source --csv --print-source cuda,sass -k regex:"^$k\$" > gpurun_out/src_${TAG}_$k.csv 2>/dev/null
done
for c in C3 C4; do
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/launches_${TAG}_$c.csv python bench.py --config $c --profile --steps 1 --warmup 1 > /dev/null 2>&1
done
python profiles/summarize.py full gpurun_out/prof_${TAG}_C2.ncu-rep > gpurun_out/full_${TAG}_C2.md 2>&1
ls -la gpurun_out
