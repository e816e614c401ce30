# source-level ncu of the step kernels on one config (CFG, KREGEX), exported to CSV for scripts/srcagg.py
set -x
mkdir -p gpurun_out
CFG=${CFG:-C2}; K=${KREGEX:-k_s3}; TAG=${TAG:-src}
timeout 900 ncu --set full --clock-control none --import-source on -k "regex:$K" -s ${SKIP:-0} -c ${COUNT:-1} \
  -o gpurun_out/prof_${TAG}_${CFG} python bench.py --config $CFG --profile --steps 1 --warmup 0 > gpurun_out/prof_${TAG}_${CFG}.log 2>&1
for k in $(echo $K | tr '|' ' '); do
ncu -i gpurun_out/prof_${TAG}_${CFG}.ncu-rep --page source --csv --print-source cuda,sass -k regex:"$k\$" > gpurun_out/src_${TAG}_${CFG}_$k.csv 2>/dev/null
done
python profiles/summarize.py full gpurun_out/prof_${TAG}_${CFG}.ncu-rep > gpurun_out/full_${TAG}_${CFG}.md 2>&1
ls -la gpurun_out
