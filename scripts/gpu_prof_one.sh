# --set full of kernels matching KREGEX in one warm call of CFG with OPTS (JSON), source page exported
mkdir -p gpurun_out
CFG=${CFG:-C2}; K=${KREGEX:-k_s3w}; TAG=${TAG:-one}
timeout 900 ncu --set full --clock-control none --import-source on --profile-from-start off -k "regex:$K" \
  -o gpurun_out/prof_${TAG}_${CFG} python scripts/prof_one.py $CFG "${OPTS:-{\}}" > gpurun_out/prof_${TAG}_${CFG}.log 2>&1
tail -3 gpurun_out/prof_${TAG}_${CFG}.log
for k in $(echo $K | tr '|' ' '); do
ncu -i gpurun_out/prof_${TAG}_${CFG}.ncu-rep --page source --csv --print-source cuda,sass -k regex:"$k" > gpurun_out/src_${TAG}_${CFG}_$k.csv 2>/dev/null
python scripts/srcprof.py gpurun_out/src_${TAG}_${CFG}_$k.csv 45 > gpurun_out/srcsum_${TAG}_${CFG}_$k.txt 2>&1
done
python profiles/summarize.py full gpurun_out/prof_${TAG}_${CFG}.ncu-rep > gpurun_out/full_${TAG}_${CFG}.md 2>&1
cat gpurun_out/full_${TAG}_${CFG}.md
