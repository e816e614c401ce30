# per-kernel launch lists (ncu, cold cache) for the given configs
mkdir -p gpurun_out
for c in ${CFGS:-C2}; do
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/launches_${TAG:-x}_$c.csv python bench.py --config $c --profile --steps 1 --warmup 1 > /dev/null 2>&1
python profiles/summarize.py launches gpurun_out/launches_${TAG:-x}_$c.csv > gpurun_out/launches_${TAG:-x}_$c.md
done
