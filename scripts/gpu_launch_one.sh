# launch list of one config (CFG) + quick bench; TAG names the files
set -x
mkdir -p gpurun_out
CFG=${CFG:-C2}; TAG=${TAG:-l}
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/launches_${TAG}_$CFG.csv python bench.py --config $CFG --profile --steps 1 --warmup 1 > /dev/null 2>&1
python scripts/summarize_launches.py gpurun_out/launches_${TAG}_$CFG.csv 2>/dev/null || true
