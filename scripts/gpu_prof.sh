# usage: bash scripts/gpu_prof.sh TAG CONFIG "regex" [count]
set -x
TAG=$1; CFG=$2; RX=$3; CNT=${4:-3}
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k "regex:$RX" -s ${SKIP:-3} -c $CNT \
  -o gpurun_out/prof_${TAG}_${CFG} python bench.py --config $CFG --profile --steps 1 --warmup 1 > gpurun_out/prof_${TAG}_${CFG}.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/launches_${TAG}_${CFG}.csv python bench.py --config $CFG --profile --steps 1 --warmup 1 > /dev/null 2>&1
ls -la gpurun_out
