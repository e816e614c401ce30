# iteration: gpu parity tests, quick benches (env variants via VARIANTS="A=1,B=2 ..."), C2 launch list
set -x
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -8 > gpurun_out/pytest_gpu.log
for v in ${VARIANTS:-base}; do
  n=$(echo $v | tr '/' '_')
  for c in ${CFGS:-C2 C3 C4}; do
    env $(echo $v | tr ',' ' ' | sed 's/^base$//') timeout 300 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/qb_${n}_$c.json 2> gpurun_out/qb_${n}_$c.err
  done
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/launches_it_C2.csv python bench.py --config C2 --profile --steps 1 --warmup 1 > /dev/null 2>&1
cat gpurun_out/pytest_gpu.log
for v in ${VARIANTS:-base}; do n=$(echo $v | tr '/' '_'); echo "== $v"; python scripts/bsum.py gpurun_out/qb_${n}_*.json; done
python profiles/summarize.py launches gpurun_out/launches_it_C2.csv | head -16
