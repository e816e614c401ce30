# C1 bench line (flush between steps) for the in-tree build and VARIANTS, twice each
for v in default ${VARIANTS:-nopdl}; do
  if [ $v = default ]; then unset TSG_LIBRARY; else export TSG_LIBRARY=$PWD/variants/$v/libtsg.so; fi
  for i in 1 2; do timeout 300 python bench.py --config C1 --steps 50 --warmup 5 --no-cpu-baseline --e2e-steps 0 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v', d['ms_per_step'], d['config']['step_ms'])"; done
done
