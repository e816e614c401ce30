# C1 per-call latency, default vs VARIANT builds (3 runs each)
for v in default ${VARIANTS:-nopdl}; do
  if [ $v = default ]; then unset TSG_LIBRARY; else export TSG_LIBRARY=$PWD/variants/$v/libtsg.so; fi
  for i in 1 2 3; do timeout 300 python scripts/c1_latency.py C1 2>/dev/null | grep '^{' | python -c "import json,sys; d=json.loads(sys.stdin.readline()); print('$v C1', round(d['event_ms_median'],4), round(d['wall_ms_median'],4), d['launches'])"; done
done
