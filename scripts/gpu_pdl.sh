# PDL A/B: full GPU suite on the default build, then C1 latency and C1-C4 probes for default vs nopdl
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -4 > gpurun_out/pdl_pytest.log
cat gpurun_out/pdl_pytest.log
for v in default nopdl; do
  if [ $v = default ]; then unset TSG_LIBRARY; else export TSG_LIBRARY=$PWD/variants/$v/libtsg.so; fi
  for i in 1 2; do timeout 300 python scripts/c1_latency.py C1 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('$v C1', d['event_ms_median'], d['wall_ms_median'], d['launches'])"; done
done
unset TSG_LIBRARY
VARIANTS="default nopdl" CFGS="C2 C3 C4" OPTS="'{}'" bash scripts/gpu_probe2.sh
