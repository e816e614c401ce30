for v in default async; do
  if [ $v = default ]; then unset TSG_LIBRARY; else export TSG_LIBRARY=$PWD/variants/$v/libtsg.so; fi
  for i in 1 2; do echo -n "$v "; timeout 300 python bench.py --config C3 --steps 20 --warmup 5 --no-cpu-baseline --e2e-steps 0 | python3 -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(round(d['value'],1), round(d['ms_per_step'],4), d['config']['step_ms'])"; done
done
