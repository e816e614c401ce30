# variant probe over library builds: VARIANTS (default = in-tree) x CFGS x OPTS
mkdir -p gpurun_out
for v in ${VARIANTS:-default}; do
  if [ $v = default ]; then unset TSG_LIBRARY; else export TSG_LIBRARY=$PWD/variants/$v/libtsg.so; fi
  for c in ${CFGS:-C2}; do
    eval "timeout 600 python scripts/variant_probe.py $c $OPTS" > gpurun_out/probe_${v}_$c.json 2> gpurun_out/probe_${v}_$c.err
    tail -3 gpurun_out/probe_${v}_$c.err
    echo "== $v $c"; python -c "
import json,sys; d=json.load(open('gpurun_out/probe_${v}_$c.json'))
for r in d['results']: print(r['opts'], r['ms'], r['step_ms'].get('ms_step2'), r['step_ms'].get('ms_step3'), r['same_as_first'])"
  done
done
