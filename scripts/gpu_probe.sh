# variant probe on one B200: CFGS configs x the option sets in OPTS (one JSON per line)
mkdir -p gpurun_out
for c in ${CFGS:-C2}; do
  eval "timeout 600 python scripts/variant_probe.py $c $OPTS" > gpurun_out/probe_$c.json 2> gpurun_out/probe_$c.err
  tail -3 gpurun_out/probe_$c.err
done
cat gpurun_out/probe_*.json
