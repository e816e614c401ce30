# variants only (no tests): VARIANTS="base TSG_LIBRARY=variants/x/libtsg.so ENV=1,ENV2=3" CFGS="C2"
set -x
mkdir -p gpurun_out
for v in ${VARIANTS:-base}; do
  n=$(echo $v | tr '/=,' '___')
  for c in ${CFGS:-C2}; do
    env $(echo $v | tr ',' ' ' | sed 's/^base$//') timeout 300 python bench.py --config $c --steps ${STEPS:-10} --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/qv_${n}_$c.json 2> gpurun_out/qv_${n}_$c.err
  done
done
for v in ${VARIANTS:-base}; do n=$(echo $v | tr '/=,' '___'); echo "== $v"; python scripts/bsum.py gpurun_out/qv_${n}_*.json; done
