# A/B of library variants: per config the median call time and the top kernels (kernel_times.py)
for v in default ${VARIANTS}; do
  if [ $v = default ]; then unset TSG_LIBRARY; else export TSG_LIBRARY=$PWD/variants/$v/libtsg.so; fi
  for c in ${CFGS:-C2 C4}; do timeout 300 python scripts/kernel_times.py $c "{}" 1 2>/dev/null | head -${TOPK:-4} | sed "s/^/$v /"; done
done
