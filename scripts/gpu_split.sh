# group-split A/B: C2 full, a C2 1/8 shard and C4 for the in-tree build and VARIANTS
for v in default ${VARIANTS}; do
  if [ $v = default ]; then unset TSG_LIBRARY; else export TSG_LIBRARY=$PWD/variants/$v/libtsg.so; fi
  for sh in 1 8; do timeout 300 python scripts/kernel_times.py C2 "{}" $sh 2>/dev/null | head -1 | sed "s/^/$v /"; done
  timeout 300 python scripts/kernel_times.py C4 "{}" 1 2>/dev/null | head -1 | sed "s/^/$v /"
done
