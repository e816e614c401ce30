# k_row_rank residency A/B on C4 (and C5's first row block via bench? no: C4 only), per-kernel times
for v in default ${VARIANTS}; do
  if [ $v = default ]; then unset TSG_LIBRARY; else export TSG_LIBRARY=$PWD/variants/$v/libtsg.so; fi
  timeout 300 python scripts/kernel_times.py C4 "{}" 1 2>/dev/null | head -2 | sed "s/^/$v /"
done
