for v in 0 2 4 8; do for c in C2 C4; do
TSG_SMALL_NNZ=$v timeout 300 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/sm_${v}_$c.json 2>/dev/null
echo "small_nnz=$v $(python scripts/bsum.py gpurun_out/sm_${v}_$c.json)"
done; done
