# round-2 closing evidence after programmatic dependent launch (STAGE=1: tests + bench lines; STAGE=2: ncu launch lists,
# DRAM traffic per step, --set full summaries).  Reports stay small: summarised on the box.
set -x
mkdir -p gpurun_out
if [ "${STAGE:-1}" = "1" ]; then
  nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/r2c_smi.txt 2>&1
  timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -15 > gpurun_out/r2c_pytest.log
  timeout 600 python bench.py > gpurun_out/r2c_bench_default.json 2> gpurun_out/r2c_bench_default.err
  timeout 600 python bench.py --config C1 --steps 50 --warmup 5 --no-cpu-baseline --e2e-steps 0 > gpurun_out/r2c_bench_C1.json 2> gpurun_out/r2c_bench_C1.err
  timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/r2c_bench_ref.json 2> gpurun_out/r2c_bench_ref.err
  for c in C3 C4; do
    timeout 600 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/r2c_bench_$c.json 2> gpurun_out/r2c_bench_$c.err
  done
  timeout 900 python bench.py --config C5 --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/r2c_bench_C5.json 2> gpurun_out/r2c_bench_C5.err
  python -m paper_conf_ppopp_niuljs0022_b200 > /dev/null 2>&1
  python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/r2c_smoke.log 2>&1
elif [ "${STAGE}" = "2" ]; then
  for c in C1 C2 C3 C4; do
    timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02c_${c}_launches.csv \
      python bench.py --config $c --steps 2 --warmup 1 --profile > /dev/null 2>&1
  done
  for c in C2 C3 C4; do
    timeout 600 ncu --profile-from-start off --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum \
      --clock-control none --csv --log-file gpurun_out/r02c_traffic_$c.csv python scripts/traffic.py $c > /dev/null 2>&1
  done
  timeout 900 ncu --set full --clock-control none --import-source on --profile-from-start off \
    -k "regex:k_num_dense_row|k_sym_rows|k_num_rows|k_row_merge" -o /tmp/prof_r2c_C3 python scripts/traffic.py C3 > /dev/null 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on --profile-from-start off \
    -k "regex:^k_s3$|k_s3_small|k_s2$|k_row_merge|k_s2_light" -o /tmp/prof_r2c_C2 python scripts/traffic.py C2 > /dev/null 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on --profile-from-start off \
    -k "regex:k_row_rank|k_s3_small|k_s2_light" -o /tmp/prof_r2c_C4 python scripts/traffic.py C4 > /dev/null 2>&1
  for c in C2 C3 C4; do
    python profiles/summarize.py full /tmp/prof_r2c_$c.ncu-rep > gpurun_out/r2c_full_$c.md 2>&1
    sz=$(stat -c %s /tmp/prof_r2c_$c.ncu-rep)
    if [ "$sz" -lt 18000000 ]; then cp /tmp/prof_r2c_$c.ncu-rep gpurun_out/; fi
  done
fi
du -sh gpurun_out
if [ "${STAGE:-1}" = "3" ]; then
  for tool in memcheck racecheck synccheck; do
    extra=""; [ $tool = memcheck ] && extra="--report-api-errors no"
    timeout 900 compute-sanitizer --tool $tool $extra python scripts/sanitize.py > gpurun_out/r2c_san_$tool.log 2>&1
    tail -3 gpurun_out/r2c_san_$tool.log
  done
fi
