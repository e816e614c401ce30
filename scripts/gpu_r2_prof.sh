# round-2 evidence on one B200 (keep gpurun_out under 64 MiB: reports are summarised on the box)
# stage 1: launch lists (C1-C4) + DRAM traffic per step of one warm call (C2-C4)
# stage 2 (STAGE=2): ncu --set full of the top kernels of C2 / C3 / C4, summarised here
set -x
mkdir -p gpurun_out
if [ "${STAGE:-1}" = "1" ]; then
for c in C1 C2 C3 C4; do
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02_${c}_launches.csv \
    python bench.py --config $c --steps 2 --warmup 1 --profile > /dev/null 2>&1
done
for c in C2 C3 C4; do
  timeout 600 ncu --profile-from-start off --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum \
    --clock-control none --csv --log-file gpurun_out/traffic_$c.csv python scripts/traffic.py $c > /dev/null 2>&1
done
else
timeout 900 ncu --set full --clock-control none --import-source on --profile-from-start off \
  -k "regex:k_s3<|k_s3_small|k_s2\\b|k_s2\\(|k_row_merge|k_s2_light" \
  -o /tmp/prof_r2final_C2 python scripts/traffic.py C2 > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on --profile-from-start off \
  -k "regex:k_num_dense|k_sym_rows|k_num_rows|k_row_merge|k_num_small" \
  -o /tmp/prof_r2final_C3 python scripts/traffic.py C3 > /dev/null 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on --profile-from-start off \
  -k "regex:k_row_rank|k_s3_small|k_s2_light|k_compact|k_row_small" \
  -o /tmp/prof_r2final_C4 python scripts/traffic.py C4 > /dev/null 2>&1
for c in C2 C3 C4; do
  python profiles/summarize.py full /tmp/prof_r2final_$c.ncu-rep > gpurun_out/r02_full_$c.md 2>&1
  ls -la /tmp/prof_r2final_$c.ncu-rep
  sz=$(stat -c %s /tmp/prof_r2final_$c.ncu-rep)
  if [ "$sz" -lt 18000000 ]; then cp /tmp/prof_r2final_$c.ncu-rep gpurun_out/; fi
done
fi
du -sh gpurun_out
