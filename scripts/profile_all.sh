#!/bin/bash
# ncu evidence for profiles/: launch lists (cold, serialised) + one full capture per hot kernel.
mkdir -p gpurun_out
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_bench_c2.csv \
    python bench.py --steps 3 --warmup 3 --no-extra --no-cpu-baseline > /dev/null 2>&1; echo "list c2 rc=$?"
for t in c4 c5 f2 f4; do
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$t.csv \
      python scripts/profile_target.py $t > /dev/null 2>&1; echo "list $t rc=$?"
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_flat_fam -c 1 \
    -o gpurun_out/full_flat -f python scripts/profile_target.py c2 > /dev/null 2>&1; echo "full flat rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_fact_gv|k_fact_dp" -c 2 \
    -o gpurun_out/full_fact -f python scripts/profile_target.py c4 > /dev/null 2>&1; echo "full fact rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_chain|k_unpermute|k_count" -c 3 \
    -o gpurun_out/full_replay -f python scripts/profile_target.py c5 > /dev/null 2>&1; echo "full replay rc=$?"
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"k_wc_lanes" -c 1 \
    -o gpurun_out/full_wc -f python scripts/profile_target.py f2 > /dev/null 2>&1; echo "full wc rc=$?"
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"k_ep_spec|k_ep_stitch|k_ep_count" -c 3 \
    -o gpurun_out/full_ep -f python scripts/profile_target.py f4 > /dev/null 2>&1; echo "full ep rc=$?"
