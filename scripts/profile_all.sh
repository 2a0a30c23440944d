#!/bin/bash
# ncu evidence for profiles/: launch lists (cold, serialised) + one full capture per hot kernel.
mkdir -p gpurun_out
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_bench_c2.csv \
    python bench.py --steps 3 --warmup 3 --no-extra --no-cpu-baseline > /dev/null 2>&1; echo "list c2 rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c4.csv \
    python scripts/profile_target.py c4 > /dev/null 2>&1; echo "list c4 rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c5.csv \
    python scripts/profile_target.py c5 > /dev/null 2>&1; echo "list c5 rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_flat_pair -c 1 \
    -o gpurun_out/full_flat -f python scripts/profile_target.py c2 > /dev/null 2>&1; echo "full flat rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_fact_gv|k_fact_dp" -c 2 \
    -o gpurun_out/full_fact -f python scripts/profile_target.py c4 > /dev/null 2>&1; echo "full fact rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_spec|k_stitch|k_unpermute|k_count" -c 4 \
    -o gpurun_out/full_replay -f python scripts/profile_target.py c5 > /dev/null 2>&1; echo "full replay rc=$?"
