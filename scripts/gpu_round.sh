#!/bin/bash
# One GPU session: parity tests, bench, ncu launch list + full captures.
# Usage (under gpurun): bash scripts/gpu_round.sh [tests|bench|ncu|all]
set -u
mkdir -p gpurun_out
what=${1:-all}
if [[ $what == tests || $what == all ]]; then
  timeout 1500 python -m pytest tests -m gpu -x -q --durations=15 > gpurun_out/pytest_gpu.log 2>&1
  echo "pytest rc=$?"; tail -25 gpurun_out/pytest_gpu.log
fi
if [[ $what == bench || $what == all ]]; then
  timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
  echo "bench rc=$?"; tail -3 gpurun_out/bench.err; cat gpurun_out/bench.json
fi
if [[ $what == ncu || $what == all ]]; then
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c2.csv \
      python bench.py --steps 2 --warmup 3 --no-extra --no-cpu-baseline > /dev/null 2>&1; echo "ncu list c2 rc=$?"
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c5.csv \
      python scripts/profile_target.py c5 > /dev/null 2>&1; echo "ncu list c5 rc=$?"
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c4.csv \
      python scripts/profile_target.py c4 > /dev/null 2>&1; echo "ncu list c4 rc=$?"
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_flat_pair -c 1 \
      -o gpurun_out/prof_flat -f python scripts/profile_target.py c2 > /dev/null 2>&1; echo "ncu full flat rc=$?"
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_spec|k_stitch" -c 2 \
      -o gpurun_out/prof_replay -f python scripts/profile_target.py c5 > /dev/null 2>&1; echo "ncu full replay rc=$?"
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_fact_g -c 1 \
      -o gpurun_out/prof_fact -f python scripts/profile_target.py c4 > /dev/null 2>&1; echo "ncu full fact rc=$?"
fi
