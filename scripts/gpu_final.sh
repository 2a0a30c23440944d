#!/bin/bash
# final pass of a round: every GPU test, smoke, the bench line, the c5 launch
# list and a full capture of the replay kernels of the default path
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c5.csv \
    python scripts/profile_target.py c5 > /dev/null 2>&1; echo "list c5 rc=$?"
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"k_chain|k_unpermute|k_count" -c 3 \
    -o gpurun_out/full_replay -f python scripts/profile_target.py c5 > /dev/null 2>&1; echo "full replay rc=$?"
tail -2 gpurun_out/pytest_gpu.log; tail -2 gpurun_out/smoke.log; head -c 300 gpurun_out/bench.json; tail -2 gpurun_out/bench.err
