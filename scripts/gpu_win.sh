#!/bin/bash
# replay pass: parity (all paths), replay timings
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_replay.py tests/test_gpu_goldens.py tests/test_gpu_epochs.py -x -q -k "not c2 and not c4 and not window" > gpurun_out/pytest_win.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_win.log
timeout 200 python scripts/replay_variants.py overlap=PROTEUS_REPLAY_CHAIN=0,PROTEUS_REPLAY_OVERLAP=1 serial=PROTEUS_REPLAY_CHAIN=0,PROTEUS_REPLAY_OVERLAP=0 > gpurun_out/win_bench.json 2> gpurun_out/win_bench.err
tail -5 gpurun_out/pytest_win.log; cat gpurun_out/win_bench.json; tail -5 gpurun_out/win_bench.err
