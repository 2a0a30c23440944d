#!/bin/bash
# replay pass: every replay parity test (all paths, full-size goldens, closed loop, sanitizers)
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 2400 python -m pytest tests/test_gpu_replay.py tests/test_gpu_goldens.py tests/test_gpu_epochs.py tests/test_gpu_sanitizer.py -x -q -k "not c2 and not c4" > gpurun_out/pytest_rall.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_rall.log
tail -15 gpurun_out/pytest_rall.log
