#!/bin/bash
# quick pass: solve parity + window replay paths + sanitizers + c2 bench line + one-vector overhead
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_solve.py tests/test_gpu_goldens.py tests/test_gpu_sanitizer.py tests/test_gpu_replay.py -q -x -k "not f4 and not gamma and (solve or c2 or c4 or sanitizer or window or edge)" > gpurun_out/pytest_chk.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_chk.log
timeout 300 python bench.py --steps 10 --warmup 3 --no-extra --no-cpu-baseline > gpurun_out/bench_chk.json 2> gpurun_out/bench_chk.err
timeout 120 python scripts/solve_overhead.py > gpurun_out/ovh.txt 2>&1
tail -3 gpurun_out/pytest_chk.log; head -c 300 gpurun_out/bench_chk.json; echo; grep -o '"time_to_optimal_ms": [0-9.]*' gpurun_out/bench_chk.json; cat gpurun_out/ovh.txt
