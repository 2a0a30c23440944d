#!/bin/bash
# round-2 final evidence: c2 parity after the flat-kernel change, launch lists
# (c2 bench step, c5), full captures of k_flat_fam and the replay kernels, the
# instruction counts bench.py's ALU rooflines read
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_solve.py tests/test_gpu_goldens.py -q -x -k "c2 or flat or c1" > gpurun_out/pytest_c2.log 2>&1; echo "pytest c2 rc=$?"; tail -2 gpurun_out/pytest_c2.log
timeout 600 python bench.py --no-extra --no-cpu-baseline > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err; echo "bench c2 rc=$?"; head -c 300 gpurun_out/bench_c2.json; echo
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_bench_c2.csv \
    python bench.py --steps 3 --warmup 3 --no-extra --no-cpu-baseline > /dev/null 2>&1; echo "list c2 rc=$?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c5.csv \
    python scripts/profile_target.py c5 > /dev/null 2>&1; echo "list c5 rc=$?"
M=sm__inst_executed_pipe_alu.sum,sm__inst_executed_pipe_fma.sum,sm__inst_executed.sum,dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,l1tex__t_sectors_pipe_lsu_mem_local_op_ld.sum,sm__warps_active.avg.pct_of_peak_sustained_active
timeout 600 ncu --metrics $M --clock-control none -k regex:"k_flat_fam" --csv --log-file gpurun_out/inst_c2.csv python scripts/profile_target.py c2 > /dev/null 2>&1; echo "inst c2 rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_flat_fam -c 1 \
    -o gpurun_out/full_flat -f python scripts/profile_target.py c2 > /dev/null 2>&1; echo "full flat rc=$?"
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"k_chain|k_unpermute|k_count" -c 3 \
    -o gpurun_out/full_replay -f python scripts/profile_target.py c5 > /dev/null 2>&1; echo "full replay rc=$?"
ls -la gpurun_out/*.ncu-rep gpurun_out/*.csv
