#!/bin/bash
# flat-kernel pass: solve parity (incl. the 64 bench vectors), bench c2 line, ncu instruction counts
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_solve.py tests/test_gpu_goldens.py -k "not f4 and not gamma" -x -q > gpurun_out/pytest_flat.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_flat.log
timeout 600 python bench.py --steps 10 --warmup 3 --no-extra > gpurun_out/bench_flat.json 2> gpurun_out/bench_flat.err
M=sm__inst_executed_pipe_alu.sum,sm__inst_executed_pipe_fma.sum,sm__inst_executed.sum,dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,l1tex__t_sectors_pipe_lsu_mem_local_op_ld.sum,sm__warps_active.avg.pct_of_peak_sustained_active
timeout 600 ncu --metrics $M --clock-control none -k regex:"k_flat" --csv --log-file gpurun_out/inst_c2_sym.csv python scripts/profile_target.py c2 > /dev/null 2>&1
tail -3 gpurun_out/pytest_flat.log; head -c 1500 gpurun_out/bench_flat.json; tail -3 gpurun_out/bench_flat.err
