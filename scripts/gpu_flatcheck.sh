#!/bin/bash
# k_flat_fam check: solve parity (c1/c2 paths + the 64 bench vectors), one-vector / 64-vector step times,
# local-memory sectors and instruction counts of the c2 launch
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_solve.py tests/test_gpu_goldens.py -q -x -k "not f4 and not gamma and not c4" > gpurun_out/pytest_fc.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_fc.log
timeout 120 python scripts/solve_overhead.py > gpurun_out/ovh.txt 2>&1
M=sm__inst_executed_pipe_alu.sum,sm__inst_executed_pipe_fma.sum,sm__inst_executed.sum,dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,l1tex__t_sectors_pipe_lsu_mem_local_op_ld.sum,sm__warps_active.avg.pct_of_peak_sustained_active
timeout 600 ncu --metrics $M --clock-control none -k regex:"k_flat_fam" --csv --log-file gpurun_out/inst_c2.csv python scripts/profile_target.py c2 > /dev/null 2>&1; echo "inst c2 rc=$?"
tail -2 gpurun_out/pytest_fc.log; cat gpurun_out/ovh.txt; grep -E "local_op_ld|time_duration|inst_executed.sum" gpurun_out/inst_c2.csv | cut -c1-20,150-400 | head
