#!/bin/bash
# ncu evidence of the current build: launch lists + full captures (profile_all.sh) and the
# integer-pipe instruction counts bench.py's rooflines read (scripts/inst_counts.py)
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
bash scripts/profile_all.sh
M=sm__inst_executed_pipe_alu.sum,sm__inst_executed_pipe_fma.sum,sm__inst_executed.sum,dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,l1tex__t_sectors_pipe_lsu_mem_local_op_ld.sum,sm__warps_active.avg.pct_of_peak_sustained_active
timeout 600 ncu --metrics $M --clock-control none -k regex:"k_flat_fam" --csv --log-file gpurun_out/inst_c2.csv python scripts/profile_target.py c2 > /dev/null 2>&1; echo "inst c2 rc=$?"
timeout 600 ncu --metrics $M --clock-control none -k regex:"k_fact_gv|k_fact_dp" --csv --log-file gpurun_out/inst_c4.csv python scripts/profile_target.py c4 > /dev/null 2>&1; echo "inst c4 rc=$?"
ls -la gpurun_out/*.ncu-rep gpurun_out/*.csv
