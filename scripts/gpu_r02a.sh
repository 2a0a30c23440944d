#!/bin/bash
# round-2 GPU pass: tests, bench, per-scenario costs, integer-pipe instruction counts
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python bench.py --steps 10 --warmup 3 > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 900 python scripts/scenario_costs.py > gpurun_out/scenario_costs.json 2> gpurun_out/scenario_costs.err
M=sm__inst_executed_pipe_alu.sum,sm__inst_executed_pipe_fma.sum,sm__inst_executed.sum,dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,l1tex__t_sectors_pipe_lsu_mem_local_op_ld.sum,sm__warps_active.avg.pct_of_peak_sustained_active
timeout 600 ncu --metrics $M --clock-control none -k regex:"k_flat_pair|k_fact_gv|k_fact_dp" --csv --log-file gpurun_out/inst_c2.csv python scripts/profile_target.py c2 > /dev/null 2>&1
timeout 600 ncu --metrics $M --clock-control none -k regex:"k_flat_pair|k_fact_gv|k_fact_dp" --csv --log-file gpurun_out/inst_c4.csv python scripts/profile_target.py c4 > /dev/null 2>&1
tail -3 gpurun_out/pytest_gpu.log; head -c 600 gpurun_out/bench.json; tail -3 gpurun_out/bench.err
