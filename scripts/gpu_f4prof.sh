#!/bin/bash
# closed-loop evidence: launch list and full capture of the chain path's kernel on f4; per-scenario costs
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_f4.csv \
    python scripts/profile_target.py f4 > /dev/null 2>&1; echo "list f4 rc=$?"
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"k_chain|k_ep_count" -c 2 \
    -o gpurun_out/full_f4 -f python scripts/profile_target.py f4 > /dev/null 2>&1; echo "full f4 rc=$?"
timeout 1500 python scripts/scenario_costs.py > gpurun_out/scenario_costs.json 2> gpurun_out/scenario_costs.err; echo "costs rc=$?"
