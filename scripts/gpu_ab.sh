#!/bin/bash
# A/B of compile-time variants of the flat kernel: c2 step and one-vector time per variant
# usage: bash scripts/gpu_ab.sh "-DFLAT_WAGG=0" "-DFLAT_SDIG=0" ...   ("" = defaults)
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
i=0
for defs in "$@"; do
  i=$((i+1))
  if [ -z "$defs" ]; then lib=$PWD/paper_conf_asplos_ahmadgfwsw24_b200/libproteus.so; else
    PROTEUS_BUILD_DEFS="$defs" python -c "from paper_conf_asplos_ahmadgfwsw24_b200 import build as b; b.build(force=True)" >> gpurun_out/build.log 2>&1
    cp paper_conf_asplos_ahmadgfwsw24_b200/libproteus_dbg.so /tmp/ab_$i.so; lib=/tmp/ab_$i.so; fi
  for rep in 1 2; do
    echo "== variant [$defs] rep $rep"
    PROTEUS_LIB=$lib timeout 120 python scripts/solve_overhead.py 2>&1 | grep -E "step ms|score_flat"
  done
done
