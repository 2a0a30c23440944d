#!/bin/bash
# chain path: variant timings (normal build), then the per-phase cycle breakdown (PX_CHAIN_DEBUG build)
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
NOTEST=1 bash scripts/gpu_chain.sh "$@"
PROTEUS_BUILD_DEFS=-DPX_CHAIN_DEBUG python -c "from paper_conf_asplos_ahmadgfwsw24_b200 import build as b; print(b.build())" >> gpurun_out/build.log 2>&1
PROTEUS_LIB=$PWD/paper_conf_asplos_ahmadgfwsw24_b200/libproteus_dbg.so \
  timeout 300 python scripts/replay_variants.py ${DBGVAR:-dbg=PROTEUS_REPLAY_CHAIN=1,PROTEUS_REPLAY_CHAIN_MINBATCH=0} > /dev/null 2> gpurun_out/chain_dbg.err
grep "chain" gpurun_out/chain_dbg.err | head -30
