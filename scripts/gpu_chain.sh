#!/bin/bash
# chain-path pass: c5 timing of path variants (checksums), then the replay parity tests
# usage: bash scripts/gpu_chain.sh [variant ...]   (scripts/replay_variants.py syntax)
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 600 python scripts/replay_variants.py "$@" > gpurun_out/chain_var.json 2> gpurun_out/chain_var.err; echo "variants rc=$?" >> gpurun_out/chain_var.err
python -c "
import json; d=json.load(open('gpurun_out/chain_var.json'))
for k,v in d.items():
    print(k, 'same' if v['same'] else 'DIFFER', {n:(round(r['ms'],2), {a:round(b,2) for a,b in r['split'].items() if b>0.1}) for n,r in v.items() if n!='same'})
"
if [ -z "$NOTEST" ]; then
timeout 1500 python -m pytest tests/test_gpu_replay.py tests/test_gpu_goldens.py -x -q -k "not c2 and not c4" > gpurun_out/pytest_chain.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_chain.log
tail -15 gpurun_out/pytest_chain.log
fi
tail -3 gpurun_out/chain_var.err
