#!/bin/bash
# per-lane k_stitch counters on c5 (PX_STITCH_DEBUG build): lanes slower than $1 cycles
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
PROTEUS_BUILD_DEFS=-DPX_STITCH_DEBUG python -c "from paper_conf_asplos_ahmadgfwsw24_b200 import build as b; print(b.build())" > gpurun_out/build_dbg.log 2>&1
for kind in poisson gamma; do
PROTEUS_LIB=$PWD/paper_conf_asplos_ahmadgfwsw24_b200/libproteus_dbg.so PROTEUS_REPLAY_DEBUG=${1:-3000000} KIND=$kind \
  timeout 300 python -c "
import os, sys
sys.path.insert(0, os.getcwd())
import torch
from paper_conf_asplos_ahmadgfwsw24_b200 import Proteus, workloads as W
px = Proteus(0)
cfg = W.config('c5', kind=os.environ['KIND'])
prof, cl = cfg['prof'], cfg['cluster']
px.load_profiles(prof)
sol = px.solve(cl.device_type, cl.slo_us, cfg['demand'], mode=2)[0]
arr = torch.from_numpy(cfg['arrival_us']).cuda(); fam = torch.from_numpy(cfg['family']).cuda()
sc = cfg['scenarios']
lat = torch.empty((len(sc), len(arr)), dtype=torch.uint32, device='cuda')
px.replay(arr, fam, sol.option, sol.z, cl.device_type, cfg['demand'][0], cl.slo_us, sc, latency=lat)
torch.cuda.synchronize()
" > gpurun_out/stitch_dbg_$kind.log 2>&1
echo "$kind rc=$?"; grep -c "^stitch" gpurun_out/stitch_dbg_$kind.log
done
