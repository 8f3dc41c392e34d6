#!/bin/bash
# n = 4032 cluster variants: reg slots x reduction rounds
OUT=gpurun_out; mkdir -p $OUT; : > $OUT/cluster_sweep.txt
for cfg in "4 3" "2 3" "2 2" "0 2"; do set -- $cfg
  BSOLVE_CLUSTER_ROUNDS=$2 timeout 300 python - "$1" "$2" >> $OUT/cluster_sweep.txt 2>&1 <<'PY'
import sys, json, numpy as np, torch
sys.path.insert(0, '.')
import xgcgen as X
from paper_conf_ipps_kashinksla22_b200 import Solver
kr, rd = int(sys.argv[1]), int(sys.argv[2])
pat = X.stencil_pattern(64, 63); B = X.make_batch(0, 16384, pattern=pat)
S = Solver(pat.row_ptr, pat.col_idx, 16384, reg_slots=kr)
v = torch.from_numpy(S.ell_values(B.values)).cuda(); b = torch.from_numpy(B.b).cuda(); o = S.alloc_outputs()
for _ in range(2): S.run(v, b, out=o)
torch.cuda.synchronize(); ts = []
for _ in range(5):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(); S.run(v, b, out=o); e1.record(); torch.cuda.synchronize(); ts.append(e0.elapsed_time(e1))
ms = sorted(ts)[2]; it = o[1].cpu().numpy(); st = o[3].cpu().numpy()
print(f"kreg={kr} rounds={rd}: {16384/ms*1e3/1e6:.3f} Msys/s  {ms:.2f} ms  iters {it.mean():.2f}  conv {np.all(st==0)}")
PY
done
