#!/bin/bash
# n = 4032 cluster plans: TMEM values vs register/SMEM values
OUT=gpurun_out; mkdir -p $OUT; : > $OUT/cluster_sweep.txt
for ct in 1 0; do
  BSOLVE_CLUSTER_TMEM=$ct timeout 300 python - $ct >> $OUT/cluster_sweep.txt 2>&1 <<'PY'
import sys, numpy as np, torch
sys.path.insert(0, '.')
import xgcgen as X
from paper_conf_ipps_kashinksla22_b200 import Solver
pat = X.stencil_pattern(64, 63); B = X.make_batch(0, 16384, pattern=pat)
S = Solver(pat.row_ptr, pat.col_idx, 16384)
v = torch.from_numpy(S.ell_values(B.values)).cuda(); b = torch.from_numpy(B.b).cuda(); o = S.alloc_outputs()
for _ in range(2): S.run(v, b, out=o)
torch.cuda.synchronize(); ts = []
for _ in range(5):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(); S.run(v, b, out=o); e1.record(); torch.cuda.synchronize(); ts.append(e0.elapsed_time(e1))
ms = sorted(ts)[2]; it = o[1].cpu().numpy(); st = o[3].cpu().numpy()
print(f"cluster tmem={sys.argv[1]}: {16384/ms*1e3/1e6:.3f} Msys/s  {ms:.2f} ms  iters {it.mean():.2f}  conv {np.all(st==0)}")
PY
done
