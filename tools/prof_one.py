"""Run one workload a few times (for ncu captures).

python tools/prof_one.py cfg3b [tile_rows] [reps] [variant]
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import paper_conf_icpp_kasagini14_b200 as libsat
from sat_inputs import make_torch
from bench import CONFIGS

cfg = sys.argv[1] if len(sys.argv) > 1 else "cfg3b"
th = int(sys.argv[2]) if len(sys.argv) > 2 else 0
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 3
variant = sys.argv[4] if len(sys.argv) > 4 else None
rows, cols, batch, dtype, v, _ = CONFIGS[cfg]
variant = variant or v
x = make_torch(rows, cols, dtype, "u32" if dtype == "int32" else "unit", seed=1, batch=batch,
               device="cuda")
y = torch.empty_like(x)
torch.cuda.synchronize()
for _ in range(reps):
    if batch is None:
        libsat.sat(x, variant=variant, out=y, tile_rows=th)
    else:
        libsat.sat_batched(x, variant=variant, out=y, tile_rows=th)
torch.cuda.synchronize()
print("done", cfg, variant, libsat.last_tile_rows())
