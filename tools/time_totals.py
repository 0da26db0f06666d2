"""Kernel-only timing of sat_column_totals (the sharded path's extra strip
read): median of CUDA-event launches, L2 flushed before each.

python tools/time_totals.py rows cols [dtype] [reps]
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import paper_conf_icpp_kasagini14_b200 as libsat
from sat_inputs import make_torch

rows, cols = int(sys.argv[1]), int(sys.argv[2])
dtype = sys.argv[3] if len(sys.argv) > 3 else "int32"
reps = int(sys.argv[4]) if len(sys.argv) > 4 else 20
x = make_torch(rows, cols, dtype, "u32" if dtype == "int32" else "unit", seed=1, device="cuda")
out = torch.empty(cols, dtype=x.dtype, device="cuda")
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
libsat.column_totals(x, out=out)
ts = []
for _ in range(reps):
    flush.fill_(1)
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    libsat.column_totals(x, out=out)
    e.record()
    e.synchronize()
    ts.append(s.elapsed_time(e))
ts.sort()
ms = ts[len(ts) // 2]
print(f"column_totals {rows}x{cols} {dtype}: {ms:.4f} ms {x.numel() * x.element_size() / ms / 1e6:.0f} GB/s (read)")
