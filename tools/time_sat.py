"""Kernel-only timing of one 1R1W shape: median of reps CUDA-event launches,
L2 flushed before each.  One line per call: shape dtype th grid ms GB/s.

python tools/time_sat.py rows cols dtype [tile_rows] [reps] [batch] [segments]
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import paper_conf_icpp_kasagini14_b200 as libsat
from sat_inputs import make_torch

rows, cols, dtype = int(sys.argv[1]), int(sys.argv[2]), sys.argv[3]
th = int(sys.argv[4]) if len(sys.argv) > 4 else 0
reps = int(sys.argv[5]) if len(sys.argv) > 5 else 20
batch = int(sys.argv[6]) if len(sys.argv) > 6 and sys.argv[6] != "0" else None
seg = int(sys.argv[7]) if len(sys.argv) > 7 else 0
x = make_torch(rows, cols, dtype, "u32" if dtype == "int32" else "unit", seed=1, batch=batch,
               device="cuda")
y = torch.empty_like(x)
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
run = (lambda: libsat.sat(x, out=y, tile_rows=th, segments=seg)) if batch is None else \
    (lambda: libsat.sat_batched(x, out=y, tile_rows=th, segments=seg))
for _ in range(3):
    run()
ts = []
for _ in range(reps):
    flush.fill_(1)
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    run()
    e.record()
    e.synchronize()
    ts.append(s.elapsed_time(e))
ts.sort()
ms = ts[len(ts) // 2]
nb = 2 * x.numel() * x.element_size()
env = f"segments={seg}"
print(f"{rows}x{cols}{'x' + str(batch) if batch else ''} {dtype} th={libsat.last_tile_rows()} "
      f"grid={libsat.last_grid()} {ms:.4f} ms {nb / ms / 1e6:.0f} GB/s [{env}]", flush=True)
