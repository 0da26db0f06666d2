"""Tuning sweep of the column-walk box filter's rows per unit (DESIGN.md
Sec. 4.12): 32 x 1080x1920, CUDA events, median of reps, L2 flushed.

python tools/box_rows.py "32,64,96,128" [radius ...]
"""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import paper_conf_icpp_kasagini14_b200 as libsat
from sat_inputs import make_torch

rbs = [int(v) for v in sys.argv[1].split(",")]
radii = [int(v) for v in sys.argv[2:]] or [4]
B, n, m = 32, 1080, 1920
u8 = make_torch(n, m, "int32", "u8", seed=5, batch=B, device="cuda").to(torch.uint8)
i32 = make_torch(n, m, "int32", "u32", seed=6, batch=B, device="cuda")
out = torch.empty(B, n, m, dtype=torch.int32, device="cuda")
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
for r in radii:
    for name, x in (("u8", u8), ("int32", i32)):
        for rb in rbs:
            libsat.set_box_rows(rb)
            libsat.box_filter(x, r, r, out=out)
            ts = []
            for _ in range(15):
                flush.fill_(1)
                s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                s.record()
                libsat.box_filter(x, r, r, out=out)
                e.record()
                e.synchronize()
                ts.append(s.elapsed_time(e))
            print(f"{name} r={r} rb={rb} {statistics.median(ts):.4f} ms", flush=True)
libsat.set_box_rows(0)
