"""Bandwidth ceilings for the band access pattern (1 GPU).

python tools/pattern_probe.py N [tile_rows]
Times (CUDA events, median of reps): torch copy of an N x N int32 matrix,
1R1W, 2R2W (col pass + row pass), and prints GB/s of each.
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import paper_conf_icpp_kasagini14_b200 as libsat
from sat_inputs import make_torch

n = int(sys.argv[1])
th = int(sys.argv[2]) if len(sys.argv) > 2 else 0
x = make_torch(n, n, "int32", "u32", seed=1, device="cuda")
y = torch.empty_like(x)
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")


def timeit(fn, reps=20):
    ts = []
    for i in range(reps + 3):
        flush.zero_()
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record()
        fn()
        e.record()
        torch.cuda.synchronize()
        if i >= 3:
            ts.append(s.elapsed_time(e))
    ts.sort()
    return ts[len(ts) // 2]


B = n * n * 4
for name, fn, nbytes in [
    ("copy", lambda: y.copy_(x), 2 * B),
    ("1r1w", lambda: libsat.sat(x, out=y, tile_rows=th), 2 * B),
    ("2r2w", lambda: libsat.sat(x, variant="2r2w", out=y, tile_rows=th), 4 * B),
    ("2r1w", lambda: libsat.sat(x, variant="2r1w", out=y, tile_rows=th), 3 * B),
]:
    ms = timeit(fn)
    print(f"{name:6s} n={n} th={libsat.last_tile_rows()} grid={libsat.last_grid()} {ms:.4f} ms {nbytes / ms / 1e6:.1f} GB/s")
