"""A/B of 1R1W band configurations (development): for each config
(tile_rows, segments) first a parity gate against the CPU oracle on a
3000 x 4096 int32 matrix, then kernel-only timing of each shape (median of
reps CUDA-event launches, L2 flushed before each), configs interleaved in
rounds to cancel clock drift.

python tools/ab_sat.py "16384x16384,65536x65536" "128:0,64:0" [reps] [rounds] [dtype]

A config is th:seg[:hg], hg = sat_options.lookback_group (0 automatic, -1 flat,
n >= 2 groups of n bands).
"""
import ctypes
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import oracle
import paper_conf_icpp_kasagini14_b200 as libsat
from sat_inputs import make_np, make_torch

shapes = [tuple(int(v) for v in s.split("x")) for s in sys.argv[1].split(",")]   # n x m, or batch x n x m
cfgs = [tuple(int(v) for v in (c + ":0").split(":")[:3]) for c in sys.argv[2].split(",")]
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 10
rounds = int(sys.argv[4]) if len(sys.argv) > 4 else 3
dtype = sys.argv[5] if len(sys.argv) > 5 else "int32"
dist = "u32" if dtype == "int32" else "unit"

def call(x, y, c):
    """c = (tile_rows, segments, lookback_group)"""
    o = libsat.options(tile_rows=c[0], segments=c[1], lookback_group=c[2])
    if x.dim() == 3:
        libsat._check(libsat._lib.sat_compute_batched(x.data_ptr(), y.data_ptr(), x.shape[0], x.shape[1], x.shape[2],
                                                      libsat._dtype_code(x), 2, ctypes.byref(o), None))
    else:
        libsat._check(libsat._lib.sat_compute_ex(x.data_ptr(), y.data_ptr(), x.shape[0], x.shape[1],
                                                 libsat._dtype_code(x), 2, ctypes.byref(o), None))
    return y


ok = {}
a = make_np(3000, 4096, dtype, dist, seed=5)
ref = oracle.sat(a)
xa = torch.from_numpy(a).cuda()
for c in cfgs:
    got = torch.empty_like(xa)
    call(xa, got, c)
    got = got.cpu().numpy()
    th, seg = c[0], c[1]
    ok[c] = bool(np.array_equal(got, ref)) if dtype == "int32" else oracle.max_rel_err(got, ref) <= 1e-5
    print(f"parity th={th} seg={seg}: {ok[c]} (th used {libsat.last_tile_rows()})", flush=True)

flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")


for shp in shapes:
    bt, (n, m) = (shp[0], shp[1:]) if len(shp) == 3 else (None, shp)
    x = make_torch(n, m, dtype, dist, seed=1, device="cuda", batch=bt)
    y = torch.empty_like(x)
    res = {c: [] for c in cfgs}
    for c in cfgs:
        for _ in range(2):
            call(x, y, c)
    for _ in range(rounds):
        for c in cfgs:
            for _ in range(reps):
                flush.fill_(1)
                s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                s.record()
                call(x, y, c)
                e.record()
                e.synchronize()
                res[c].append(s.elapsed_time(e))
    nb = 2 * x.numel() * x.element_size()
    for c in cfgs:
        ms = statistics.median(res[c])
        print(f"{'x'.join(map(str, shp))} {dtype} th={c[0]} seg={c[1]} x={c[2]} median {ms:.4f} ms min {min(res[c]):.4f} "
              f"{nb / ms / 1e6:.0f} GB/s frac {nb / ms / 1e6 / 6550.1:.3f} parity={ok[c]}", flush=True)
    del x, y
    torch.cuda.empty_cache()
