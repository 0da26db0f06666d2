"""Repeat 1R1W on one input and report mismatches vs the oracle per tile height.

python tools/stress.py rows cols reps [tile_rows ...]
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import oracle
import paper_conf_icpp_kasagini14_b200 as libsat
from sat_inputs import make_np

rows, cols, reps = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3])
ths = [int(t) for t in sys.argv[4:]] or [16, 32, 48, 64]
a = make_np(rows, cols, "int32", "u32", seed=9)
ref = oracle.sat(a)
x = torch.from_numpy(a).cuda()
for th in ths:
    bad = 0
    for r in range(reps):
        y = libsat.sat(x, tile_rows=th).cpu().numpy()
        d = np.argwhere(y != ref)
        if len(d):
            bad += 1
            i0, j0 = d[0]
            rws = np.unique(d[:, 0] // th)
            chs = np.unique(d[:, 1] // 128)
            print(f"th={th} rep={r}: {len(d)} wrong; first ({i0},{j0}); bands {rws[:10]}... ({len(rws)}) chunks {chs[:10]}... ({len(chs)})")
            # is the error a constant per column within a band (carry) or per element?
            b = rws[0]
            blk = (y.astype(np.int64) - ref.astype(np.int64))[b * th:(b + 1) * th]
            print("   diff rows of first bad band constant per column:", bool((blk == blk[0:1]).all()))
    print(f"th={th}: {bad}/{reps} runs wrong", flush=True)
