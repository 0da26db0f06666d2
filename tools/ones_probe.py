"""All-ones closed-form check of 1R1W over shapes / tile heights / segment
counts / in place, reporting the first wrong (row, col) per case.

python tools/ones_probe.py
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import paper_conf_icpp_kasagini14_b200 as libsat

cases = [(8192, 8192), (32768, 8192), (65536, 4096), (16384, 65536), (65536, 16384)]
for rows, cols in cases:
    ii = torch.arange(1, rows + 1, device="cuda", dtype=torch.int64).view(-1, 1)
    jj = torch.arange(1, cols + 1, device="cuda", dtype=torch.int64).view(1, -1)
    for th in (64, 128):
        for seg in (1, 4, 16):
            for inplace in (False, True):
                x = torch.ones(rows, cols, dtype=torch.int32, device="cuda")
                try:
                    y = libsat.sat(x, out=x if inplace else None, tile_rows=th, segments=seg)
                    torch.cuda.synchronize()
                except Exception as e:
                    print(rows, cols, th, seg, inplace, "ERROR", e, flush=True)
                    sys.exit(1)
                bad = None
                for r0 in range(0, rows, 4096):
                    ref = ((ii[r0:r0 + 4096] * jj) % (1 << 32)).to(torch.int64)
                    got = y[r0:r0 + 4096].to(torch.int64) % (1 << 32)
                    d = (got != ref).nonzero()
                    if len(d):
                        bad = (int(d[0, 0]) + r0, int(d[0, 1]), len(d))
                        break
                print(rows, cols, "th", th, "seg", seg, "inplace", inplace, "grid", libsat.last_grid(),
                      "OK" if bad is None else f"BAD first {bad}", flush=True)
                del x, y
