"""Randomised parity sweep (development): random shapes, dtypes, band heights,
look-back groups, segments, publication jitter, batches, variants and box
filters, each checked against the CPU oracle.  Runs for --seconds, prints one
line per failure and a summary.

python tools/fuzz.py [--seconds 300] [--seed 1]
"""
import argparse
import os
import random
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import oracle
import paper_conf_icpp_kasagini14_b200 as libsat
from sat_inputs import make_np


def same(got, ref, dtype):
    if dtype in ("int32", "float64"):
        return np.array_equal(got, ref)            # int32 exact; float64 inputs are dyadic
    return oracle.max_rel_err(got, ref) <= 1e-5


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--seconds", type=float, default=300)
    ap.add_argument("--seed", type=int, default=1)
    args = ap.parse_args()
    rng = random.Random(args.seed)
    t_end = time.time() + args.seconds
    n = fails = 0
    while time.time() < t_end:
        kind = rng.choice(["sat", "sat", "sat", "batched", "variant", "box"])
        rows = rng.choice([1, 7, 64, 129, 300, 1000, 2047, 4096, rng.randint(1, 5000)])
        cols = rng.choice([1, 4, 100, 128, 515, 1920, 2048, 4100, rng.randint(1, 5000)])
        if rows * cols > 12_000_000:
            continue
        dtype = rng.choice(["int32", "float32", "float64"])
        dist = "u32" if dtype == "int32" else "unit"
        seed = rng.randint(0, 1 << 30)
        desc = ""
        try:
            if kind == "sat":
                a = make_np(rows, cols, dtype, dist, seed=seed)
                kw = dict(tile_rows=rng.choice([0, 16, 32, 64, 128]),
                          segments=rng.choice([0, 0, 1, 2, 3, 5]),
                          lookback_group=rng.choice([0, 0, -1, 2, 3, 4, 8]),
                          jitter=rng.choice([0, 0, 0, 5000, 20000]))
                desc = f"sat {rows}x{cols} {dtype} {kw}"
                got = libsat.sat(torch.from_numpy(a).cuda(), **kw).cpu().numpy()
                ok = same(got, oracle.sat(a), dtype)
            elif kind == "batched":
                b = rng.randint(1, 6)
                if b * rows * cols > 12_000_000:
                    continue
                a = make_np(b * rows, cols, dtype, dist, seed=seed).reshape(b, rows, cols)
                kw = dict(tile_rows=rng.choice([0, 32, 64, 128]), segments=rng.choice([0, 0, 2, 3]),
                          lookback_group=rng.choice([0, -1, 4]))
                desc = f"batched {b}x{rows}x{cols} {dtype} {kw}"
                got = libsat.sat_batched(torch.from_numpy(a).cuda(), **kw).cpu().numpy()
                ok = all(same(got[i], oracle.sat(a[i]), dtype) for i in range(b))
            elif kind == "variant":
                v = rng.choice(["2r2w", "2r1w", "1+rr1w", "4r4w"])
                if dtype == "float64" and v == "4r4w":
                    dtype, dist = "int32", "u32"
                a = make_np(rows, cols, dtype, dist, seed=seed)
                kw = dict(r=rng.choice([0.0, 0.1, 0.25, 0.5]))
                desc = f"{v} {rows}x{cols} {dtype} {kw}"
                got = libsat.sat(torch.from_numpy(a).cuda(), variant=v, **kw).cpu().numpy()
                ok = same(got, oracle.sat(a), dtype)
            else:
                b = rng.randint(1, 3)
                if b * rows * cols > 6_000_000:
                    continue
                src = rng.choice(["u8", "int32", "float32"])
                rr, rc = rng.choice([0, 1, 4, 8, 16, 40]), rng.choice([0, 1, 4, 33, 63, 64, 127, 200])
                if src == "u8":
                    a = make_np(b * rows, cols, "int32", "u8", seed=seed).astype(np.uint8).reshape(b, rows, cols)
                    got = libsat.box_filter(torch.from_numpy(a).cuda(), rr, rc).cpu().numpy()
                    ok = all(np.array_equal(got[i], oracle.box_filter(a[i].astype(np.int32), rr, rc))
                             for i in range(b))
                elif src == "int32":
                    a = make_np(b * rows, cols, "int32", "u32", seed=seed).reshape(b, rows, cols)
                    got = libsat.box_filter(torch.from_numpy(a).cuda(), rr, rc).cpu().numpy()
                    ok = all(np.array_equal(got[i], oracle.box_filter(a[i], rr, rc)) for i in range(b))
                else:
                    a = make_np(b * rows, cols, "float32", "unit", seed=seed).reshape(b, rows, cols)
                    got = libsat.box_filter(torch.from_numpy(a).cuda(), rr, rc).cpu().numpy()
                    ok = all(np.array_equal(got[i], oracle.box_filter(a[i], rr, rc).astype(np.float32))
                             for i in range(b))
                desc = f"box {src} {b}x{rows}x{cols} rr={rr} rc={rc} launches={libsat.last_launch_count()}"
        except Exception as e:          # noqa: BLE001 -- reported, then the sweep goes on
            ok = False
            desc += f" raised {type(e).__name__}: {e}"
        n += 1
        if not ok:
            fails += 1
            print("FAIL", desc, flush=True)
    print(f"fuzz: {n} cases, {fails} failures", flush=True)
    return 1 if fails else 0


if __name__ == "__main__":
    sys.exit(main())
