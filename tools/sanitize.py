"""Small-shape workload for compute-sanitizer (memcheck / racecheck /
synccheck / initcheck): every variant and dtype, band segments and the unit
queue (many short units), seeded and sharded entry points, widening inputs,
the fused box filter -- each checked against the oracle so a sanitizer run is
also a parity run.

compute-sanitizer --tool memcheck python tools/sanitize.py
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import oracle
import paper_conf_icpp_kasagini14_b200 as libsat
from sat_inputs import make_np


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def check(got, ref, dtype):
    got = got.cpu().numpy()
    if dtype in ("int32", "float64"):
        assert np.array_equal(got, ref), "mismatch"
    else:
        assert oracle.max_rel_err(got, ref) <= 1e-5


n_calls = 0
for dtype in ("int32", "float32", "float64"):
    dist = "u32" if dtype == "int32" else "unit"
    for shape in [(70, 300), (257, 129), (130, 516)]:
        a = make_np(*shape, dtype, dist, seed=shape[0])
        ref = oracle.sat(a)
        for variant in ("1r1w", "2r2w", "2r1w", "1+rr1w", "4r4w"):
            for th in (0, 16, 64, 128):
                check(libsat.sat(dev(a), variant=variant, tile_rows=th), ref, dtype)
                n_calls += 1
        check(libsat.sat(dev(a), tile_rows=16, segments=3), ref, dtype)      # segments + unit queue
        check(libsat.sat(dev(a), tile_rows=16, force_generic=True), ref, dtype)
        r0 = shape[0] // 3
        if dtype == "int32":
            carry = oracle.column_totals(a[:r0])
        else:
            carry = a[:r0].astype(np.float64).sum(axis=0).astype(a.dtype)
        check(libsat.sat_seeded(dev(a[r0:]), carry_row=dev(carry)), ref[r0:], dtype)
        n_calls += 3
# sharded ABI, 3 virtual ranks
a = make_np(300, 260, "int32", "u32", seed=9)
ref = oracle.sat(a)
bounds = [(0, 100), (100, 180), (180, 300)]
strips = [dev(a[r0:r1]) for r0, r1 in bounds]
totals = [libsat.column_totals(s) for s in strips]
totals[-1] = torch.zeros_like(totals[-1])
outs = []
for p in range(3):
    def ag(send, recv):
        torch.cuda.synchronize()
        recv.copy_(torch.stack(totals))
    o, _ = libsat.sat_sharded_abi(strips[p], p, 3, ag)
    outs.append(o.cpu().numpy())
assert np.array_equal(np.concatenate(outs), ref)
# widening + fused box filter
u8 = make_np(130, 320, "int32", "u8", seed=4, batch=2).astype(np.uint8)
y = libsat.sat_widening(dev(u8), torch.int32).cpu().numpy()
for b in range(2):
    assert np.array_equal(y[b], oracle.sat(u8[b].astype(np.int32)))
bx = libsat.box_filter(dev(u8), 4, 5).cpu().numpy()
for b in range(2):
    assert np.array_equal(bx[b], oracle.box_filter(u8[b].astype(np.int32), 4, 5))
f = make_np(100, 200, "float32", "unit", seed=5)
assert np.array_equal(libsat.box_filter(dev(f), 3, 3, out_dtype=torch.float64).cpu().numpy(),
                      oracle.box_filter(f, 3, 3))
torch.cuda.synchronize()
print(f"sanitize workload ok ({n_calls} SAT calls + sharded, widening, box filter)", flush=True)
