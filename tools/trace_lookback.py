"""Record per-(band, chunk) look-back event times of one 1R1W launch.

python tools/trace_lookback.py rows cols tile_rows out.npz [segments] [batch] [lookback_group]
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import paper_conf_icpp_kasagini14_b200 as libsat
from sat_inputs import make_torch

rows, cols, th = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3])
out = sys.argv[4]
seg = int(sys.argv[5]) if len(sys.argv) > 5 else 0
batch = (int(sys.argv[6]) or None) if len(sys.argv) > 6 else None
x = make_torch(rows, cols, "int32", "u32", seed=1, device="cuda", batch=batch)
y = torch.empty_like(x)
hg = int(sys.argv[7]) if len(sys.argv) > 7 else 0       # sat_options.lookback_group


def run():
    import ctypes
    o = libsat.options(tile_rows=th, segments=seg, lookback_group=hg)
    if batch is None:
        libsat._check(libsat._lib.sat_compute_ex(x.data_ptr(), y.data_ptr(), rows, cols, libsat._dtype_code(x), 2,
                                                 ctypes.byref(o), None))
    else:
        libsat._check(libsat._lib.sat_compute_batched(x.data_ptr(), y.data_ptr(), batch, rows, cols,
                                                      libsat._dtype_code(x), 2, ctypes.byref(o), None))
for _ in range(3):
    run()
nb, nc = (batch or 1) * ((rows + th - 1) // th), (cols + 127) // 128
buf = torch.zeros(nb * nc * 8, dtype=torch.int64, device="cuda")
torch.cuda.synchronize()
s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
libsat.debug_trace(buf)
s.record()
run()
e.record()
torch.cuda.synchronize()
print("ms", s.elapsed_time(e), "th", libsat.last_tile_rows(), "grid", libsat.last_grid())
np.savez_compressed(out, trace=buf.cpu().numpy().reshape(nb, nc, 8), ms=s.elapsed_time(e))
