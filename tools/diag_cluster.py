"""Run one 1R1W launch with the spin diagnostics armed; dump them on failure."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import paper_conf_icpp_kasagini14_b200 as libsat
from sat_inputs import make_torch

n, m, th = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3])
x = make_torch(n, m, "int32", "u32", seed=1, device="cuda")
torch.cuda.synchronize()
libsat.lib.sat_debug_diag_enable()
try:
    y = libsat.sat(x, tile_rows=th)
    torch.cuda.synchronize()
    print("ok grid", libsat.last_grid())
except Exception as e:
    print("failed:", str(e)[:80])
print("records:", libsat.lib.sat_debug_diag_dump(), flush=True)
