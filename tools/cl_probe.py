import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle
import paper_conf_icpp_kasagini14_b200 as libsat
from sat_inputs import make_np
n, m = int(sys.argv[1]), int(sys.argv[2])
a = make_np(n, m, "int32", "u32", seed=5)
libsat.lib.sat_debug_diag_enable()
try:
    y = libsat.sat(torch.from_numpy(a).cuda(), tile_rows=64).cpu().numpy()
    ref = oracle.sat(a)
    bad = np.argwhere(y != ref)
    print(n, m, "grid", libsat.last_grid(), "wrong", len(bad), bad[:3].tolist())
except Exception as e:
    print(n, m, "failed", str(e)[:60])
    libsat.lib.sat_debug_diag_dump()
