"""Host-side cost of one sat() call vs its GPU time (small sizes are
launch-bound).  python tools/host_overhead.py [n]"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import paper_conf_icpp_kasagini14_b200 as libsat
from sat_inputs import make_torch

n = int(sys.argv[1]) if len(sys.argv) > 1 else 1024
x = make_torch(n, n, "int32", "u32", seed=1, device="cuda")
y = torch.empty_like(x)
for _ in range(10):
    libsat.sat(x, out=y)
torch.cuda.synchronize()
N = 200
t0 = time.perf_counter()
for _ in range(N):
    libsat.sat(x, out=y)
t1 = time.perf_counter()
torch.cuda.synchronize()
t2 = time.perf_counter()
s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
s.record()
for _ in range(N):
    libsat.sat(x, out=y)
e.record()
torch.cuda.synchronize()
print(f"n={n}: host enqueue {1e6 * (t1 - t0) / N:.1f} us/call, wall incl. drain {1e6 * (t2 - t0) / N:.1f} us/call, "
      f"back-to-back GPU {1e3 * s.elapsed_time(e) / N:.1f} us/call")
