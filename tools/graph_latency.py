"""Per-call time of sat() eager vs replayed from a CUDA graph (DESIGN.md
Sec. 4: the device-side ticket base).  Three arms per size, CUDA events on the
launching stream, back-to-back calls:
  eager      host counter base (a workspace never captured)
  eager_dev  the same stream after a capture: +1-2 small kernels per call
  graph      G calls captured in one graph, replayed
python tools/graph_latency.py  -> one JSON line per size"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import paper_conf_icpp_kasagini14_b200 as libsat
from sat_inputs import make_torch

N, G = 200, 20


def timed(fn, s, reps):
    with torch.cuda.stream(s):
        for _ in range(5):
            fn()
    s.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(s)
    with torch.cuda.stream(s):
        for _ in range(reps):
            fn()
    b.record(s)
    b.synchronize()
    return a.elapsed_time(b) / reps


for n, m, dt in [(1024, 1024, "int32"), (4096, 4096, "float32"), (16384, 16384, "int32")]:
    x = make_torch(n, m, dt, "u32" if dt == "int32" else "unit", seed=1, device="cuda")
    y = torch.empty_like(x)
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    eager = timed(lambda: libsat.sat(x, out=y, stream=s1), s1, N)
    with torch.cuda.stream(s2):
        libsat.sat(x, out=y)
    s2.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s2):
        for _ in range(G):
            libsat.sat(x, out=y)
    graph = timed(g.replay, s2, N // G) / G
    eager_dev = timed(lambda: libsat.sat(x, out=y, stream=s2), s2, N)
    print(json.dumps({"rows": n, "cols": m, "dtype": dt, "eager_us": round(1e3 * eager, 2),
                      "eager_dev_epoch_us": round(1e3 * eager_dev, 2), "graph_us": round(1e3 * graph, 2)}))
