"""PCIe ceilings for the end-to-end path: pinned H2D alone, D2H alone, both
at once (separate streams), and sat_host at several strip counts.

python tools/pcie_probe.py [rows] [cols]
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import paper_conf_icpp_kasagini14_b200 as libsat

rows = int(sys.argv[1]) if len(sys.argv) > 1 else 32768
cols = int(sys.argv[2]) if len(sys.argv) > 2 else 32768
hin = torch.empty(rows, cols, dtype=torch.int32, pin_memory=True)
hout = torch.empty_like(hin, pin_memory=True)
d = torch.empty(rows, cols, dtype=torch.int32, device="cuda")
d2 = torch.empty_like(d)
nb = hin.numel() * 4
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()


def timed(fn, reps=3):
    fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(reps):
        fn()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / reps


def both():
    ev = torch.cuda.Event()
    ev.record()
    s1.wait_event(ev)
    s2.wait_event(ev)
    with torch.cuda.stream(s1):
        d.copy_(hin, non_blocking=True)
    with torch.cuda.stream(s2):
        hout.copy_(d2, non_blocking=True)
    torch.cuda.current_stream().wait_stream(s1)
    torch.cuda.current_stream().wait_stream(s2)


t = timed(lambda: d.copy_(hin, non_blocking=True))
print(f"H2D alone  {t:.1f} ms  {nb / t / 1e6:.1f} GB/s")
t = timed(lambda: hout.copy_(d2, non_blocking=True))
print(f"D2H alone  {t:.1f} ms  {nb / t / 1e6:.1f} GB/s")
t = timed(both)
print(f"H2D+D2H concurrent  {t:.1f} ms  {nb / t / 1e6:.1f} GB/s per direction")
t = timed(lambda: libsat.sat_host(hin, hout))
print(f"sat_host (32 strips)  {t:.1f} ms  {rows * cols / t / 1e6:.3e} elem/s")
