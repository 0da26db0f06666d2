"""Throughput of the SAT's consumers and widening inputs on
the image workload of BASELINE config 5 (per GPU: 32 images of 1080 x 1920).

python tools/bench_box.py [--images 32] [--radius 4] [--reps 20]

Lines (JSON): widening 1R1W uint8 -> int32 (1 + 4 B per pixel), float32 ->
float64 (4 + 8 B), the box filter from uint8 pixels (SAT pass 1 + 4 B, box
pass 4 + 4 B: 13 B per pixel in round 1; the fused kernel moves 1 x (1 +
2r/TH) + 4 B), and
rectangle-sum queries (random rectangles over the same images).  CUDA events
around each call, median of --reps, a 512 MB L2 flush before each; bytes are
algorithmic; peak = MEASURED_PEAKS.json hbm_gbs.
"""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_icpp_kasagini14_b200 as libsat  # noqa: E402
from sat_inputs import make_torch  # noqa: E402


def timed(fn, reps, flush):
    ts = []
    for _ in range(reps):
        flush.fill_(1)
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record()
        fn()
        e.record()
        e.synchronize()
        ts.append(s.elapsed_time(e))
    return statistics.median(ts)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--images", type=int, default=32)
    ap.add_argument("--radius", type=int, default=4)
    ap.add_argument("--reps", type=int, default=20)
    args = ap.parse_args()
    peak = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"]
    B, n, m, r = args.images, 1080, 1920, args.radius
    px = B * n * m
    flush = torch.empty(512 * 2**20 // 4, dtype=torch.int32, device="cuda")
    u8 = make_torch(n, m, "int32", "u8", seed=5, batch=B, device="cuda").to(torch.uint8)
    f32 = make_torch(n, m, "float32", "unit", seed=6, batch=B, device="cuda")
    i32 = torch.empty(B, n, m, dtype=torch.int32, device="cuda")
    f64 = torch.empty(B, n, m, dtype=torch.float64, device="cuda")
    box = torch.empty(B, n, m, dtype=torch.int32, device="cuda")
    f32o = torch.empty(B, n, m, dtype=torch.float32, device="cuda")
    rects = torch.stack([torch.randint(0, B, (1 << 20,)), torch.randint(0, n, (1 << 20,)),
                         torch.randint(0, m, (1 << 20,)), torch.randint(0, n, (1 << 20,)),
                         torch.randint(0, m, (1 << 20,))], 1).to(torch.int32).cuda()
    rects[:, 1], rects[:, 3] = torch.minimum(rects[:, 1], rects[:, 3]), torch.maximum(rects[:, 1], rects[:, 3])
    rects[:, 2], rects[:, 4] = torch.minimum(rects[:, 2], rects[:, 4]), torch.maximum(rects[:, 2], rects[:, 4])
    qout = torch.empty(1 << 20, dtype=torch.int32, device="cuda")
    cases = [
        ("widen u8->i32 1R1W", lambda: libsat.sat_widening(u8, torch.int32, out=i32), 5 * px, px),
        ("widen f32->f64 1R1W", lambda: libsat.sat_widening(f32, torch.float64, out=f64), 12 * px, px),
        ("sat i32 1R1W (same images)", lambda: libsat.sat_batched(i32, out=box), 8 * px, px),
        # column walk (sat_boxw.cuh, rc <= 63): input (1 + 2r/64) x eb_in (row-block warm-up), 4 B out
        (f"box filter u8 r={r} walk (1 B in x (1 + 2r/64) + 4 B out)", lambda: libsat.box_filter(u8, r, r, out=box),
         int((1 + 2 * r / 64) * px) + 4 * px, px),
        (f"box filter f32->f32 r={r} walk (float64 sums)", lambda: libsat.box_filter(f32, r, r, out=f32o),
         int(4 * (1 + 2 * r / 64) * px) + 4 * px, px),
        (f"box filter int32 r={r} walk (4 B in x (1 + 2r/64) + 4 B out)", lambda: libsat.box_filter(i32, r, r, out=box),
         int(4 * (1 + 2 * r / 64) * px) + 4 * px, px),
        # band kernel with the SAT on chip (sat_boxf.cuh) for 64 <= rc < 128
        (f"box filter u8 rr={r} rc=100 fused band (1 B in x (1 + 2r/32) + 4 B out)",
         lambda: libsat.box_filter(u8, r, 100, out=box), int((1 + 2 * r / 32) * px) + 4 * px, px),
        ("rect sums (1M queries)", lambda: libsat.rect_sums(i32, rects, out=qout), None, 1 << 20),
    ]
    for name, fn, nbytes, units in cases:
        fn()
        torch.cuda.synchronize()
        ms = timed(fn, args.reps, flush)
        line = {"case": name, "images": B, "shape": [n, m], "ms": round(ms, 4),
                "units_per_s": units / (ms / 1e3), "launches": libsat.last_launch_count()}
        if nbytes:
            line["alg_bytes"] = nbytes
            line["GB/s"] = round(nbytes / (ms / 1e3) / 1e9, 1)
            line["frac_of_peak"] = round(nbytes / (ms / 1e3) / 1e9 / peak, 4)
        print(json.dumps(line), flush=True)


if __name__ == "__main__":
    main()
