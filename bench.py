#!/usr/bin/env python
"""bench.py -- libsat throughput on B200 (driver contract).

Default workload (BASELINE.json config 4, the one the metric "... at
1/2/4/8 B200" is quoted on; it fits one GPU): the SAT of one 65536 x 65536
int32 matrix (uint32 wrapping arithmetic), 1R1W.  At N=1 one GPU computes it
with one kernel launch per step; at N>1 the matrix is split into N row strips
(one per rank, the last one 1.5x as tall: it skips the totals pass) and each
step is: column totals (one launch) -> NCCL all-gather -> seeded 1R1W whose
band 0 does the rank exclusive scan (one launch); rank 0's SAT does not wait
for the gather (strong scaling: total work fixed).

Timing: W untimed warm-up steps, then exactly K steps bracketed by barrier +
cuda synchronize, CUDA events on the launching stream, max over ranks.  Inputs
(16 GiB) are far larger than L2 (126 MB), so no flush is needed; configs whose
working set is < 4 x L2 (cfg1, cfg2, cfg5) write a 2 x L2 buffer between steps
(the hot, un-flushed number is reported beside it).
`--impl reference` times the CPU oracle (the reference arm of this tier).
Other BASELINE configs: `--config cfg1|cfg2|cfg3|cfg3b|cfg4|cfg5`.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

BASELINE_METRIC = "SAT elements/sec and % of HBM roofline (1R1W bytes) at 1/2/4/8 B200"

CONFIGS = {
    # name: (rows, cols, batch, dtype, variant, description)
    "cfg1": (1024, 1024, None, "int32", "1r1w", "cfg1: 1024x1024 int32 SAT, 1R1W"),
    "cfg2": (4096, 4096, None, "float32", "1r1w", "cfg2: 4096x4096 float32 SAT"),
    "cfg3": (18432, 18432, None, "int32", "1r1w", "cfg3: 18432x18432 int32 SAT, 1R1W"),
    "cfg3b": (16384, 16384, None, "int32", "1r1w", "cfg3': 16384x16384 int32 SAT, 1R1W (north-star gate)"),
    "cfg4": (65536, 65536, None, "int32", "1r1w",
             "cfg4: 65536x65536 int32 SAT, row strips over N GPUs, 1R1W"),
    "cfg5": (1080, 1920, 32, "float32", "1r1w",
             "cfg5: 32 images/GPU x 1080x1920 float32 SATs (data parallel)"),
}


def log(*a):
    print(*a, file=sys.stderr, flush=True)


# ------------------------------------------------------------------ clocks
REASON_BITS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap",
               0x8: "hw_slowdown", 0x10: "sync_boost", 0x20: "sw_thermal_slowdown",
               0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown",
               0x100: "display_clocks_setting"}


class ClockSampler:
    """nvidia-smi sampled every 100 ms during the timed region."""

    def __init__(self, gpu_index: int):
        self.gpu = gpu_index
        self.proc = None
        self.lines = []

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.gpu),
                 "--query-gpu=clocks.sm,clocks.max.sm,clocks_event_reasons.active",
                 "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def __exit__(self, *exc):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()

    def summary(self):
        sm, mx, reasons = [], [], set()
        for ln in self.lines:
            parts = [p.strip() for p in ln.split(",")]
            if len(parts) < 3:
                continue
            try:
                sm.append(float(parts[0]))
                mx.append(float(parts[1]))
                bits = int(parts[2], 16)
            except ValueError:
                continue
            for b, name in REASON_BITS.items():
                if bits & b:
                    reasons.add(name)
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"], "samples": 0}
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": max(mx),
                "reasons": sorted(reasons), "samples": len(sm)}


# ------------------------------------------------------------------ helpers
def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured"
    return 6650.0, "fallback"


def ncu_traffic(workload_key: str, kernel_regex: str = "sat_band_kernel"):
    """Per-launch DRAM bytes of the dominant kernel from the committed ncu
    summary (profiles/ncu_summary.json), or None."""
    p = os.path.join(ROOT, "profiles", "ncu_summary.json")
    if not os.path.exists(p):
        return None
    with open(p) as f:
        d = json.load(f)
    e = d.get(workload_key)
    if not e:
        return None
    return e.get("dram_bytes_per_launch")


def cpu_model():
    try:
        with open("/proc/cpuinfo") as f:
            for ln in f:
                if ln.startswith("model name"):
                    return ln.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def oracle_leg(x, y, dtype: str, budget_s: float = 25.0):
    """CPU oracle (single-threaded C, as it stands) streamed over the bench
    workload ``x`` in row strips (D2H copies outside the clock), and checked
    against the GPU result ``y`` strip by strip: a parity check of the timed
    launch configuration at full size.  Stops after ``budget_s`` seconds of
    oracle time.  Returns (elements/s, elements, seconds, parity_ok, max_err)."""
    import numpy as np
    import oracle
    oracle.build()
    imgs = x.view(-1, x.shape[-2], x.shape[-1])
    outs = y.view(-1, y.shape[-2], y.shape[-1])
    cols = imgs.shape[2]
    step = max(1, (1 << 26) // cols)                 # 256 MiB strips
    secs, n_el, ok, err = 0.0, 0, True, 0.0
    for b in range(imgs.shape[0]):
        st = oracle.Stream(cols, dtype == "int32")
        for r0 in range(0, imgs.shape[1], step):
            a = imgs[b, r0:r0 + step].cpu().numpy()
            t0 = time.perf_counter()
            ref = st.feed(a)
            secs += time.perf_counter() - t0
            n_el += a.size
            got = outs[b, r0:r0 + step].cpu().numpy()
            if dtype == "int32":
                ok = ok and bool(np.array_equal(got, ref))
            else:
                e = oracle.max_rel_err(got, ref)
                err = max(err, e)
                ok = ok and e <= 1e-5
            if secs >= budget_s:
                return n_el / secs, n_el, secs, ok, err
    return n_el / secs, n_el, secs, ok, err


# ------------------------------------------------------------------ reference arm
def run_reference(args, cfg_key):
    rows, cols, batch, dtype, variant, desc = CONFIGS[cfg_key]
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    import numpy as np
    import oracle
    from sat_inputs import make_np
    oracle.build()
    # each step: the oracle on a bounded sample (full width, `srows` rows)
    srows = max(1, min(rows, (1 << 24) // cols))
    x = make_np(srows, cols, dtype, "u32" if dtype == "int32" else "unit", seed=1)
    for _ in range(args.warmup):
        oracle.sat(x)
    times = []
    for _ in range(args.steps):
        t0 = time.perf_counter()
        oracle.sat(x)
        times.append(time.perf_counter() - t0)
    tot = sum(times)
    elems = srows * cols
    value = elems * args.steps / tot
    line = {
        "impl": "reference", "metric": BASELINE_METRIC, "value": value, "unit": "elem/s",
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": 1000 * tot / args.steps, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "u32" if dtype == "int32" else "f64",
        "data": "synthetic", "config": {"workload": desc + " [oracle sample]"},
        "cpu_baseline": {"value": value, "unit": "elem/s", "cores": 1, "kind": "oracle",
                         "sample": f"{srows} rows x {cols} cols per step (first rows of the workload)",
                         "cpu": cpu_model()},
        "e2e": {"value": value, "unit": "elem/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
        "gpu_launches": 0,
    }
    print(json.dumps(line), flush=True)
    return 0


# ------------------------------------------------------------------ our arm
def _coll(fn, t, *a, **k):
    """A small collective on a CUDA tensor; through host memory when the
    process group is gloo (multi-process tests sharing one GPU)."""
    import torch.distributed as dist
    if dist.get_backend() == "gloo" and t.is_cuda:
        h = t.cpu()
        fn(h, *a, **k)
        t.copy_(h)
    else:
        fn(t, *a, **k)

def strip_parity(x, y, dtype, r0, rows_above_gen, check_rows=256):
    """Parity of this rank's strip (first ``check_rows`` rows) against the CPU
    oracle streamed from the column sums of every row above the strip.  Those
    sums are computed with torch (int64 / float64 accumulation of the seeded
    generator's rows, independent of libsat), the strip rows by the oracle."""
    import numpy as np
    import torch
    import oracle
    cols = x.shape[1]
    acc = torch.zeros(cols, dtype=torch.int64 if dtype == "int32" else torch.float64, device=x.device)
    step = max(1, (1 << 27) // cols)
    for a in range(0, r0, step):
        blk = rows_above_gen(a, min(r0, a + step))
        acc += blk.to(acc.dtype).sum(dim=0)
    st = oracle.Stream(cols, dtype == "int32")
    if dtype == "int32":
        st.colsum[:] = (acc % (1 << 32)).cpu().numpy().astype(np.uint32)
    else:
        st.colsum[:] = acc.cpu().numpy()
    n = min(check_rows, x.shape[0])
    ref = st.feed(x[:n].cpu().numpy())
    got = y[:n].cpu().numpy()
    if dtype == "int32":
        return bool(np.array_equal(got, ref))
    return bool(oracle.max_rel_err(got, ref) <= 1e-5)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=None)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="cfg4", choices=sorted(CONFIGS))
    ap.add_argument("--variant", default=None)
    ap.add_argument("--tile-rows", type=int, default=0)
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--flush-l2", default="auto", choices=["auto", "on", "off"],
                    help="write a 2 x L2 buffer between timed steps (auto: when the working set < 4 x L2)")
    ap.add_argument("--last-weight", type=float, default=1.5,
                    help="N>1 row strips: the last rank's share (it skips the totals pass)")
    ap.add_argument("--dist-backend", default="nccl", choices=["nccl", "gloo"],
                    help="N>1 process group (gloo: host-memory exchange, for multi-process tests on one GPU)")
    ap.add_argument("--exchange", default="nccl", choices=["nccl", "libsat-nccl", "fused"],
                    help="N>1 row strips: NCCL all-gather via torch.distributed (with the step breakdown), "
                         "the C-ABI call with libsat's own NCCL communicator (sat_compute_sharded_nccl), "
                         "or the fused peer exchange (IPC mailboxes)")
    args = ap.parse_args()
    if args.warmup < 3:
        ap.error("--warmup must be >= 3")
    cfg_key = args.config
    rows, cols, batch, dtype, variant, desc = CONFIGS[cfg_key]
    if args.variant:
        variant = args.variant
    if args.steps is None:
        args.steps = {"cfg1": 2000, "cfg2": 1000, "cfg3": 300, "cfg3b": 400, "cfg4": 200,
                      "cfg5": 500}[cfg_key]
    if args.impl == "reference":
        return run_reference(args, cfg_key)

    import torch
    import torch.distributed as dist
    import paper_conf_icpp_kasagini14_b200 as libsat
    from paper_conf_icpp_kasagini14_b200.dist import partition_rows
    from sat_inputs import make_torch

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus:
        log(f"warning: --gpus {args.gpus} but WORLD_SIZE {world}")
    # --dist-backend gloo lets the N>1 path run as several processes sharing
    # fewer GPUs (tests on a one-GPU box); the driver's runs use NCCL
    gpu = local % max(1, torch.cuda.device_count())
    torch.cuda.set_device(gpu)
    if world > 1:
        if args.dist_backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", gpu))
        else:
            dist.init_process_group("gloo")
    dev = torch.device("cuda", gpu)
    stream = torch.cuda.current_stream()
    tdt = torch.int32 if dtype == "int32" else torch.float32
    dist_name = "u32" if dtype == "int32" else "unit"
    eb = 4
    l2_bytes = torch.cuda.get_device_properties(dev).L2_cache_size

    # ---------------- per-rank work unit
    r0, r1 = 0, rows
    if batch is None:
        if world > 1:
            r0, r1 = partition_rows(rows, world, rank, args.last_weight)
        x = make_torch(r1 - r0, cols, dtype, dist_name, seed=4001, row0=r0, device=dev)
        y = torch.empty_like(x)
        my_elems = (r1 - r0) * cols
        total_elems = rows * cols
        scaling = "strong"
    else:
        # data parallel images: `batch` images per GPU (weak scaling)
        x = make_torch(rows, cols, dtype, dist_name, seed=5001 + rank, batch=batch, device=dev)
        y = torch.empty_like(x)
        my_elems = batch * rows * cols
        total_elems = my_elems * world
        scaling = "weak"
    sharded = world > 1 and batch is None
    opts = dict(tile_rows=args.tile_rows) if args.tile_rows else {}
    flush = args.flush_l2 == "on" or (args.flush_l2 == "auto" and 2 * my_elems * eb < 4 * l2_bytes)
    flushbuf = torch.empty(2 * l2_bytes, dtype=torch.uint8, device=dev) if flush else None

    launches = [0]
    breakdown = None
    # kernel events: (start, end) around the band kernel of each step
    if sharded and args.exchange == "fused":
        from paper_conf_icpp_kasagini14_b200.dist import make_peer_exchange
        xchg, _ = make_peer_exchange(cols, tdt, device=dev)

        def step(ev=None):
            if ev:
                ev[0].record(stream)
            xchg.sat(x, out=y)
            if ev:
                ev[1].record(stream)
            launches[0] += libsat.last_launch_count()
    elif sharded and args.exchange == "libsat-nccl":
        # one C-ABI call per step: column totals, ncclAllGather on libsat's
        # communicator, seeded SAT (the events bracket the whole call)
        uid = [libsat.nccl_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(uid, src=0)
        ncomm = libsat.NcclComm(uid[0], rank, world)

        def step(ev=None):
            if ev:
                ev[0].record(stream)
            libsat.sat_sharded_nccl(x, ncomm, variant=variant, out=y)
            if ev:
                ev[1].record(stream)
            launches[0] += libsat.last_launch_count()
    elif sharded:
        from paper_conf_icpp_kasagini14_b200.dist import RowStripSAT
        op = RowStripSAT(cols, tdt, device=dev, host_exchange=args.dist_backend != "nccl")
        breakdown = {"totals_ms": [], "gather_ms": [], "sat_ms": []}
        step_events = []

        def step(ev=None):
            e = None
            if ev:
                e = {k: torch.cuda.Event(enable_timing=True) for k in ("t0", "totals", "gather", "sat")}
                if rank == 0:
                    e.pop("gather")
                step_events.append(e)
            op(x, out=y, events=e)
            n = 1 + (1 if rank < world - 1 else 0)
            launches[0] += n
            if ev:
                # the band kernel: after the gather (ranks > 0), right after the totals (rank 0)
                ev[0] = e["gather"] if "gather" in e else e["totals"]
                ev[1] = e["sat"]
    else:
        def step(ev=None):
            if ev:
                ev[0].record(stream)
            if batch is None:
                libsat.sat(x, variant=variant, out=y, **opts)
            else:
                libsat.sat_batched(x, variant=variant, out=y, **opts)
            if ev:
                ev[1].record(stream)
            launches[0] += libsat.last_launch_count()

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    # ---------------- warm-up + quick parity re-check of the timed path
    for _ in range(args.warmup):
        step()
    barrier()
    parity = None
    if not sharded and rank == 0:
        import numpy as np
        import oracle

        def same(got, ref):
            return bool(np.array_equal(got, ref)) if dtype == "int32" else \
                bool(oracle.max_rel_err(got, ref) <= 1e-5)
        if batch is None:
            srow = min(r1 - r0, 256)
            parity = same(y[:srow].cpu().numpy(), oracle.sat(x[:srow].cpu().numpy()))
        else:
            # first and last image of the batch, whole
            parity = all(same(y[i].cpu().numpy(), oracle.sat(x[i].cpu().numpy()))
                         for i in (0, batch - 1))
    elif sharded:
        # every rank: the first 256 rows of its strip against the oracle
        # seeded with the column sums of all rows above it
        ok = strip_parity(x, y, dtype, r0,
                          lambda a, b: make_torch(b - a, cols, dtype, dist_name, seed=4001, row0=a,
                                                  device=dev))
        t = torch.tensor([0 if ok else 1], device=dev)
        _coll(dist.all_reduce, t)
        parity = {"ranks_checked": world, "rows_per_rank": 256, "ok": int(t.item()) == 0}

    # ---------------- timed region
    def timed(flush_between):
        launches[0] = 0
        if breakdown is not None:
            step_events.clear()
        ev0 = torch.cuda.Event(enable_timing=True)
        ev1 = torch.cuda.Event(enable_timing=True)
        kev = [[torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)]
               for _ in range(args.steps)]
        barrier()
        ev0.record(stream)
        for i in range(args.steps):
            if flush_between:
                flushbuf.zero_()
            step(kev[i])
        ev1.record(stream)
        barrier()
        kern_ms = [a.elapsed_time(b) for a, b in kev]
        return ev0.elapsed_time(ev1), kern_ms

    with ClockSampler(gpu) as clk:
        time.sleep(0.3)                     # let the sampler start
        ms_local, kern_ms = timed(flush)
    clocks = clk.summary()
    tile_rows = libsat.last_tile_rows()
    step_launches = launches[0]
    if flush:
        # the flush writes sit between steps: the step time is the band
        # kernel's event time (one launch per step at N = 1)
        ms_local = sum(kern_ms)
    if breakdown is not None:
        for e in step_events:
            breakdown["totals_ms"].append(e["t0"].elapsed_time(e["totals"]))
            if "gather" in e:
                breakdown["gather_ms"].append(e["totals"].elapsed_time(e["gather"]))
                breakdown["sat_ms"].append(e["gather"].elapsed_time(e["sat"]))
            else:
                breakdown["sat_ms"].append(e["totals"].elapsed_time(e["sat"]))
    t = torch.tensor([ms_local, statistics.mean(kern_ms)], dtype=torch.float64, device=dev)
    if world > 1:
        _coll(dist.all_reduce, t, op=dist.ReduceOp.MAX)
    ms_total, kern_avg_ms = float(t[0]), float(t[1])
    ms_per_step = ms_total / args.steps
    value = total_elems * args.steps / (ms_total / 1e3)
    hot = None
    if flush and not sharded:
        hot_ms, hot_k = timed(False)
        hot = {"value": total_elems * args.steps / (hot_ms / 1e3), "unit": "elem/s",
               "ms_per_step": hot_ms / args.steps, "kernel_ms": statistics.mean(hot_k),
               "l2": "no flush between steps (inputs may be L2-resident)"}

    # ---------------- roofline of the dominant kernel (the band kernel)
    peak, peak_kind = measured_peaks()
    alg_bytes = 2 * eb * my_elems                      # 1R1W: one read + one write
    if variant == "2r2w":
        alg_bytes = 4 * eb * my_elems
    elif variant == "2r1w":
        alg_bytes = 3 * eb * my_elems
    elif variant == "1+rr1w":                          # (2 + r_eff) eb, Theorem 7
        alg_bytes = int((2 + libsat.last_r_effective()) * eb * my_elems)
    elif variant == "4r4w":                            # four read+write passes, Lemma 3
        alg_bytes = 8 * eb * my_elems
    elif variant == "4r1w":                            # Formula (1): 4 reads + 1 write, Lemma 5
        alg_bytes = 5 * eb * my_elems
    mine = torch.tensor([alg_bytes / (statistics.mean(kern_ms) / 1e3) / 1e9], dtype=torch.float64, device=dev)
    if world > 1:
        _coll(dist.all_reduce, mine, op=dist.ReduceOp.MIN)    # the slowest rank's band kernel
    achieved = float(mine[0])
    traffic = ncu_traffic(f"{cfg_key}:{variant}:n{world}")
    roofline = {"bound": "hbm", "achieved": round(achieved, 1), "peak": peak, "unit": "GB/s",
                "frac": round(achieved / peak, 4), "traffic": traffic,
                "peak_kind": peak_kind, "kernel": "sat_band_kernel",
                "alg_bytes_per_launch": alg_bytes, "kernel_ms": round(kern_avg_ms, 4),
                "frac_of_8TBs": round(achieved / 8000.0, 4)}
    if world > 1:
        roofline["note"] = "min over ranks of the band kernel's 1R1W byte rate on its own strip"

    # ---------------- end to end through the public API from pinned host memory
    e2e = None
    if not args.no_e2e:
        e2e = run_e2e(args, libsat, x, rows, cols, batch, dtype, world, rank, dev, sharded,
                      total_elems, barrier)

    # ---------------- CPU oracle baseline (rank 0, N=1 only) + full-size parity
    cpu = None
    full_parity = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        rate, n_el, secs, ok, err = oracle_leg(x, y, dtype)
        whole = n_el == x.numel()
        cpu = {"value": rate, "unit": "elem/s", "cores": 1, "kind": "oracle",
               "sample": (f"the whole workload ({n_el} elements)" if whole else
                          f"the first {n_el} elements of the workload in row order")
                         + f", {secs:.1f} s of single-threaded C (streaming column/row prefix), "
                           "D2H copies excluded",
               "cpu": cpu_model(), "host_cores": os.cpu_count()}
        full_parity = {"elements": n_el, "ok": ok,
                       "rule": "bit-exact" if dtype == "int32" else "max rel err <= 1e-5",
                       "max_rel_err": err if dtype != "int32" else None}

    bd = None
    if breakdown is not None:
        vals = torch.tensor([statistics.mean(breakdown["totals_ms"]),
                             statistics.mean(breakdown["gather_ms"]) if breakdown["gather_ms"] else 0.0,
                             statistics.mean(breakdown["sat_ms"])], dtype=torch.float64, device=dev)
        src = vals.cpu() if args.dist_backend == "gloo" else vals
        allv = [torch.zeros_like(src) for _ in range(world)]
        dist.all_gather(allv, src)
        allv = [a.cpu() for a in allv]
        bd = {"per_rank_ms": [[round(float(v), 4) for v in a.tolist()] for a in allv],
              "columns": ["totals (extra read)", "all-gather wait", "seeded SAT (band kernel)"],
              "rows": [list(partition_rows(rows, world, p, args.last_weight)) for p in range(world)]}

    if rank == 0:
        line = {
            "metric": BASELINE_METRIC, "value": value, "unit": "elem/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_per_step,
            "higher_is_better": True, "scaling": scaling, "vs_baseline": None,
            "dtype": "u32" if dtype == "int32" else "f32",
            "data": "synthetic (splitmix64 counter hash: uniform 32-bit int / dyadic [0,1) float)",
            "config": {"workload": desc + (f" [{variant}]" if variant != "1r1w" else ""),
                       "rows": rows, "cols": cols, "batch": batch,
                       "parallelism": (f"row-strips x{world} ({args.exchange} exchange, last weight "
                                       f"{args.last_weight})" if sharded else
                                       (f"dp{world}" if world > 1 else "1 GPU")),
                       "l2": ("flushed: a 2 x L2 buffer written between steps; the step time is the "
                              "band kernel's event time" if flush else "inputs > 4 x L2, no flush"),
                       "tile_rows": tile_rows},
            "roofline": roofline,
            "cpu_baseline": cpu,
            "e2e": e2e,
            "gpu_launches": step_launches,
            "clocks": clocks,
            "parity_recheck": parity,
            "parity_full": full_parity,
        }
        if hot:
            line["hot"] = hot
        if bd:
            line["breakdown"] = bd
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0


def run_e2e(args, libsat, x, rows, cols, batch, dtype, world, rank, dev, sharded,
            total_elems, barrier):
    """Same metric through the public API with host buffers: H2D of the step's
    input from pinned memory, the SAT, D2H of the result, all timed."""
    import torch
    import torch.distributed as dist
    steps = max(1, args.e2e_steps)
    try:
        hin = torch.empty(x.shape, dtype=x.dtype, pin_memory=True)
        hout = torch.empty(x.shape, dtype=x.dtype, pin_memory=True)
    except RuntimeError as e:
        return {"value": None, "unit": "elem/s", "error": f"pinned alloc failed: {e}"}
    hin.copy_(x.cpu() if x.numel() * 4 < (1 << 31) else x.to("cpu"))
    nbytes = x.numel() * x.element_size()
    if not sharded and batch is None:
        def step():
            libsat.sat_host(hin, hout)
    elif batch is not None:
        dx = torch.empty_like(x)
        dy = torch.empty_like(x)

        def step():
            dx.copy_(hin, non_blocking=True)
            libsat.sat_batched(dx, out=dy)
            hout.copy_(dy, non_blocking=True)
            torch.cuda.current_stream().synchronize()
    else:
        from paper_conf_icpp_kasagini14_b200.dist import sharded_sat
        dx = torch.empty_like(x)
        dy = torch.empty_like(x)

        def step():
            dx.copy_(hin, non_blocking=True)
            sharded_sat(dx, out=dy)
            hout.copy_(dy, non_blocking=True)
            torch.cuda.current_stream().synchronize()
    step()                                           # warm
    barrier()
    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    ev0.record()
    for _ in range(steps):
        step()
    ev1.record()
    barrier()
    ms = torch.tensor([ev0.elapsed_time(ev1)], dtype=torch.float64, device=dev)
    if world > 1:
        _coll(dist.all_reduce, ms, op=dist.ReduceOp.MAX)
    ms = float(ms[0])
    return {"value": total_elems * steps / (ms / 1e3), "unit": "elem/s",
            "h2d_bytes_per_step": nbytes, "d2h_bytes_per_step": nbytes, "steps": steps,
            "ms_per_step": ms / steps, "api": "sat_host (pinned)" if (not sharded and batch is None)
            else "copy + public API + copy"}


if __name__ == "__main__":
    sys.exit(main())
