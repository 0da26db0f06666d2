"""Multi-GPU row-strip partitioner (north star (3)).

One process per GPU.  Rank p owns rows [r0(p), r1(p)) x all cols of one
global matrix.  The exchange step is a single all-gather of m-length vectors:

  1. colsum_p = column totals of the strip (the extra strip read, one launch;
     the last rank skips it and sends zeros -- nobody consumes its totals);
  2. all-gather colsum over the process group (NCCL over NVLink/NVSwitch on
     GPUs; gloo in the CPU tests);
  3. + 4. seeded local 1R1W SAT of the strip whose band 0 adds
     carry_p = sum_{q<p} colsum_q (q ascending) to its first row: the
     exclusive scan over ranks runs inside the SAT kernel (one launch).

Rank 0's carry is zero, so its SAT does not wait for the all-gather: the
collective runs on a side stream while the SAT runs on the caller's.

The per-rank compute steps are libsat kernels (``CudaOps``).  ``ops`` is
injectable so that the orchestration (partition, exchange, ordering) can be
tested with world_size 2 on CPU/gloo without a GPU.
"""
from __future__ import annotations

import torch
import torch.distributed as dist


def partition_rows(n: int, nranks: int, rank: int, last_weight: float = 1.0):
    """Row range of ``rank``.  ``last_weight`` > 1 gives the last rank more rows
    (it skips the totals pass, SURVEY 8.4 load balance: with 1.5 every rank
    moves about the same bytes, 3 units per row for ranks < P-1 and 2 for the
    last); 1.0 = equal strips."""
    if nranks < 1 or not (0 <= rank < nranks):
        raise ValueError("bad rank / nranks")
    total_w = (nranks - 1) + last_weight
    base = n / total_w
    bounds = [0]
    for p in range(nranks - 1):
        bounds.append(min(n, int(round(base * (p + 1)))))
    bounds.append(n)
    return bounds[rank], bounds[rank + 1]


class CudaOps:
    """Per-rank steps on libsat's CUDA kernels."""

    def __init__(self):
        from . import column_totals, sat_seeded
        self._totals, self._seeded = column_totals, sat_seeded

    def column_totals(self, strip, out=None):
        return self._totals(strip, out=out)

    def seeded_sat(self, strip, gathered, rank, out=None):
        if gathered is None or rank == 0:
            return self._seeded(strip, out=out)
        return self._seeded(strip, gathered=gathered, rank=rank, out=out)


class RowStripSAT:
    """This rank's end of the row-strip sharded SAT, with its exchange
    buffers allocated once (``send``: cols, ``gathered``: P x cols)."""

    def __init__(self, cols: int, dtype, device=None, group=None, ops=None, host_exchange=None):
        """``host_exchange``: all-gather through host memory (gloo process
        groups, e.g. several processes sharing one GPU in tests); default:
        when the group is gloo and the buffers live on a GPU."""
        self.group = group
        on_gpu = device is not None and torch.device(device).type == "cuda"
        if host_exchange is None:
            host_exchange = on_gpu and dist.get_backend(group) == "gloo"
        self.host_exchange = host_exchange
        self.rank = dist.get_rank(group)
        self.P = dist.get_world_size(group)
        self.cols = int(cols)
        self.ops = ops or CudaOps()
        self.send = torch.zeros(self.cols, dtype=dtype, device=device)
        self.flat = torch.empty(self.P * self.cols, dtype=dtype, device=device)
        self.gathered = self.flat.view(self.P, self.cols)
        if host_exchange:
            self.flat_h = torch.empty(self.P * self.cols, dtype=dtype)
        self.side = None
        if self.P > 1 and self.rank == 0 and self.send.is_cuda and not host_exchange:
            self.side = torch.cuda.Stream(device=self.send.device)

    def __call__(self, strip, out=None, events=None):
        """SAT rows of this rank's strip.  ``events`` (optional dict of CUDA
        events "t0", "totals", "gather", "sat") brackets the steps for a
        breakdown.  Returns (out, stats)."""
        rows, cols = strip.shape
        assert cols == self.cols
        eb = strip.element_size()
        ev = events or {}
        if "t0" in ev:
            ev["t0"].record()
        if self.P > 1:
            if self.rank < self.P - 1 and rows > 0:
                self.ops.column_totals(strip, out=self.send)
            if "totals" in ev:
                ev["totals"].record()
            if self.host_exchange:
                dist.all_gather_into_tensor(self.flat_h, self.send.cpu(), group=self.group)
                self.flat.copy_(self.flat_h)
                if "gather" in ev:
                    ev["gather"].record()
                out = self.ops.seeded_sat(strip, self.gathered, self.rank, out=out)
            elif self.side is not None:
                # rank 0: its SAT does not need the gather; the collective
                # runs beside it on a side stream
                cur = torch.cuda.current_stream()
                self.side.wait_stream(cur)
                with torch.cuda.stream(self.side):
                    dist.all_gather_into_tensor(self.flat, self.send, group=self.group)
                out = self.ops.seeded_sat(strip, None, 0, out=out)
                if "gather" in ev:
                    ev["gather"].record()
                cur.wait_stream(self.side)
            else:
                dist.all_gather_into_tensor(self.flat, self.send, group=self.group)
                if "gather" in ev:
                    ev["gather"].record()
                out = self.ops.seeded_sat(strip, self.gathered, self.rank, out=out)
        else:
            if "totals" in ev:
                ev["totals"].record()
            if "gather" in ev:
                ev["gather"].record()
            out = self.ops.seeded_sat(strip, None, 0, out=out)
        if "sat" in ev:
            ev["sat"].record()
        stats = dict(strip_bytes_read=rows * cols * eb, strip_bytes_written=rows * cols * eb,
                     extra_bytes_read=(rows * cols * eb if (self.P > 1 and self.rank < self.P - 1) else 0),
                     allgather_bytes=(self.P * cols * eb if self.P > 1 else 0))
        return out, stats


_CACHE = {}


def sharded_sat(strip: torch.Tensor, group=None, ops=None, out=None, timings=None):
    """SAT rows of this rank's strip of the global matrix (see module doc).

    Buffers are cached per (group, cols, dtype, device).  Returns
    ``(out, stats)``; stats counts the bytes each step moved.
    """
    key = (id(group), strip.shape[1], strip.dtype, str(strip.device), id(ops) if ops else None)
    r = _CACHE.get(key)
    if r is None:
        r = _CACHE[key] = RowStripSAT(strip.shape[1], strip.dtype, strip.device, group, ops)
    return r(strip, out=out, events=timings)


def make_peer_exchange(cols: int, dtype, group=None, device=None, ipc=None, factory=None):
    """Set up this rank's fused peer exchange.

    Every rank allocates a zeroed mailbox on its GPU, publishes its CUDA IPC
    handle with one ``all_gather_object`` (set-up only, not per call) and maps
    the other ranks' mailboxes.  ``ipc`` = (get_handle, open) and ``factory``
    (the PeerExchange constructor) are injectable so the set-up can be tested
    on CPU with gloo.  Returns ``(exchange, peer_ptrs)``.
    """
    from . import PeerExchange, ipc_handle, ipc_open
    get_handle, open_handle = ipc or (ipc_handle, ipc_open)
    factory = factory or PeerExchange
    rank = dist.get_rank(group)
    P = dist.get_world_size(group)
    nbytes = PeerExchange.mailbox_bytes(cols, P, dtype) if factory is PeerExchange else 4096
    mailbox = torch.zeros(nbytes, dtype=torch.uint8, device=device)
    handles = [None] * P
    dist.all_gather_object(handles, get_handle(mailbox), group=group)
    ptrs = [mailbox.data_ptr() if q == rank else open_handle(handles[q]) for q in range(P)]
    ex = factory(rank, P, cols, dtype, mailbox, ptrs)
    # every rank's mailbox is zeroed before any rank's first call
    dist.barrier(group=group)
    return ex, ptrs
