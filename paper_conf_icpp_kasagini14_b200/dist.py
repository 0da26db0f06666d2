"""Multi-GPU row-strip partitioner (north star (3)).

One process per GPU.  Rank p owns rows [r0(p), r1(p)) x all cols of one
global matrix.  The exchange step is a single all-gather of m-length vectors:

  1. colsum_p = column totals of the strip (the extra strip read; the last
     rank skips it and sends zeros -- nobody consumes its totals);
  2. all-gather colsum over the process group (NCCL over NVLink/NVSwitch on
     GPUs; gloo in the CPU tests);
  3. carry_p = sum_{q<p} colsum_q (fixed q order);
  4. seeded local 1R1W SAT of the strip.

The per-rank compute steps are libsat kernels (``CudaOps``).  ``ops`` is
injectable so that the orchestration (partition, exchange, ordering) can be
tested with world_size 2 on CPU/gloo without a GPU.
"""
from __future__ import annotations

import torch
import torch.distributed as dist


def partition_rows(n: int, nranks: int, rank: int, last_weight: float = 1.0):
    """Row range of ``rank``.  ``last_weight`` > 1 gives the last rank more rows
    (it skips the totals pass, SURVEY 8.4 load balance); 1.0 = equal strips."""
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
        from . import column_totals, rank_exscan, sat_seeded
        self._totals, self._exscan, self._seeded = column_totals, rank_exscan, sat_seeded

    def column_totals(self, strip):
        return self._totals(strip)

    def exscan(self, gathered, rank):
        return self._exscan(gathered, rank)

    def seeded_sat(self, strip, carry, out=None):
        return self._seeded(strip, carry_row=carry, out=out)


def sharded_sat(strip: torch.Tensor, group=None, ops=None, out=None, timings=None):
    """SAT rows of this rank's strip of the global matrix (see module doc).

    Returns ``(out, stats)``; stats counts the bytes each step moved.
    """
    ops = ops or CudaOps()
    rank = dist.get_rank(group)
    P = dist.get_world_size(group)
    rows, cols = strip.shape
    eb = strip.element_size()
    if P > 1:
        if rank < P - 1 and rows > 0:
            send = ops.column_totals(strip)
        else:
            send = torch.zeros(cols, dtype=strip.dtype, device=strip.device)
        flat = torch.empty(P * cols, dtype=strip.dtype, device=strip.device)
        dist.all_gather_into_tensor(flat, send.contiguous(), group=group)
        gathered = flat.view(P, cols)
        carry = ops.exscan(gathered, rank) if rank > 0 else None
    else:
        carry = None
    out = ops.seeded_sat(strip, carry, out=out)
    stats = dict(strip_bytes_read=rows * cols * eb, strip_bytes_written=rows * cols * eb,
                 extra_bytes_read=(rows * cols * eb if (P > 1 and rank < P - 1) else 0),
                 allgather_bytes=(P * cols * eb if P > 1 else 0))
    return out, stats


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
    return ex, ptrs
