"""Row-strip sharding host logic at world_size 2 (and 3) over gloo on CPU.

The per-rank compute steps are replaced by oracle-based stand-ins (this is a
test of partitioning, the all-gather exchange and the rank-ordered carry; the
CUDA steps are covered by the -m gpu tests)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
from sat_inputs import make_np


class OracleOps:
    """Oracle stand-ins with CudaOps' interface: column totals into the
    exchange buffer; the seeded SAT takes the gathered totals and the rank
    (the exclusive scan over ranks happens inside it, as in the kernel)."""

    def column_totals(self, strip, out=None):
        t = torch.from_numpy(oracle.column_totals(strip.numpy()).astype(np.int32))
        if out is not None:
            out.copy_(t)
            return out
        return t

    def seeded_sat(self, strip, gathered, rank, out=None):
        loc = oracle.sat(strip.numpy()).view(np.uint32)
        if gathered is not None and rank > 0:
            carry = np.ascontiguousarray(oracle.rank_exscan(gathered.numpy(), rank)).view(np.uint32)
            top = np.cumsum(carry.astype(np.uint64)).astype(np.uint32)
            with np.errstate(over="ignore"):
                loc = loc + top[None, :]
        return torch.from_numpy(loc.view(np.int32).copy())


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, n, m, weight, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_icpp_kasagini14_b200.dist import partition_rows, sharded_sat
    r0, r1 = partition_rows(n, world, rank, weight)
    full = make_np(n, m, "int32", "u32", seed=31)
    strip = torch.from_numpy(make_np(r1 - r0, m, "int32", "u32", seed=31, row0=r0))
    assert np.array_equal(strip.numpy(), full[r0:r1])
    out, stats = sharded_sat(strip, ops=OracleOps())
    q.put((rank, r0, r1, out.numpy(), stats))
    dist.barrier()
    dist.destroy_process_group()


def _run(world, n, m, weight=1.0):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, n, m, weight, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=60) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    return sorted(res, key=lambda t: t[0])


@pytest.mark.parametrize("world,weight", [(2, 1.0), (3, 1.5)])
def test_sharded_matches_unsharded(world, weight):
    n, m = 97, 70
    res = _run(world, n, m, weight)
    ref = oracle.sat(make_np(n, m, "int32", "u32", seed=31))
    got = np.concatenate([r[3] for r in res])
    assert np.array_equal(got, ref)
    assert res[0][1] == 0 and res[-1][2] == n
    for rank, r0, r1, _, st in res:
        assert st["strip_bytes_read"] == (r1 - r0) * m * 4
        assert st["extra_bytes_read"] == (0 if rank == world - 1 else (r1 - r0) * m * 4)
        assert st["allgather_bytes"] == world * m * 4


def test_partition_rows():
    from paper_conf_icpp_kasagini14_b200.dist import partition_rows
    for n, P in [(65536, 8), (10, 3), (5, 8), (0, 2)]:
        b = [partition_rows(n, P, p) for p in range(P)]
        assert b[0][0] == 0 and b[-1][1] == n
        assert all(b[i][1] == b[i + 1][0] for i in range(P - 1))
    r = [partition_rows(65536, 8, p, 1.5) for p in range(8)]
    assert r[-1][1] - r[-1][0] > r[0][1] - r[0][0]


def _xchg_worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_icpp_kasagini14_b200.dist import make_peer_exchange
    opened = []

    def get_handle(t):
        return f"mailbox-of-{rank}".encode()

    def open_handle(h):
        opened.append(h)
        return 1000 + int(h.decode().rsplit("-", 1)[1])      # fake peer address of that rank

    made = {}

    def factory(r, P, cols, dtype, mailbox, ptrs):
        made.update(rank=r, P=P, cols=cols, nbytes=mailbox.numel(), ptrs=list(ptrs),
                    own=mailbox.data_ptr())
        return "exchange"
    ex, ptrs = make_peer_exchange(777, torch.int32, ipc=(get_handle, open_handle), factory=factory)
    q.put((rank, ex, made, opened))
    dist.barrier()
    dist.destroy_process_group()


def test_peer_exchange_setup_world3():
    """Fused-exchange set-up: every rank maps every OTHER rank's
    mailbox from its published handle, in rank order, and keeps its own."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    world = 3
    procs = [ctx.Process(target=_xchg_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted([q.get(timeout=60) for _ in range(world)], key=lambda t: t[0])
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for rank, ex, made, opened in res:
        assert ex == "exchange" and made["rank"] == rank and made["P"] == world and made["cols"] == 777
        assert made["ptrs"][rank] == made["own"]
        assert [made["ptrs"][qq] for qq in range(world) if qq != rank] == \
            [1000 + qq for qq in range(world) if qq != rank]
        assert sorted(opened) == sorted(f"mailbox-of-{qq}".encode() for qq in range(world) if qq != rank)
