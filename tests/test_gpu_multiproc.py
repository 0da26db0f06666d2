"""Row-strip sharding across real PROCESSES on one GPU (north star (3);
SURVEY 8.4, 8(f4)).

Every GPU call of this build has one device, so the multi-process data plane
runs as two (or three) processes sharing cuda:0:

* ``RowStripSAT`` with the real CUDA ops (libsat column totals + seeded SAT
  whose band 0 does the rank exclusive scan), the all-gather over a gloo
  process group through host memory;
* the fused peer exchange with REAL CUDA-IPC mailboxes opened in the other
  process (``cudaIpcOpenMemHandle``): the totals kernel's epilogue stores into
  the other process's mailbox and raises its flag with st.release.sys; the
  consumer's band 0 waits with ld.acquire.sys and acknowledges.

Expected values come from the CPU oracle only.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.multiprocessing as mp

import oracle
from sat_inputs import make_np

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _init(rank, world, port):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    return dist


def _gen(n, m, dtype, seed, row0=0):
    return make_np(n, m, dtype, "u32" if dtype == "int32" else "unit", seed=seed, row0=row0)


def _strip_worker(rank, world, port, n, m, dtype, weight, calls, q):
    try:
        dist = _init(rank, world, port)
        from paper_conf_icpp_kasagini14_b200.dist import RowStripSAT, partition_rows
        r0, r1 = partition_rows(n, world, rank, weight)
        tdt = {"int32": torch.int32, "float32": torch.float32}[dtype]
        op = RowStripSAT(m, tdt, device="cuda", host_exchange=True)
        outs = []
        for c in range(calls):
            strip = torch.from_numpy(_gen(r1 - r0, m, dtype, seed=50 + c, row0=r0)).cuda()
            out, st = op(strip)
            torch.cuda.synchronize()
            outs.append(out.cpu().numpy())
        q.put((rank, r0, r1, outs, st, None))
        dist.barrier()
        dist.destroy_process_group()
    except Exception as e:  # reported to the parent
        q.put((rank, 0, 0, None, None, repr(e)))
        raise


def _xchg_worker(rank, world, port, n, m, dtype, calls, q):
    try:
        dist = _init(rank, world, port)
        from paper_conf_icpp_kasagini14_b200.dist import make_peer_exchange, partition_rows
        import paper_conf_icpp_kasagini14_b200 as libsat
        r0, r1 = partition_rows(n, world, rank, 1.5)
        tdt = {"int32": torch.int32, "float32": torch.float32, "float64": torch.float64}[dtype]
        ex, ptrs = make_peer_exchange(m, tdt, device="cuda")
        outs, launches = [], []
        for c in range(calls):
            strip = torch.from_numpy(_gen(r1 - r0, m, dtype, seed=70 + c, row0=r0)).cuda()
            out = ex.sat(strip)
            launches.append(libsat.last_launch_count())
            torch.cuda.synchronize()
            outs.append(out.cpu().numpy())
        dist.barrier()                       # nobody unmaps a mailbox still in use
        for qq, p in enumerate(ptrs):
            if qq != rank:
                libsat.ipc_close(p)
        ex.close()
        q.put((rank, r0, r1, outs, launches, None))
        dist.barrier()
        dist.destroy_process_group()
    except Exception as e:
        q.put((rank, 0, 0, None, None, repr(e)))
        raise


def _spawn(target, world, args, timeout=300):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=target, args=(r, world, port) + args + (q,)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=timeout) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    errs = [r[5] for r in res if r[5]]
    assert not errs, errs
    for p in procs:
        assert p.exitcode == 0
    return sorted(res, key=lambda t: t[0])


def _compare(got, ref, dtype):
    if dtype == "float32":
        assert oracle.max_rel_err(got, ref) <= 1e-5
    else:
        assert np.array_equal(got, ref)


@pytest.mark.parametrize("world,dtype", [(2, "int32"), (2, "float32"), (3, "int32")])
def test_row_strips_two_processes_cuda_ops(world, dtype):
    """dist.RowStripSAT in separate processes with the real CUDA kernels;
    strips weighted 1.5 for the last rank (it skips the totals pass)."""
    n, m, calls = 3001, 2304, 2
    res = _spawn(_strip_worker, world, (n, m, dtype, 1.5, calls))
    assert res[0][1] == 0 and res[-1][2] == n
    for c in range(calls):
        full = _gen(n, m, dtype, seed=50 + c)
        got = np.concatenate([r[3][c] for r in res])
        _compare(got, oracle.sat(full), dtype)
    for rank, r0, r1, _, st, _ in res:
        assert st["extra_bytes_read"] == (0 if rank == world - 1 else (r1 - r0) * m * 4)


@pytest.mark.parametrize("world,dtype", [(2, "int32"), (2, "float64"), (3, "float32")])
def test_fused_exchange_ipc_processes(world, dtype):
    """The fused exchange over real CUDA-IPC mailboxes between processes: 5
    consecutive calls (both mailbox parities, acknowledgements) without any
    barrier between calls; two launches per rank < P-1, one for the last."""
    n, m, calls = 2500, 1700, 5
    res = _spawn(_xchg_worker, world, (n, m, dtype, calls))
    for c in range(calls):
        full = _gen(n, m, dtype, seed=70 + c)
        got = np.concatenate([r[3][c] for r in res])
        _compare(got, oracle.sat(full), dtype)
    for rank, _, _, _, launches, _ in res:
        assert launches == [2 if rank < world - 1 else 1] * calls
