"""libsat Python binding: summed area tables on B200 (sm_100a).

Thin ctypes marshalling over the C ABI in ``include/sat.h`` -- every step of
every variant runs in the CUDA kernels of ``libsat.so``; there is no CPU or
PyTorch fallback.  If the shared library is missing this module raises on
import.  Torch is used only for device memory and streams.

The operation: ``b[i][j] = sum_{k<=i, l<=j} a[k][l]``.
"""
from __future__ import annotations

import ctypes
import os

from ._build import LIB as _LIB_PATH

# tools may load the debug build (event traces): LIBSAT_SO=.../libsat_debug.so
_LIB_PATH = os.environ.get("LIBSAT_SO", _LIB_PATH)

if not os.path.exists(_LIB_PATH):
    raise ImportError(
        f"libsat.so not found at {_LIB_PATH}; run __graft_entry__.build() "
        "(or python -m paper_conf_icpp_kasagini14_b200._build)")

_lib = ctypes.CDLL(_LIB_PATH)

SAT_INT32, SAT_FLOAT32, SAT_FLOAT64, SAT_UINT8 = 0, 1, 2, 3
VARIANTS = {"2r2w": 0, "2r1w": 1, "1r1w": 2, "1+rr1w": 3, "4r4w": 4, "4r1w": 5}
SAT_OK = 0


class SatOptions(ctypes.Structure):
    _fields_ = [("r", ctypes.c_double), ("tile_rows", ctypes.c_int),
                ("force_generic", ctypes.c_int), ("jitter", ctypes.c_int),
                ("segments", ctypes.c_int), ("lookback_group", ctypes.c_int),
                ("reserved", ctypes.c_int * 2)]


class SatShardStats(ctypes.Structure):
    _fields_ = [("strip_bytes_read", ctypes.c_int64), ("strip_bytes_written", ctypes.c_int64),
                ("extra_bytes_read", ctypes.c_int64), ("allgather_bytes", ctypes.c_int64)]


ALLGATHER_FN = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p,
                                ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p)

_P, _I64, _I = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int
_SIGS = {
    "sat_options_init": ([ctypes.POINTER(SatOptions)], None),
    "sat_compute": ([_P, _P, _I64, _I64, _I, _I, _P], _I),
    "sat_compute_ex": ([_P, _P, _I64, _I64, _I, _I, ctypes.POINTER(SatOptions), _P], _I),
    "sat_compute_batched": ([_P, _P, _I64, _I64, _I64, _I, _I, ctypes.POINTER(SatOptions), _P], _I),
    "sat_compute_widening": ([_P, _I, _P, _I, _I64, _I64, _I64, ctypes.POINTER(SatOptions), _P], _I),
    "sat_box_filter": ([_P, _I, _P, _I, _I64, _I64, _I64, _I, _I, _I, _P], _I),
    "sat_rect_sums": ([_P, _I, _I64, _I64, _I64, _P, _I64, _P, _P], _I),
    "sat_exchange_mailbox_bytes": ([_I64, _I, _I], ctypes.c_size_t),
    "sat_exchange_create": ([ctypes.POINTER(ctypes.c_void_p), _I, _I, _I64, _I, _P,
                             ctypes.POINTER(ctypes.c_void_p)], _I),
    "sat_exchange_destroy": ([_P], _I),
    "sat_compute_sharded_fused": ([_P, _P, _I64, _P, _P], _I),
    "sat_ipc_get_handle": ([_P, _P], _I),
    "sat_ipc_open": ([_P, ctypes.POINTER(ctypes.c_void_p)], _I),
    "sat_ipc_close": ([_P], _I),
    "sat_compute_seeded": ([_P, _P, _I64, _I64, _I, _P, _P], _I),
    "sat_compute_seeded_sum": ([_P, _P, _I64, _I64, _I, _P, _I64, _I64, _P], _I),
    "sat_compute_seeded_satrow": ([_P, _P, _I64, _I64, _I, _P, _P], _I),
    "sat_column_totals": ([_P, _P, _I64, _I64, _I, _P], _I),
    "sat_rank_exscan": ([_P, _P, _I64, _I64, _I, _I, _P], _I),
    "sat_compute_sharded": ([_P, _P, _I64, _I64, _I, _I, _I, ALLGATHER_FN, _P, _P, _P,
                             ctypes.POINTER(SatShardStats)], _I),
    "sat_sharded_workspace_bytes": ([_I64, _I, _I], ctypes.c_size_t),
    "sat_compute_sharded_ex": ([_P, _P, _I64, _I64, _I, _I, _I, _I, ALLGATHER_FN, _P, _P, _P,
                                ctypes.POINTER(SatShardStats)], _I),
    "sat_nccl_unique_id": ([_P], _I),
    "sat_nccl_comm_create": ([ctypes.POINTER(ctypes.c_void_p), _P, _I, _I], _I),
    "sat_nccl_comm_destroy": ([_P], _I),
    "sat_compute_sharded_nccl": ([_P, _P, _I64, _I64, _I, _I, _P, _P, _P, ctypes.POINTER(SatShardStats)], _I),
    "sat_compute_host": ([_P, _P, _I64, _I64, _I, _I, _P], _I),
    "sat_release_workspace": ([_P], _I),
    "sat_debug_set_tag_space": ([ctypes.c_uint64], _I),
    "sat_debug_set_box_rows": ([ctypes.c_int], _I),
    "sat_debug_trace": ([_P], _I),
    "sat_debug_diag_enable": ([], _I),
    "sat_debug_diag_dump": ([], _I),
    "sat_last_launch_count": ([], _I),
    "sat_last_tile_rows": ([], _I),
    "sat_last_grid": ([], _I),
    "sat_last_lookback_group": ([], _I),
    "sat_last_r_effective": ([], ctypes.c_double),
    "sat_strerror": ([_I], ctypes.c_char_p),
    "sat_last_error": ([], ctypes.c_char_p),
    "sat_abi_version": ([], _I),
}
for _name, (_args, _res) in _SIGS.items():
    _f = getattr(_lib, _name)
    _f.argtypes = _args
    _f.restype = _res

# every symbol include/sat.h declares (checked by tests/test_abi.py)
EXPORTED = tuple(_SIGS)


class SatError(RuntimeError):
    pass


def _check(status: int):
    if status != SAT_OK:
        msg = f"{_lib.sat_strerror(status).decode()}: {_lib.sat_last_error().decode()}"
        if status == -1:
            raise ValueError(msg)
        raise SatError(msg)


def _dtype_code(t) -> int:
    import torch
    if t.dtype == torch.int32:
        return SAT_INT32
    if t.dtype == torch.float32:
        return SAT_FLOAT32
    if t.dtype == torch.float64:
        return SAT_FLOAT64
    if t.dtype == torch.uint8:
        return SAT_UINT8
    raise TypeError(f"libsat supports int32, float32 and float64, got {t.dtype}")


def _stream(stream) -> int:
    import torch
    if stream is None:
        stream = torch.cuda.current_stream()
    return stream.cuda_stream


def _check_dev(*ts):
    for t in ts:
        if t is None:
            continue
        if not t.is_cuda:
            raise ValueError("libsat takes CUDA tensors (use sat_host for host memory)")
        if not t.is_contiguous():
            raise ValueError("libsat takes contiguous row-major tensors")


def options(r: float = 0.25, tile_rows: int = 0, force_generic: bool = False,
            jitter: int = 0, segments: int = 0, lookback_group: int = 0) -> SatOptions:
    o = SatOptions()
    _lib.sat_options_init(ctypes.byref(o))
    o.r = float(r)
    o.tile_rows = int(tile_rows)
    o.force_generic = int(bool(force_generic))
    o.jitter = int(jitter)
    o.segments = int(segments)
    o.lookback_group = int(lookback_group)
    return o


def sat(x, variant: str = "1r1w", out=None, r: float = 0.25, tile_rows: int = 0,
        force_generic: bool = False, jitter: int = 0, segments: int = 0, stream=None,
        lookback_group: int = 0):
    """SAT of a 2-D CUDA tensor (int32 wraps mod 2^32, float32/float64 IEEE).

    ``out`` may be ``x`` itself (in place).  ``variant`` in
    {"1r1w", "2r2w", "2r1w", "1+rr1w"}.
    """
    import torch
    if x.dim() != 2:
        raise ValueError("sat expects a 2-D tensor (use sat_batched for 3-D)")
    if out is None:
        out = torch.empty_like(x)
    _check_dev(x, out)
    if out.shape != x.shape or out.dtype != x.dtype:
        raise ValueError("out must match x in shape and dtype")
    o = options(r, tile_rows, force_generic, jitter, segments, lookback_group)
    _check(_lib.sat_compute_ex(x.data_ptr(), out.data_ptr(), x.shape[0], x.shape[1],
                               _dtype_code(x), VARIANTS[variant], ctypes.byref(o), _stream(stream)))
    return out


def sat_batched(x, variant: str = "1r1w", out=None, r: float = 0.25, tile_rows: int = 0,
                force_generic: bool = False, segments: int = 0, stream=None,
                lookback_group: int = 0):
    """SATs of a (batch, rows, cols) CUDA tensor, one launch for the batch."""
    import torch
    if x.dim() != 3:
        raise ValueError("sat_batched expects (batch, rows, cols)")
    if out is None:
        out = torch.empty_like(x)
    _check_dev(x, out)
    o = options(r, tile_rows, force_generic, 0, segments, lookback_group)
    _check(_lib.sat_compute_batched(x.data_ptr(), out.data_ptr(), x.shape[0], x.shape[1],
                                    x.shape[2], _dtype_code(x), VARIANTS[variant],
                                    ctypes.byref(o), _stream(stream)))
    return out


def _as3(x):
    return x if x.dim() == 3 else x.unsqueeze(0)


def sat_widening(x, dtype, out=None, tile_rows: int = 0, force_generic: bool = False, segments: int = 0,
                 stream=None):
    """1R1W SAT of a uint8 (-> int32 sums) or float32 (-> float64 sums) CUDA
    tensor, 2-D or (batch, rows, cols), widened on load (no extra pass)."""
    import torch
    x3 = _as3(x)
    if out is None:
        out = torch.empty(x.shape, dtype=dtype, device=x.device)
    _check_dev(x, out)
    o = options(0.25, tile_rows, force_generic, 0, segments)
    _check(_lib.sat_compute_widening(x.data_ptr(), _dtype_code(x), out.data_ptr(), _dtype_code(out),
                                     x3.shape[0], x3.shape[1], x3.shape[2], ctypes.byref(o),
                                     _stream(stream)))
    return out


def box_filter(x, rr: int, rc: int, normalize: bool = False, out_dtype=None, out=None, stream=None):
    """Box filter through a SAT: window (2rr+1) x (2rc+1),
    clipped.  uint8/int32 input -> int32 sums; float32/float64 input -> float
    (``out_dtype``, default the input's), SAT in float64."""
    import torch
    x3 = _as3(x)
    if out is None:
        if out_dtype is None:
            out_dtype = torch.int32 if x.dtype in (torch.uint8, torch.int32) else x.dtype
        out = torch.empty(x.shape, dtype=out_dtype, device=x.device)
    _check_dev(x, out)
    _check(_lib.sat_box_filter(x.data_ptr(), _dtype_code(x), out.data_ptr(), _dtype_code(out),
                               x3.shape[0], x3.shape[1], x3.shape[2], int(rr), int(rc),
                               int(bool(normalize)), _stream(stream)))
    return out


def rect_sums(sat_t, rects, out=None, stream=None):
    """Rectangle sums from a SAT: ``rects`` (K, 5) int32 CUDA tensor of
    (image, r0, c0, r1, c1), inclusive, clipped."""
    import torch
    s3 = _as3(sat_t)
    rects = rects.to(torch.int32).contiguous()
    if out is None:
        out = torch.empty(rects.shape[0], dtype=sat_t.dtype, device=sat_t.device)
    _check_dev(sat_t, rects, out)
    _check(_lib.sat_rect_sums(sat_t.data_ptr(), _dtype_code(sat_t), s3.shape[0], s3.shape[1],
                              s3.shape[2], rects.data_ptr(), rects.shape[0], out.data_ptr(),
                              _stream(stream)))
    return out


def sat_seeded(x, carry_row=None, out=None, sat_row=None, gathered=None, rank: int = 0, stream=None):
    """Rows of the SAT of a taller matrix: ``carry_row`` = column sums of
    everything above ``x``; or ``gathered`` (nranks, cols) all-gathered column
    totals of the strips of every rank, of which ranks < ``rank`` lie above
    ``x`` (the sharded mode: the exclusive scan runs inside the SAT kernel);
    or ``sat_row`` = the SAT row just above."""
    import torch
    if out is None:
        out = torch.empty_like(x)
    _check_dev(x, out, carry_row, sat_row, gathered)
    if sat_row is not None:
        _check(_lib.sat_compute_seeded_satrow(x.data_ptr(), out.data_ptr(), x.shape[0], x.shape[1],
                                              _dtype_code(x), sat_row.data_ptr(), _stream(stream)))
    elif gathered is not None:
        g = gathered.view(-1, x.shape[1]) if gathered.dim() == 1 else gathered
        if not (0 <= rank <= g.shape[0]):
            raise ValueError("rank out of range")
        _check(_lib.sat_compute_seeded_sum(x.data_ptr(), out.data_ptr(), x.shape[0], x.shape[1],
                                           _dtype_code(x), g.data_ptr(), int(rank), g.stride(0),
                                           _stream(stream)))
    else:
        _check(_lib.sat_compute_seeded(x.data_ptr(), out.data_ptr(), x.shape[0], x.shape[1],
                                       _dtype_code(x),
                                       carry_row.data_ptr() if carry_row is not None else None,
                                       _stream(stream)))
    return out


def column_totals(x, out=None, stream=None):
    import torch
    if out is None:
        out = torch.empty(x.shape[1], dtype=x.dtype, device=x.device)
    _check_dev(x, out)
    _check(_lib.sat_column_totals(x.data_ptr(), out.data_ptr(), x.shape[0], x.shape[1],
                                  _dtype_code(x), _stream(stream)))
    return out


def rank_exscan(gathered, rank: int, out=None, stream=None):
    import torch
    if out is None:
        out = torch.empty(gathered.shape[1], dtype=gathered.dtype, device=gathered.device)
    _check_dev(gathered, out)
    _check(_lib.sat_rank_exscan(gathered.data_ptr(), out.data_ptr(), gathered.shape[0],
                                gathered.shape[1], int(rank), _dtype_code(gathered),
                                _stream(stream)))
    return out


def sat_host(x_host, out_host=None, variant: str = "1r1w", stream=None):
    """End to end from host memory (pinned tensors overlap copies and compute)."""
    import torch
    if x_host.is_cuda:
        raise ValueError("sat_host takes CPU tensors")
    if not x_host.is_contiguous():
        raise ValueError("sat_host takes contiguous tensors")
    if out_host is None:
        out_host = torch.empty_like(x_host, pin_memory=x_host.is_pinned())
    _check(_lib.sat_compute_host(x_host.data_ptr(), out_host.data_ptr(), x_host.shape[0],
                                 x_host.shape[1], _dtype_code(x_host), VARIANTS[variant],
                                 _stream(stream)))
    return out_host


def sat_sharded_abi(strip, rank: int, nranks: int, allgather, out=None, stream=None,
                    variant: str = "1r1w"):
    """Row-strip sharded SAT through the single C-ABI call
    (sat_compute_sharded_ex; variant "1r1w" or "2r2w").

    ``allgather(send, recv)`` receives torch views of the library's send
    (cols) and receive (nranks x cols) buffers and must fill ``recv``.
    Returns (out, stats dict).
    """
    import torch
    if out is None:
        out = torch.empty_like(strip)
    _check_dev(strip, out)
    cols = strip.shape[1]
    nbytes = _lib.sat_sharded_workspace_bytes(cols, nranks, _dtype_code(strip))
    ws = torch.empty(max(nbytes, 1), dtype=torch.uint8, device=strip.device)
    eb = strip.element_size()
    row = ((cols * eb) + 255) // 256 * 256
    send = ws[:cols * eb].view(strip.dtype)
    recv = ws[2 * row:2 * row + nranks * cols * eb].view(strip.dtype).view(nranks, cols)
    err = []

    def cb(ctx, send_p, recv_p, nb, st):
        try:
            assert send_p == send.data_ptr() and recv_p == recv.data_ptr() and nb == cols * eb
            allgather(send, recv)
            return 0
        except Exception as e:  # reported through SAT_ERR_COMM
            err.append(e)
            return 1
    cfun = ALLGATHER_FN(cb)
    stats = SatShardStats()
    st = _lib.sat_compute_sharded_ex(strip.data_ptr(), out.data_ptr(), strip.shape[0], cols,
                                     _dtype_code(strip), VARIANTS[variant], int(rank), int(nranks), cfun,
                                     None, ws.data_ptr(), _stream(stream), ctypes.byref(stats))
    if err:
        raise err[0]
    _check(st)
    return out, {f: getattr(stats, f) for f, _ in SatShardStats._fields_}


def nccl_unique_id() -> bytes:
    """128-byte NCCL id for sat_nccl_comm_create (rank 0 makes it, every rank gets it)."""
    buf = ctypes.create_string_buffer(128)
    _check(_lib.sat_nccl_unique_id(buf))
    return buf.raw


class NcclComm:
    """libsat's own NCCL communicator (sat_nccl_comm_create) on the current device."""

    def __init__(self, uid: bytes, rank: int, nranks: int):
        if len(uid) != 128:
            raise ValueError("NCCL unique id is 128 bytes")
        h = ctypes.c_void_p()
        _check(_lib.sat_nccl_comm_create(ctypes.byref(h), ctypes.c_char_p(uid), int(rank), int(nranks)))
        self.handle, self.rank, self.nranks = h, rank, nranks

    def close(self):
        if self.handle:
            _check(_lib.sat_nccl_comm_destroy(self.handle))
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def sat_sharded_nccl(strip, comm: "NcclComm", variant: str = "1r1w", out=None, stream=None):
    """Row-strip sharded SAT with the all-gather inside libsat (ncclAllGather,
    sat_compute_sharded_nccl).  Returns (out, stats dict)."""
    import torch
    if out is None:
        out = torch.empty_like(strip)
    _check_dev(strip, out)
    stats = SatShardStats()
    _check(_lib.sat_compute_sharded_nccl(strip.data_ptr(), out.data_ptr(), strip.shape[0], strip.shape[1],
                                         _dtype_code(strip), VARIANTS[variant], comm.handle, None,
                                         _stream(stream), ctypes.byref(stats)))
    return out, {f: getattr(stats, f) for f, _ in SatShardStats._fields_}


class PeerExchange:
    """One rank's end of the fused peer exchange (sat_exchange_create).

    ``mailbox``: this rank's mailbox (a CUDA uint8 tensor of
    ``mailbox_bytes`` bytes); ``peer_ptrs``: integer device pointers of every
    rank's mailbox as seen from this rank (IPC-mapped for other processes).
    Keep the tensors alive as long as the exchange.
    """

    def __init__(self, rank: int, nranks: int, cols: int, dtype, mailbox, peer_ptrs):
        import torch
        self.dtype = dtype
        self.cols = int(cols)
        self.mailbox = mailbox
        code = {torch.int32: SAT_INT32, torch.float32: SAT_FLOAT32, torch.float64: SAT_FLOAT64}[dtype]
        arr = (ctypes.c_void_p * nranks)(*[int(p) for p in peer_ptrs])
        h = ctypes.c_void_p()
        _check(_lib.sat_exchange_create(ctypes.byref(h), int(rank), int(nranks), self.cols, code,
                                        mailbox.data_ptr(), arr))
        self._h = h

    @staticmethod
    def mailbox_bytes(cols: int, nranks: int, dtype) -> int:
        import torch
        code = {torch.int32: SAT_INT32, torch.float32: SAT_FLOAT32, torch.float64: SAT_FLOAT64}[dtype]
        return int(_lib.sat_exchange_mailbox_bytes(int(cols), int(nranks), code))

    def sat(self, strip, out=None, stream=None):
        import torch
        if out is None:
            out = torch.empty_like(strip)
        _check_dev(strip, out)
        _check(_lib.sat_compute_sharded_fused(strip.data_ptr(), out.data_ptr(), strip.shape[0],
                                              self._h, _stream(stream)))
        return out

    def close(self):
        if self._h:
            _lib.sat_exchange_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def ipc_handle(t) -> bytes:
    buf = ctypes.create_string_buffer(64)
    _check(_lib.sat_ipc_get_handle(t.data_ptr(), buf))
    return buf.raw


def ipc_open(handle: bytes) -> int:
    p = ctypes.c_void_p()
    _check(_lib.sat_ipc_open(ctypes.create_string_buffer(handle, 64), ctypes.byref(p)))
    return int(p.value)


def ipc_close(ptr: int) -> None:
    _check(_lib.sat_ipc_close(ctypes.c_void_p(ptr)))


def release_workspace(stream=None) -> None:
    """Free libsat's workspace of ``stream`` (sat_release_workspace)."""
    _check(_lib.sat_release_workspace(_stream(stream)))


def set_box_rows(rows: int) -> None:
    """Tests / tuning only: output rows per column-walk box-filter unit (0 = automatic)."""
    _check(_lib.sat_debug_set_box_rows(int(rows)))


def set_tag_space(space: int) -> None:
    """Tests only: shrink the look-back tag space (0 = default 2^30)."""
    _check(_lib.sat_debug_set_tag_space(int(space)))


def last_launch_count() -> int:
    return _lib.sat_last_launch_count()


def last_tile_rows() -> int:
    return _lib.sat_last_tile_rows()


def last_grid() -> int:
    return _lib.sat_last_grid()


def last_lookback_group() -> int:
    return _lib.sat_last_lookback_group()


def last_r_effective() -> float:
    return _lib.sat_last_r_effective()


def abi_version() -> int:
    return _lib.sat_abi_version()


lib = _lib


def debug_trace(buf) -> None:
    """Arm event tracing of the next band launch on this thread (see
    ``sat_debug_trace`` in include/sat.h); ``buf`` is a CUDA int64 tensor."""
    _check(_lib.sat_debug_trace(None if buf is None else buf.data_ptr()))
