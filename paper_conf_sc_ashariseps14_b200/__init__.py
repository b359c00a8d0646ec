"""ACSR on B200: adaptive CSR SpMV (Ashari et al., SC'14), sm_100a.

Thin ctypes binding over ``lib/libacsr.so`` (C ABI declared in ``include/acsr.h``).
The functions carry the C names and only marshal arguments: every step of the path
runs in the library's CUDA kernels.  PyTorch provides device memory
(``tensor.data_ptr()``) and streams (``torch.cuda.current_stream()``); there is no
CPU fallback -- importing this package fails loudly if the library is missing, and
every call requires CUDA tensors.

Entry points (same names as the C ABI):
  acsr_bin            row binning + SpMV work map   (Alg. 1)
  acsr_spmv           y = A x on CSR                (Alg. 2-4)
  acsr_pagerank_step  one fused PageRank step       (Alg. 5)
  acsr_pagerank_scale xs = x / outdeg
  acsr_update_edges   dynamic-graph update          (§VII)
Helpers: ``ACSRMatrix`` (owns CSR + plan), ``spmv_from_host`` (end-to-end path with
host buffers), ``pagerank`` (single-GPU Alg. 5 loop) and
``paper_conf_sc_ashariseps14_b200.dist`` (row-partitioned multi-GPU PageRank).
"""
from __future__ import annotations

import ctypes
import os

import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
# ACSR_LIB_VARIANT=<name> loads lib/libacsr_<name>.so (compile-time A/B variants built by
# tools/build_variants.sh; measurements only).
_VARIANT = os.environ.get("ACSR_LIB_VARIANT", "")
LIB_PATH = os.path.join(_HERE, "lib", f"libacsr_{_VARIANT}.so" if _VARIANT else "libacsr.so")

ACSR_OK = 0
ACSR_ERR_INVALID_VALUE = 1
ACSR_ERR_WORKSPACE = 2
ACSR_ERR_CAPACITY = 3
ACSR_ERR_CUDA = 4
ACSR_ERR_NCCL = 5
ACSR_COMM_ID_BYTES = 128
ACSR_F32 = 0
ACSR_F64 = 1
NBINS = 32

if not os.path.exists(LIB_PATH):
    raise ImportError(f"libacsr.so not built ({LIB_PATH}); run `python -c 'import __graft_entry__ as g; "
                      f"g.build()'` -- there is no CPU fallback")

_lib = ctypes.CDLL(LIB_PATH)
_i64, _vp, _sz, _dbl = ctypes.c_int64, ctypes.c_void_p, ctypes.c_size_t, ctypes.c_double
_lib.acsr_bin_workspace_bytes.argtypes = [_i64, _i64, _i64]
_lib.acsr_bin_workspace_bytes.restype = _sz
_lib.acsr_bin.argtypes = [_i64, _i64, _i64, _vp, _vp, _vp, _vp, _vp, _vp, _sz, _vp]
_lib.acsr_bin.restype = ctypes.c_int
_lib.acsr_bin_ex.argtypes = [_i64, _i64, _i64, _vp, _vp, _vp, _vp, _vp, _vp, _sz, ctypes.c_uint, _vp]
_lib.acsr_bin_ex.restype = ctypes.c_int
_lib.acsr_spmv.argtypes = [ctypes.c_int, _i64, _i64, _vp, _vp, _vp, _vp, _vp, _vp, _vp, _vp, _vp, _sz,
                           _vp]
_lib.acsr_spmv.restype = ctypes.c_int
_lib.acsr_pagerank_scale.argtypes = [_i64, _vp, _vp, _vp, _vp]
_lib.acsr_pagerank_scale.restype = ctypes.c_int
_lib.acsr_update_workspace_bytes.argtypes = [_i64]
_lib.acsr_update_workspace_bytes.restype = _sz
_lib.acsr_update_edges.argtypes = [ctypes.c_int, _i64, _i64, _vp, _vp, _vp, _vp, _vp, _i64, _vp, _vp,
                                   _vp, _vp, _vp, _vp, _vp, _vp, _vp, _sz, _vp]
_lib.acsr_update_edges.restype = ctypes.c_int
_lib.acsr_update_edges_dev.argtypes = [ctypes.c_int, _i64, _i64, _vp, _vp, _vp, _vp, _vp, _i64, _vp, _vp, _vp,
                                       _vp, _vp, _vp, _vp, _vp, _vp, _vp, _sz, _vp]
_lib.acsr_update_edges_dev.restype = ctypes.c_int
_lib.acsr_relayout.argtypes = [ctypes.c_int, _i64, _vp, _vp, _vp, _vp, _vp, _vp, _vp, _vp, _vp]
_lib.acsr_relayout.restype = ctypes.c_int
_lib.acsr_status_string.argtypes = [ctypes.c_int]
_lib.acsr_status_string.restype = ctypes.c_char_p
_lib.acsr_last_error.restype = ctypes.c_char_p
_lib.acsr_version.restype = ctypes.c_int


class PrArgs(ctypes.Structure):
    """Mirror of ``acsr_pr_args`` (include/acsr.h)."""
    _fields_ = [("n_rows", _i64), ("n_cols", _i64), ("row_begin", _vp), ("row_end", _vp),
                ("col_idx", _vp), ("bin_rows", _vp), ("bin_offsets", _vp), ("plan_ws", _vp),
                ("plan_ws_bytes", _sz), ("xs", _vp), ("x", _vp), ("outdeg", _vp), ("x_new", _vp),
                ("xs_next", _vp), ("damping", _dbl), ("teleport", _dbl), ("delta2", _vp),
                ("restart", _i64), ("restart_weight", _dbl), ("ctrl", _vp), ("eps2", _dbl),
                ("comm", _vp), ("xs_all", _vp), ("slice_len", _i64), ("slice_counts", ctypes.POINTER(_i64))]


_lib.acsr_pagerank_step.argtypes = [ctypes.POINTER(PrArgs), _vp]
_lib.acsr_pagerank_step.restype = ctypes.c_int
_lib.acsr_pagerank_step_peer.argtypes = [ctypes.POINTER(PrArgs), _vp, _vp]
_lib.acsr_pagerank_step_peer.restype = ctypes.c_int
_lib.acsr_peer_create.argtypes = [ctypes.POINTER(_vp), ctypes.c_int, ctypes.c_int, _i64, _i64, _i64, _vp]
_lib.acsr_peer_create.restype = ctypes.c_int
_lib.acsr_peer_open.argtypes = [_vp, _vp]
_lib.acsr_peer_open.restype = ctypes.c_int
_lib.acsr_peer_destroy.argtypes = [_vp]
_lib.acsr_peer_destroy.restype = ctypes.c_int
_lib.acsr_peer_push.argtypes = [_vp, _i64, _vp, _vp, _vp, _vp]
_lib.acsr_peer_push.restype = ctypes.c_int
_lib.acsr_peer_delta2.argtypes = [_vp, _vp, _vp, _dbl, _vp]
_lib.acsr_peer_delta2.restype = ctypes.c_int
_lib.acsr_peer_query.argtypes = [_vp, ctypes.POINTER(_i64), ctypes.POINTER(ctypes.c_int32), ctypes.POINTER(_vp)]
_lib.acsr_peer_query.restype = ctypes.c_int
_lib.acsr_peer_read_xs.argtypes = [_vp, _vp, _vp]
_lib.acsr_peer_read_xs.restype = ctypes.c_int
_lib.acsr_hits_workspace_bytes.argtypes = [_i64]
_lib.acsr_hits_workspace_bytes.restype = _sz
_lib.acsr_hits_normalize.argtypes = [_i64, _vp, _vp, _vp, _vp, _vp, _sz, _vp]
_lib.acsr_hits_normalize.restype = ctypes.c_int
_lib.acsr_hits_normalize_ctrl.argtypes = [_i64, _vp, _vp, _vp, _vp, _vp, _dbl, _vp, _sz, _vp]
_lib.acsr_hits_normalize_ctrl.restype = ctypes.c_int
_lib.acsr_plan_status.argtypes = [_vp, _sz, _vp]
_lib.acsr_plan_status.restype = ctypes.c_int
_lib.acsr_comm_get_unique_id.argtypes = [_vp]
_lib.acsr_comm_get_unique_id.restype = ctypes.c_int
_lib.acsr_comm_init.argtypes = [ctypes.POINTER(_vp), ctypes.c_int, ctypes.c_int, _vp]
_lib.acsr_comm_init.restype = ctypes.c_int
_lib.acsr_comm_destroy.argtypes = [_vp]
_lib.acsr_comm_destroy.restype = ctypes.c_int
_lib.acsr_comm_query.argtypes = [_vp, ctypes.POINTER(ctypes.c_int), ctypes.POINTER(ctypes.c_int)]
_lib.acsr_comm_query.restype = ctypes.c_int
_lib.acsr_comm_allgather.argtypes = [_vp, _vp, _vp, _sz, _vp]
_lib.acsr_comm_allgather.restype = ctypes.c_int
_lib.acsr_comm_allgatherv.argtypes = [_vp, _vp, _vp, _sz, ctypes.POINTER(_i64), _vp]
_lib.acsr_comm_allgatherv.restype = ctypes.c_int
_lib.acsr_pagerank_init.argtypes = [ctypes.POINTER(PrArgs), _vp]
_lib.acsr_pagerank_init.restype = ctypes.c_int
_lib.acsr_partition_workspace_bytes.argtypes = [_i64]
_lib.acsr_partition_workspace_bytes.restype = _sz
_lib.acsr_partition.argtypes = [_i64, _vp, _vp, _i64, _i64, ctypes.c_int, _i64, _vp, _vp, _sz, _vp]
_lib.acsr_partition.restype = ctypes.c_int
_lib.acsr_exchange_layout_workspace_bytes.argtypes = [_i64]
_lib.acsr_exchange_layout_workspace_bytes.restype = _sz
_lib.acsr_exchange_layout.argtypes = [_i64, ctypes.c_int, _vp, _vp, ctypes.c_int, _vp, _vp, _vp, _vp, _vp, _sz, _vp]
_lib.acsr_exchange_layout.restype = ctypes.c_int
_lib.acsr_permute_workspace_bytes.argtypes = [_i64]
_lib.acsr_permute_workspace_bytes.restype = _sz
_lib.acsr_permute_graph.argtypes = [_i64, _vp, _vp, _vp, _vp, _vp, _vp, _vp, _sz, _vp]
_lib.acsr_permute_graph.restype = ctypes.c_int
_lib.acsr_grow_workspace_bytes.argtypes = [_i64]
_lib.acsr_grow_workspace_bytes.restype = _sz
_lib.acsr_grow_layout.argtypes = [_i64, _vp, _vp, _vp, ctypes.c_int32, ctypes.c_int32, _vp, _vp, _vp, _vp, _sz, _vp]
_lib.acsr_grow_layout.restype = ctypes.c_int
_lib.acsr_relabel_workspace_bytes.argtypes = [_i64, _i64, ctypes.c_uint]
_lib.acsr_relabel_workspace_bytes.restype = _sz
_lib.acsr_degree_relabel.argtypes = [_i64, _i64, _vp, _vp, _vp, _vp, _vp, _vp, _vp, ctypes.c_uint, _vp, _sz, _vp]
_lib.acsr_degree_relabel.restype = ctypes.c_int

ACSR_BIN_SHORT_ALG2 = 1  # include/acsr.h: per-bin Alg. 2 units for bins 0..5
ACSR_PEER_MAX = 8
ACSR_IPC_HANDLE_BYTES = 64

EXPORTED = ("acsr_bin_workspace_bytes", "acsr_bin", "acsr_bin_ex", "acsr_spmv", "acsr_pagerank_step",
            "acsr_pagerank_scale", "acsr_pagerank_step_peer", "acsr_peer_create", "acsr_peer_open",
            "acsr_peer_destroy", "acsr_peer_push", "acsr_peer_delta2", "acsr_peer_query", "acsr_peer_read_xs", "acsr_update_workspace_bytes", "acsr_update_edges", "acsr_update_edges_dev", "acsr_relayout",
            "acsr_hits_workspace_bytes", "acsr_hits_normalize", "acsr_hits_normalize_ctrl", "acsr_plan_status",
            "acsr_comm_get_unique_id", "acsr_comm_init", "acsr_comm_destroy", "acsr_comm_query",
            "acsr_comm_allgather", "acsr_comm_allgatherv", "acsr_pagerank_init", "acsr_partition_workspace_bytes", "acsr_partition",
            "acsr_relabel_workspace_bytes", "acsr_degree_relabel", "acsr_grow_workspace_bytes",
            "acsr_grow_layout", "acsr_exchange_layout_workspace_bytes", "acsr_exchange_layout",
            "acsr_permute_workspace_bytes", "acsr_permute_graph",
            "acsr_status_string", "acsr_last_error", "acsr_version")


class ACSRError(RuntimeError):
    def __init__(self, code, what):
        self.code = code
        msg = _lib.acsr_status_string(code).decode()
        detail = (_lib.acsr_last_error() or b"").decode()
        super().__init__(f"{what}: {msg} {detail}")


def _check(code, what):
    if code != ACSR_OK:
        raise ACSRError(code, what)


def _dev(t, dtype, name, allow_none=False):
    if t is None:
        if allow_none:
            return None
        raise TypeError(f"{name} is required")
    if not isinstance(t, torch.Tensor) or not t.is_cuda:
        raise TypeError(f"{name} must be a CUDA tensor (no CPU fallback)")
    if dtype is not None and t.dtype != dtype:
        raise TypeError(f"{name} must be {dtype}, got {t.dtype}")
    if not t.is_contiguous():
        raise TypeError(f"{name} must be contiguous")
    return t.data_ptr()


def _stream(stream):
    s = torch.cuda.current_stream() if stream is None else stream
    return s.cuda_stream


def _dt(t):
    if t.dtype == torch.float64:
        return ACSR_F64
    if t.dtype == torch.float32:
        return ACSR_F32
    raise TypeError(f"unsupported value dtype {t.dtype}")


# --------------------------------------------------------------------------- binning
def acsr_bin_workspace_bytes(n_rows: int, n_cols: int, nnz_max: int) -> int:
    return int(_lib.acsr_bin_workspace_bytes(int(n_rows), int(n_cols), int(nnz_max)))


def acsr_bin(row_begin, row_end=None, nnz_max=None, bin_rows=None, bin_offsets=None, plan_ws=None,
             stream=None, col_idx=None, n_cols=0, short_rows="window"):
    """Bin the rows.  Returns (bin_rows, bin_offsets, plan_ws).  col_idx (with
    n_cols) additionally builds the hot-column table of the SpMV x cache.  short_rows selects
    the SpMV mapping of bins 0..5 recorded in the plan: "window" (default, acsr_bin) or
    "alg2" (the paper's sub-warp per row, acsr_bin_ex(..., ACSR_BIN_SHORT_ALG2))."""
    if short_rows not in ("window", "alg2"):
        raise ValueError(f"short_rows must be 'window' or 'alg2', not {short_rows!r}")
    n = row_begin.numel() - 1 if row_end is None else row_begin.numel()
    dev = row_begin.device
    if nnz_max is None:
        raise TypeError("nnz_max (bound on stored entries) is required")
    if bin_rows is None:
        bin_rows = torch.empty(max(n, 0), dtype=torch.int32, device=dev)
    if bin_offsets is None:
        bin_offsets = torch.empty(NBINS + 1, dtype=torch.int32, device=dev)
    need = acsr_bin_workspace_bytes(n, n_cols, nnz_max)
    if plan_ws is None:
        plan_ws = torch.empty(need, dtype=torch.uint8, device=dev)
    _check(_lib.acsr_bin_ex(n, int(n_cols), int(nnz_max), _dev(row_begin, torch.int32, "row_begin"),
                            _dev(row_end, torch.int32, "row_end", True),
                            _dev(col_idx, torch.int32, "col_idx") if col_idx is not None and col_idx.numel() else None,
                            _dev(bin_rows, torch.int32, "bin_rows") if n > 0 else None,
                            _dev(bin_offsets, torch.int32, "bin_offsets"),
                            _dev(plan_ws, torch.uint8, "plan_ws"), plan_ws.numel(),
                            ACSR_BIN_SHORT_ALG2 if short_rows == "alg2" else 0, _stream(stream)),
           "acsr_bin")
    return bin_rows, bin_offsets, plan_ws


def acsr_plan_status(plan_ws, stream=None):
    """Synchronising health check of a plan (include/acsr.h): raises ACSRError
    (ACSR_ERR_CAPACITY) if acsr_bin's nnz_max understated the stored entries, in which case
    every SpMV / PageRank output of the plan is NaN."""
    _check(_lib.acsr_plan_status(_dev(plan_ws, torch.uint8, "plan_ws"), plan_ws.numel(), _stream(stream)),
           "acsr_plan_status")


ACSR_CTRL_PLAN_ERROR = 2

# --------------------------------------------------------------------------- SpMV
def acsr_spmv(row_begin, col_idx, values, x, bin_rows, bin_offsets, plan_ws, row_end=None, y=None,
              stream=None):
    """y = A x with the bin-specific kernels.  values None => pattern matrix."""
    n = row_begin.numel() - 1 if row_end is None else row_begin.numel()
    if y is None:
        y = torch.empty(n, dtype=x.dtype, device=x.device)
    if values is not None and values.dtype != x.dtype:
        raise TypeError("values and x must have the same dtype")
    _check(_lib.acsr_spmv(_dt(x), n, x.numel(), _dev(row_begin, torch.int32, "row_begin"),
                          _dev(row_end, torch.int32, "row_end", True),
                          _dev(col_idx, torch.int32, "col_idx") if col_idx.numel() else None,
                          _dev(values, x.dtype, "values", True) if values is None or values.numel() else None,
                          _dev(x, x.dtype, "x") if x.numel() else None,
                          _dev(y, x.dtype, "y") if n else None,
                          _dev(bin_rows, torch.int32, "bin_rows") if n else None,
                          _dev(bin_offsets, torch.int32, "bin_offsets"),
                          _dev(plan_ws, torch.uint8, "plan_ws"), plan_ws.numel(), _stream(stream)),
           "acsr_spmv")
    return y


# --------------------------------------------------------------------------- PageRank
def acsr_pagerank_scale(x, outdeg, xs=None, stream=None):
    xs = torch.empty_like(x) if xs is None else xs
    _check(_lib.acsr_pagerank_scale(x.numel(), _dev(x, torch.float64, "x"),
                                    _dev(outdeg, torch.int32, "outdeg"), _dev(xs, torch.float64, "xs"),
                                    _stream(stream)), "acsr_pagerank_scale")
    return xs


def acsr_pagerank_step(row_begin, col_idx, bin_rows, bin_offsets, plan_ws, xs, x, outdeg, x_new,
                       xs_next, delta2, damping=0.85, teleport=None, n_global=None, row_end=None,
                       stream=None, restart=-1, restart_weight=0.0, ctrl=None, eps2=-1.0, comm=None,
                       xs_all=None, slice_len=0, slice_counts=None):
    """One fused PageRank step on the local rows (Alg. 5).  delta2: 1-element float64.
    With teleport=0, damping=c, restart=i, restart_weight=1-c it is an RWR step (Eq. 8).
    comm (AcsrComm): multi-GPU -- the step is followed by the library's exchange: xs_next[:slice_len]
    of every rank all-gathered into xs_all, delta2 = the global Delta^2 (include/acsr.h)."""
    n = row_begin.numel() - 1 if row_end is None else row_begin.numel()
    ng = xs.numel() if n_global is None else n_global
    tel = (1.0 - damping) / ng if teleport is None else teleport
    a = PrArgs(n, xs.numel(), _dev(row_begin, torch.int32, "row_begin"),
               _dev(row_end, torch.int32, "row_end", True),
               _dev(col_idx, torch.int32, "col_idx") if col_idx.numel() else None,
               _dev(bin_rows, torch.int32, "bin_rows") if n else None,
               _dev(bin_offsets, torch.int32, "bin_offsets"), _dev(plan_ws, torch.uint8, "plan_ws"),
               plan_ws.numel(), _dev(xs, torch.float64, "xs") if xs.numel() else None,
               _dev(x, torch.float64, "x") if n else None,
               _dev(outdeg, torch.int32, "outdeg") if n else None,
               _dev(x_new, torch.float64, "x_new") if n else None,
               _dev(xs_next, torch.float64, "xs_next") if n else None, float(damping), float(tel),
               _dev(delta2, torch.float64, "delta2"), int(restart), float(restart_weight),
               _dev(ctrl, torch.int32, "ctrl", True), float(eps2),
               comm._c if comm is not None else None,
               _dev(xs_all, torch.float64, "xs_all") if comm is not None else None, int(slice_len),
               _counts(slice_counts))
    _check(_lib.acsr_pagerank_step(ctypes.byref(a), _stream(stream)), "acsr_pagerank_step")
    return x_new, xs_next, delta2


def _counts(slice_counts):
    """HOST int64 array for acsr_pr_args.slice_counts (kept alive by the caller's list)."""
    if slice_counts is None:
        return None
    arr = (_i64 * len(slice_counts))(*[int(c) for c in slice_counts])
    _counts.keep = arr  # the call is synchronous on the host side; keep until the next call
    return ctypes.cast(arr, ctypes.POINTER(_i64))


def acsr_pagerank_init(x, outdeg, xs_next, comm=None, xs_all=None, slice_len=0, stream=None, slice_counts=None):
    """xs_next[:n] = x / outdeg (first iterate, P:285 / warm start); with comm the
    slices are all-gathered into xs_all (include/acsr.h)."""
    n = x.numel()
    a = PrArgs()
    a.n_rows = n
    a.n_cols = xs_all.numel() if xs_all is not None else n
    a.x = _dev(x, torch.float64, "x") if n else None
    a.outdeg = _dev(outdeg, torch.int32, "outdeg") if n else None
    a.xs_next = _dev(xs_next, torch.float64, "xs_next") if xs_next.numel() else None
    a.comm = comm._c if comm is not None else None
    a.xs_all = _dev(xs_all, torch.float64, "xs_all") if comm is not None else None
    a.slice_len = int(slice_len)
    a.slice_counts = _counts(slice_counts)
    _check(_lib.acsr_pagerank_init(ctypes.byref(a), _stream(stream)), "acsr_pagerank_init")
    return xs_next


# --------------------------------------------------------------------------- multi-GPU
class AcsrComm:
    """Owner of one ``acsr_comm`` (include/acsr.h): the library's NCCL communicator.
    Rank 0's ``unique_id()`` bytes must reach every rank (any host transport) before
    every rank constructs ``AcsrComm(nranks, rank, uid)`` with its GPU current."""

    @staticmethod
    def unique_id() -> bytes:
        buf = ctypes.create_string_buffer(ACSR_COMM_ID_BYTES)
        _check(_lib.acsr_comm_get_unique_id(buf), "acsr_comm_get_unique_id")
        return bytes(buf.raw)

    def __init__(self, nranks: int, rank: int, uid: bytes):
        if len(uid) != ACSR_COMM_ID_BYTES:
            raise ValueError("unique id must be ACSR_COMM_ID_BYTES bytes")
        self._c = _vp()
        buf = ctypes.create_string_buffer(bytes(uid), ACSR_COMM_ID_BYTES)
        _check(_lib.acsr_comm_init(ctypes.byref(self._c), int(nranks), int(rank), buf), "acsr_comm_init")
        self.nranks, self.rank = int(nranks), int(rank)

    @classmethod
    def from_process_group(cls, group=None):
        """Build the communicator over the ranks of a torch.distributed group (the group
        only carries the 128-byte id; the data path is the library's NCCL)."""
        import torch.distributed as dist
        if not dist.is_initialized():
            return cls(1, 0, cls.unique_id())
        rank, world = dist.get_rank(group), dist.get_world_size(group)
        obj = [cls.unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=dist.get_global_rank(group, 0) if group is not None else 0,
                                   group=group)
        return cls(world, rank, obj[0])

    def query(self):
        nr, rk = ctypes.c_int(), ctypes.c_int()
        _check(_lib.acsr_comm_query(self._c, ctypes.byref(nr), ctypes.byref(rk)), "acsr_comm_query")
        return int(nr.value), int(rk.value)

    def allgather(self, send, recv, stream=None):
        """recv (nranks x send.numel(), same dtype) <- every rank's send (in place allowed)."""
        if recv.numel() != self.nranks * send.numel() or recv.dtype != send.dtype:
            raise ValueError("recv must hold nranks * send.numel() elements of send's dtype")
        _check(_lib.acsr_comm_allgather(self._c, _dev(send, None, "send") if send.numel() else None,
                                        _dev(recv, None, "recv") if recv.numel() else None,
                                        send.numel() * send.element_size(), _stream(stream)),
               "acsr_comm_allgather")
        return recv

    def allgatherv(self, send, recv, counts, stream=None):
        """recv viewed as nranks slices of recv.numel() // nranks elements; slice q receives
        counts[q] elements of rank q's send (acsr_comm_allgatherv)."""
        es = recv.element_size()
        stride = recv.numel() // self.nranks * es
        arr = (_i64 * self.nranks)(*[int(c) * es for c in counts])
        _check(_lib.acsr_comm_allgatherv(self._c, _dev(send, None, "send") if send.numel() else None,
                                         _dev(recv, None, "recv") if recv.numel() else None, stride, arr,
                                         _stream(stream)), "acsr_comm_allgatherv")
        return recv

    def close(self):
        if self._c:
            _check(_lib.acsr_comm_destroy(self._c), "acsr_comm_destroy")
            self._c = _vp()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


ACSR_RELABEL_SORT_ROWS = 1


def acsr_exchange_layout(nd, splits, rank=-1, stream=None):
    """Compact exchange layout (include/acsr.h).  nd: CUDA uint8 [n_global] non-dangling mask;
    splits: CUDA int64 [P + 1].  Returns (pos int32 [n_global], order int32 [local rows] or None,
    counts int64 [P] (host list), Lx int)."""
    n = nd.numel()
    P = splits.numel() - 1
    dev = nd.device
    pos = torch.empty(n, dtype=torch.int32, device=dev)
    counts = torch.empty(P, dtype=torch.int64, device=dev)
    lx = torch.empty(1, dtype=torch.int64, device=dev)
    order = None
    if rank >= 0:
        sp = splits.cpu()
        order = torch.empty(int(sp[rank + 1] - sp[rank]), dtype=torch.int32, device=dev)
    ws = torch.empty(int(_lib.acsr_exchange_layout_workspace_bytes(n)), dtype=torch.uint8, device=dev)
    _check(_lib.acsr_exchange_layout(n, P, _dev(splits, torch.int64, "splits"),
                                     _dev(nd, torch.uint8, "nd") if n else None, int(rank),
                                     _dev(pos, torch.int32, "pos") if n else None,
                                     _dev(order, torch.int32, "order") if order is not None and order.numel() else None,
                                     _dev(counts, torch.int64, "counts"), _dev(lx, torch.int64, "lx"),
                                     _dev(ws, torch.uint8, "ws"), ws.numel(), _stream(stream)), "acsr_exchange_layout")
    return pos, order, [int(c) for c in counts.cpu()], int(lx.item())


def acsr_permute_graph(row_ptr, col_idx, order, col_map=None, stream=None):
    """Rows reordered (new row i = old row order[i]), columns mapped through col_map."""
    n = row_ptr.numel() - 1
    dev = row_ptr.device
    rp2 = torch.empty(n + 1, dtype=torch.int32, device=dev)
    c2 = torch.empty_like(col_idx)
    ws = torch.empty(int(_lib.acsr_permute_workspace_bytes(n)), dtype=torch.uint8, device=dev)
    _check(_lib.acsr_permute_graph(n, _dev(row_ptr, torch.int32, "row_ptr"),
                                   _dev(col_idx, torch.int32, "col_idx") if col_idx.numel() else None,
                                   _dev(order, torch.int32, "order") if n else None,
                                   _dev(col_map, torch.int32, "col_map", True), _dev(rp2, torch.int32, "row_ptr_out"),
                                   _dev(c2, torch.int32, "col_out") if c2.numel() else None,
                                   _dev(ws, torch.uint8, "ws"), ws.numel(), _stream(stream)), "acsr_permute_graph")
    return rp2, c2


def acsr_grow_layout(row_begin, row_end, row_cap, min_slack=8, frac=2, stream=None):
    """Reading R4's grown layout on the device.  Returns (new_begin, new_cap, total) with
    total an int (synchronising read: the caller sizes the new col / val arrays with it)."""
    n = row_begin.numel()
    dev = row_begin.device
    nb = torch.empty(n, dtype=torch.int32, device=dev)
    nc = torch.empty(n, dtype=torch.int32, device=dev)
    tot = torch.zeros(1, dtype=torch.int64, device=dev)
    ws = torch.empty(int(_lib.acsr_grow_workspace_bytes(n)), dtype=torch.uint8, device=dev)
    _check(_lib.acsr_grow_layout(n, _dev(row_begin, torch.int32, "row_begin") if n else None,
                                 _dev(row_end, torch.int32, "row_end") if n else None,
                                 _dev(row_cap, torch.int32, "row_cap") if n else None, int(min_slack), int(frac),
                                 _dev(nb, torch.int32, "new_begin") if n else None,
                                 _dev(nc, torch.int32, "new_cap") if n else None, _dev(tot, torch.int64, "total"),
                                 _dev(ws, torch.uint8, "ws"), ws.numel(), _stream(stream)), "acsr_grow_layout")
    return nb, nc, int(tot.item())


def acsr_degree_relabel(row_ptr, col_idx, outdeg, sort_rows=False, stream=None):
    """Degree-ordered relabelling on the device (include/acsr.h).  Returns
    (row_ptr', col', outdeg', perm) with perm[v] = new id of vertex v (int32).
    sort_rows: columns of every new row sorted ascending (ACSR_RELABEL_SORT_ROWS)."""
    n = row_ptr.numel() - 1
    dev = row_ptr.device
    nnz = col_idx.numel() if col_idx is not None else 0
    flags = ACSR_RELABEL_SORT_ROWS if sort_rows else 0
    rp2 = torch.empty(n + 1, dtype=torch.int32, device=dev)
    c2 = torch.empty_like(col_idx) if col_idx is not None else None
    od2 = torch.empty(n, dtype=torch.int32, device=dev)
    perm = torch.empty(n, dtype=torch.int32, device=dev)
    ws = torch.empty(int(_lib.acsr_relabel_workspace_bytes(n, nnz, flags)), dtype=torch.uint8, device=dev)
    _check(_lib.acsr_degree_relabel(n, nnz, _dev(row_ptr, torch.int32, "row_ptr"),
                                    _dev(col_idx, torch.int32, "col_idx") if c2 is not None and c2.numel() else None,
                                    _dev(outdeg, torch.int32, "outdeg") if n else None,
                                    _dev(rp2, torch.int32, "row_ptr_out"),
                                    _dev(c2, torch.int32, "col_out") if c2 is not None and c2.numel() else None,
                                    _dev(od2, torch.int32, "outdeg_out") if n else None,
                                    _dev(perm, torch.int32, "perm_out") if n else None, flags,
                                    _dev(ws, torch.uint8, "ws"), ws.numel(), _stream(stream)), "acsr_degree_relabel")
    return rp2, c2, od2, perm


def acsr_partition(row_begin, nranks, b_nnz, b_row, row_end=None, align=1, stream=None):
    """O8 split points on the device (int64 CUDA tensor [nranks + 1]), rounded up to a
    multiple of `align` (reading R7)."""
    n = row_begin.numel() - 1 if row_end is None else row_begin.numel()
    dev = row_begin.device
    splits = torch.empty(int(nranks) + 1, dtype=torch.int64, device=dev)
    ws = torch.empty(int(_lib.acsr_partition_workspace_bytes(n)), dtype=torch.uint8, device=dev)
    _check(_lib.acsr_partition(n, _dev(row_begin, torch.int32, "row_begin") if n else None,
                               _dev(row_end, torch.int32, "row_end", True), int(b_nnz), int(b_row), int(nranks),
                               int(align), _dev(splits, torch.int64, "splits"), _dev(ws, torch.uint8, "ws"), ws.numel(),
                               _stream(stream)), "acsr_partition")
    return splits


# --------------------------------------------------------------------------- peer exchange
class AcsrPeer:
    """Owner of one ``acsr_peer`` (include/acsr.h): the library-owned region holding this
    rank's replicated xs double buffer and exchange flags, mapped into every other rank.
    Protocol: ``handle`` (64 host bytes) -> caller all-gathers -> ``open(handles)``."""

    def __init__(self, nranks, rank, xs_len, slice_off, slice_len):
        self._p = _vp()
        self.handle = ctypes.create_string_buffer(ACSR_IPC_HANDLE_BYTES)
        _check(_lib.acsr_peer_create(ctypes.byref(self._p), int(nranks), int(rank), int(xs_len),
                                     int(slice_off), int(slice_len), self.handle), "acsr_peer_create")
        self.nranks, self.rank, self.xs_len = int(nranks), int(rank), int(xs_len)
        self.slice_off, self.slice_len = int(slice_off), int(slice_len)

    def handle_bytes(self) -> bytes:
        return bytes(self.handle.raw)

    def open(self, handles):
        """handles: list of every rank's handle_bytes() in rank order."""
        if len(handles) != self.nranks:
            raise ValueError("one handle per rank")
        buf = ctypes.create_string_buffer(b"".join(bytes(h) for h in handles), ACSR_IPC_HANDLE_BYTES * self.nranks)
        _check(_lib.acsr_peer_open(self._p, buf), "acsr_peer_open")

    def push(self, x, outdeg, xs_local=None, stream=None):
        n = x.numel()
        _check(_lib.acsr_peer_push(self._p, n, _dev(x, torch.float64, "x") if n else None,
                                   _dev(outdeg, torch.int32, "outdeg") if n else None,
                                   _dev(xs_local, torch.float64, "xs_local", True), _stream(stream)),
               "acsr_peer_push")

    def delta2(self, out, ctrl=None, eps2=-1.0, stream=None):
        _check(_lib.acsr_peer_delta2(self._p, _dev(out, torch.float64, "delta2"),
                                     _dev(ctrl, torch.int32, "ctrl", True), float(eps2), _stream(stream)),
               "acsr_peer_delta2")
        return out

    def query(self):
        """(pushes, error word, device address of the buffer holding the last push)."""
        pushes, err, ptr = _i64(), ctypes.c_int32(), _vp()
        _check(_lib.acsr_peer_query(self._p, ctypes.byref(pushes), ctypes.byref(err), ctypes.byref(ptr)),
               "acsr_peer_query")
        return int(pushes.value), int(err.value), ptr.value

    def read_xs(self, out=None, stream=None):
        """This rank's replicated xs as left by the last push (enqueued copy)."""
        if out is None:
            out = torch.empty(self.xs_len, dtype=torch.float64, device="cuda")
        _check(_lib.acsr_peer_read_xs(self._p, _dev(out, torch.float64, "out"), _stream(stream)),
               "acsr_peer_read_xs")
        return out

    def close(self):
        if self._p:
            _check(_lib.acsr_peer_destroy(self._p), "acsr_peer_destroy")
            self._p = _vp()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def acsr_pagerank_step_peer(peer: AcsrPeer, row_begin, col_idx, bin_rows, bin_offsets, plan_ws, x, outdeg,
                            x_new, xs_next, delta2, damping=0.85, teleport=None, n_global=None, row_end=None,
                            stream=None, ctrl=None, eps2=-1.0):
    """One fused PageRank step whose xs' slice is stored straight into every rank's
    replicated xs (peer memory); reads the xs of the previous push.  xs_next may be None
    (no local copy).  delta2 receives this rank's partial; the global one comes from
    peer.delta2().  With ctrl, the step is a no-op once the global Delta^2 of the previous
    step is <= eps2 (ctrl[0] set, identically on every rank)."""
    n = row_begin.numel() - 1 if row_end is None else row_begin.numel()
    ng = peer.xs_len if n_global is None else n_global
    tel = (1.0 - damping) / ng if teleport is None else teleport
    a = PrArgs(n, peer.xs_len, _dev(row_begin, torch.int32, "row_begin"),
               _dev(row_end, torch.int32, "row_end", True),
               _dev(col_idx, torch.int32, "col_idx") if col_idx.numel() else None,
               _dev(bin_rows, torch.int32, "bin_rows") if n else None,
               _dev(bin_offsets, torch.int32, "bin_offsets"), _dev(plan_ws, torch.uint8, "plan_ws"),
               plan_ws.numel(), None, _dev(x, torch.float64, "x") if n else None,
               _dev(outdeg, torch.int32, "outdeg") if n else None,
               _dev(x_new, torch.float64, "x_new") if n else None,
               _dev(xs_next, torch.float64, "xs_next", True) if n else None, float(damping), float(tel),
               _dev(delta2, torch.float64, "delta2"), -1, 0.0, _dev(ctrl, torch.int32, "ctrl", True), float(eps2))
    _check(_lib.acsr_pagerank_step_peer(ctypes.byref(a), peer._p, _stream(stream)), "acsr_pagerank_step_peer")
    return x_new, delta2


# --------------------------------------------------------------------------- update
def acsr_update_workspace_bytes(n_upd: int) -> int:
    return int(_lib.acsr_update_workspace_bytes(int(n_upd)))


def acsr_update_edges(n_cols, row_begin, row_end, row_cap, col_idx, values, upd_rows, ins_ptr,
                      ins_cols, ins_vals=None, del_ptr=None, del_cols=None, outdeg=None, status=None,
                      ws=None, dtype=torch.float64, stream=None, n_upd_dev=None):
    """Apply one change batch in place (§VII).  Returns the device status tensor [code, index].
    n_upd_dev (1-element int64 CUDA tensor): the batch size is read on the device and
    upd_rows/ins_ptr/... are capacity buffers (acsr_update_edges_dev, graph-capturable)."""
    n = row_begin.numel()
    dev = row_begin.device
    n_upd = upd_rows.numel()
    if status is None:
        status = torch.empty(2, dtype=torch.int32, device=dev)
    if ws is None:
        ws = torch.empty(acsr_update_workspace_bytes(n_upd), dtype=torch.uint8, device=dev)
    vdt = values.dtype if values is not None else dtype
    if del_ptr is not None and (del_cols is None or del_cols.numel() == 0):
        del_ptr, del_cols = None, None  # insert-only batch
    dt = ACSR_F64 if vdt == torch.float64 else ACSR_F32
    opt = lambda t, d, nm: (_dev(t, d, nm) if t is not None and t.numel() else None)
    if n_upd_dev is not None:
        _check(_lib.acsr_update_edges_dev(dt, n, int(n_cols), _dev(row_begin, torch.int32, "row_begin"),
                                          _dev(row_end, torch.int32, "row_end"),
                                          _dev(row_cap, torch.int32, "row_cap"),
                                          _dev(col_idx, torch.int32, "col_idx"), opt(values, vdt, "values"), n_upd,
                                          _dev(n_upd_dev, torch.int64, "n_upd_dev"),
                                          opt(upd_rows, torch.int32, "upd_rows"),
                                          _dev(del_ptr, torch.int32, "del_ptr", True),
                                          opt(del_cols, torch.int32, "del_cols") if del_ptr is not None else None,
                                          opt(ins_ptr, torch.int32, "ins_ptr"), opt(ins_cols, torch.int32, "ins_cols"),
                                          opt(ins_vals, vdt, "ins_vals"), _dev(outdeg, torch.int32, "outdeg", True),
                                          _dev(status, torch.int32, "status"), _dev(ws, torch.uint8, "ws"),
                                          ws.numel(), _stream(stream)), "acsr_update_edges_dev")
        return status
    _check(_lib.acsr_update_edges(dt, n, int(n_cols), _dev(row_begin, torch.int32, "row_begin"),
                                  _dev(row_end, torch.int32, "row_end"), _dev(row_cap, torch.int32, "row_cap"),
                                  _dev(col_idx, torch.int32, "col_idx"), opt(values, vdt, "values"), n_upd,
                                  opt(upd_rows, torch.int32, "upd_rows"),
                                  _dev(del_ptr, torch.int32, "del_ptr", True),
                                  opt(del_cols, torch.int32, "del_cols") if del_ptr is not None else None,
                                  opt(ins_ptr, torch.int32, "ins_ptr"), opt(ins_cols, torch.int32, "ins_cols"),
                                  opt(ins_vals, vdt, "ins_vals"), _dev(outdeg, torch.int32, "outdeg", True),
                                  _dev(status, torch.int32, "status"), _dev(ws, torch.uint8, "ws"), ws.numel(),
                                  _stream(stream)), "acsr_update_edges")
    return status


def acsr_relayout(old_begin, old_end, old_col, old_val, new_begin, new_end, new_col, new_val,
                  dtype=torch.float64, stream=None):
    """Copy every row of a slack CSR into a new layout (after a CAPACITY rejection)."""
    n = old_begin.numel()
    vdt = old_val.dtype if old_val is not None else dtype
    dt = ACSR_F64 if vdt == torch.float64 else ACSR_F32
    _check(_lib.acsr_relayout(dt, n, _dev(old_begin, torch.int32, "old_begin"),
                              _dev(old_end, torch.int32, "old_end"), _dev(old_col, torch.int32, "old_col"),
                              _dev(old_val, vdt, "old_val", True), _dev(new_begin, torch.int32, "new_begin"),
                              _dev(new_end, torch.int32, "new_end"), _dev(new_col, torch.int32, "new_col"),
                              _dev(new_val, vdt, "new_val", True), _stream(stream)), "acsr_relayout")
    return new_end


def acsr_hits_workspace_bytes(n: int) -> int:
    return int(_lib.acsr_hits_workspace_bytes(int(n)))


def acsr_hits_normalize(y, v, v_next, dist2, ws=None, stream=None, ctrl=None, eps2=-1.0):
    """HITS normalisation of y = [A^T h; A a] into v_next (Eq. 5-7, reading R6).  ctrl:
    device-side convergence (acsr_hits_normalize_ctrl)."""
    n = y.numel() // 2
    if ws is None:
        ws = torch.empty(acsr_hits_workspace_bytes(n), dtype=torch.uint8, device=y.device)
    _check(_lib.acsr_hits_normalize_ctrl(n, _dev(y, torch.float64, "y"), _dev(v, torch.float64, "v"),
                                         _dev(v_next, torch.float64, "v_next"), _dev(dist2, torch.float64, "dist2"),
                                         _dev(ctrl, torch.int32, "ctrl", True), float(eps2),
                                         _dev(ws, torch.uint8, "ws"), ws.numel(), _stream(stream)),
           "acsr_hits_normalize")
    return v_next, dist2


def version() -> int:
    return int(_lib.acsr_version())


from .matrix import (ACSRMatrix, UpdateGraph, degree_relabel, hits, hits_matrix, pagerank, rwr,  # noqa: E402
                     spmv_from_host)
