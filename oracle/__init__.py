"""CPU oracle for the ACSR hot path (Ashari et al., SC'14) -- TEST INFRASTRUCTURE.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  The product package
``paper_conf_sc_ashariseps14_b200`` never imports it and shares no code with it.

The arithmetic lives in ``acsr_oracle.c`` (plain sequential C, compiled with
``-O2 -ffp-contract=off``); this module is argument marshalling over numpy
arrays (host memory).  Function-level citations are in the C file:

* ``bin_of``            O2, P:51 / P:64 (§III-A bin ranges)
* ``bins``              O3, P:47 (Alg. 1) + reading Q3 (stable order)
* ``spmv``              O4, P:19 / P:59 (Alg. 2) -- Dot2 parity path + ``den``
* ``spmv_plain``        O4', the timed plain sequential SpMV (cpu_baseline)
* ``pagerank_step``     O6, P:279-291 (Alg. 5) with readings Q11/Q12
* ``pagerank``          O6', P:285-289, P:297, P:326 with reading Q9
* ``rwr_step``/``rwr``   Eq. 8, P:318-324 (RWR) with reading R5
* ``hits_step``/``hits`` Eq. 5-7, P:299-317 (HITS) with reading R6
* ``update``            O7, P:334-335 (§VII) with reading Q13
* ``partition``         O8, replaces P:345 (reading Q19)
* ``csr_build``         O1, P:30 (§II)
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "acsr_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

OK = 0
ERR_INVALID_VALUE = 1
ERR_CAPACITY = 3


def build_oracle(force: bool = False) -> str:
    """Compile liboracle.so with gcc (plain C, OpenMP only for the timed variant)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        cmd = ["gcc", "-O2", "-ffp-contract=off", "-fno-fast-math", "-std=c11", "-fPIC",
               "-shared", "-fopenmp", "-o", _LIB, _SRC, "-lm"]
        subprocess.check_call(cmd)
    return _LIB


_lib = None


def _L():
    global _lib
    if _lib is None:
        build_oracle()
        _lib = ctypes.CDLL(_LIB)
        i64, i32p, vp, dp = ctypes.c_int64, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_double
        _lib.oracle_bin_of.argtypes = [i64]
        _lib.oracle_bin_of.restype = ctypes.c_int
        _lib.oracle_bins.argtypes = [i64, i32p, i32p, i32p, i32p]
        for f in ("oracle_spmv_f64", "oracle_spmv_f32"):
            getattr(_lib, f).argtypes = [i64, i32p, i32p, i32p, vp, vp, vp, vp]
        for f in ("oracle_spmv_plain_f64", "oracle_spmv_plain_f32"):
            getattr(_lib, f).argtypes = [i64, i32p, i32p, i32p, vp, vp, vp, ctypes.c_int]
        _lib.oracle_pagerank_step.argtypes = [i64, i32p, i32p, i32p, i32p, vp, dp, dp, vp]
        _lib.oracle_pagerank_step.restype = ctypes.c_double
        _lib.oracle_pagerank.argtypes = [i64, i32p, i32p, i32p, i32p, vp, dp, dp, dp, ctypes.c_int,
                                         vp, vp]
        _lib.oracle_pagerank.restype = ctypes.c_int
        _lib.oracle_rwr_step.argtypes = [i64, i32p, i32p, i32p, i32p, vp, dp, i64, vp]
        _lib.oracle_rwr_step.restype = ctypes.c_double
        _lib.oracle_rwr.argtypes = [i64, i32p, i32p, i32p, i32p, vp, dp, i64, dp, ctypes.c_int, vp, vp]
        _lib.oracle_rwr.restype = ctypes.c_int
        _lib.oracle_hits_step.argtypes = [i64, i32p, i32p, i32p, i32p, vp, vp, vp, vp, vp]
        _lib.oracle_hits.argtypes = [i64, i32p, i32p, i32p, i32p, vp, vp, dp, ctypes.c_int, vp]
        _lib.oracle_hits.restype = ctypes.c_int
        _lib.oracle_update.argtypes = [i64, i64, i32p, i32p, i32p, i32p, vp, ctypes.c_int, i64,
                                       i32p, i32p, i32p, i32p, i32p, vp, i32p, i32p]
        _lib.oracle_update.restype = ctypes.c_int
        _lib.oracle_partition.argtypes = [i64, i32p, i32p, i64, i64, ctypes.c_int, i64, vp]
        _lib.oracle_csr_build.argtypes = [i64, i64, i32p, i32p, vp, ctypes.c_int, ctypes.c_int,
                                          i32p, i32p, vp]
        _lib.oracle_csr_build.restype = i64
    return _lib


def _p(a):
    """Pointer of a C-contiguous numpy array (None -> NULL)."""
    if a is None:
        return None
    assert isinstance(a, np.ndarray) and a.flags["C_CONTIGUOUS"], "oracle needs contiguous numpy"
    return a.ctypes.data


def _i32(a):
    return None if a is None else np.ascontiguousarray(a, dtype=np.int32)


def bin_of(length: int) -> int:
    return int(_L().oracle_bin_of(int(length)))


def bins(row_begin, row_end=None):
    """Returns (bin_rows int32[n], bin_offsets int32[33]).  row_end None => standard CSR."""
    rb = _i32(row_begin)
    re = _i32(row_end)
    n = rb.size - 1 if re is None else rb.size
    bin_rows = np.empty(max(n, 0), np.int32)
    off = np.empty(33, np.int32)
    _L().oracle_bins(n, _p(rb), _p(re), _p(bin_rows), _p(off))
    return bin_rows, off


def _n_rows(rb, re):
    return rb.size - 1 if re is None else rb.size


def spmv(row_begin, col, val, x, row_end=None):
    """Dot2 parity SpMV.  Returns (y, den) with y in the dtype of x."""
    rb, re, c = _i32(row_begin), _i32(row_end), _i32(col)
    n = _n_rows(rb, re)
    x = np.ascontiguousarray(x)
    den = np.empty(n, np.float64)
    if x.dtype == np.float64:
        v = None if val is None else np.ascontiguousarray(val, np.float64)
        y = np.empty(n, np.float64)
        _L().oracle_spmv_f64(n, _p(rb), _p(re), _p(c), _p(v), _p(x), _p(y), _p(den))
    elif x.dtype == np.float32:
        v = None if val is None else np.ascontiguousarray(val, np.float32)
        y = np.empty(n, np.float32)
        _L().oracle_spmv_f32(n, _p(rb), _p(re), _p(c), _p(v), _p(x), _p(y), _p(den))
    else:
        raise TypeError(x.dtype)
    return y, den


def spmv_plain(row_begin, col, val, x, row_end=None, threads: int = 1, out=None):
    """The timed plain sequential SpMV (O4')."""
    rb, re, c = _i32(row_begin), _i32(row_end), _i32(col)
    n = _n_rows(rb, re)
    x = np.ascontiguousarray(x)
    y = out if out is not None else np.empty(n, x.dtype)
    f = _L().oracle_spmv_plain_f64 if x.dtype == np.float64 else _L().oracle_spmv_plain_f32
    v = None if val is None else np.ascontiguousarray(val, x.dtype)
    f(n, _p(rb), _p(re), _p(c), _p(v), _p(x), _p(y), int(threads))
    return y


def pagerank_step(row_begin, col, outdeg, x, teleport, d, row_end=None):
    rb, re, c, od = _i32(row_begin), _i32(row_end), _i32(col), _i32(outdeg)
    n = _n_rows(rb, re)
    x = np.ascontiguousarray(x, np.float64)
    xn = np.empty(n, np.float64)
    d2 = _L().oracle_pagerank_step(n, _p(rb), _p(re), _p(c), _p(od), _p(x), float(teleport),
                                   float(d), _p(xn))
    return xn, float(d2)


def pagerank(row_begin, col, outdeg, x0=None, d=0.85, eps=1e-6, max_iter=1000, row_end=None,
             teleport=None):
    """Alg. 5 power iteration.  Returns (x, iterations, last_delta2)."""
    rb, re, c, od = _i32(row_begin), _i32(row_end), _i32(col), _i32(outdeg)
    n = _n_rows(rb, re)
    x = np.full(n, 1.0 / n) if x0 is None else np.array(x0, np.float64, copy=True)
    if teleport is None:
        teleport = (1.0 - d) / n
    work = np.empty(n, np.float64)
    d2 = np.zeros(1, np.float64)
    it = _L().oracle_pagerank(n, _p(rb), _p(re), _p(c), _p(od), _p(x), float(teleport), float(d),
                              float(eps), int(max_iter), _p(work), _p(d2))
    return x, int(it), float(d2[0])


def rwr_step(row_begin, col, outdeg, r, c, restart, row_end=None):
    """Eq. 8 step (reading R5).  Returns (r_new, delta2)."""
    rb, re, cc, od = _i32(row_begin), _i32(row_end), _i32(col), _i32(outdeg)
    n = _n_rows(rb, re)
    r = np.ascontiguousarray(r, np.float64)
    rn = np.empty(n, np.float64)
    d2 = _L().oracle_rwr_step(n, _p(rb), _p(re), _p(cc), _p(od), _p(r), float(c), int(restart), _p(rn))
    return rn, float(d2)


def rwr(row_begin, col, outdeg, restart, c=0.85, eps=1e-6, max_iter=1000, row_end=None, r0=None):
    """Eq. 8 loop from r^0 = e_i.  Returns (r, iterations, last_delta2)."""
    rb, re, cc, od = _i32(row_begin), _i32(row_end), _i32(col), _i32(outdeg)
    n = _n_rows(rb, re)
    if r0 is None:
        r = np.zeros(n, np.float64)
        r[restart] = 1.0
    else:
        r = np.array(r0, np.float64, copy=True)
    work = np.empty(n, np.float64)
    d2 = np.zeros(1, np.float64)
    it = _L().oracle_rwr(n, _p(rb), _p(re), _p(cc), _p(od), _p(r), float(c), int(restart), float(eps),
                         int(max_iter), _p(work), _p(d2))
    return r, int(it), float(d2[0])


def hits_step(out_ptr, out_col, in_ptr, in_col, a, h):
    """Eq. 5-7 step with reading R6 (unit L2 norm).  Returns (a', h', [da2, dh2])."""
    op, oc, ip, ic = (_i32(t) for t in (out_ptr, out_col, in_ptr, in_col))
    n = op.size - 1
    a = np.ascontiguousarray(a, np.float64)
    h = np.ascontiguousarray(h, np.float64)
    an, hn, d2 = np.empty(n), np.empty(n), np.empty(2)
    _L().oracle_hits_step(n, _p(op), _p(oc), _p(ip), _p(ic), _p(a), _p(h), _p(an), _p(hn), _p(d2))
    return an, hn, d2


def hits(out_ptr, out_col, in_ptr, in_col, eps=1e-6, max_iter=1000):
    """Eq. 5-7 loop from a = h = 1/|V|.  Returns (a, h, iterations)."""
    op, oc, ip, ic = (_i32(t) for t in (out_ptr, out_col, in_ptr, in_col))
    n = op.size - 1
    a = np.full(n, 1.0 / n)
    h = np.full(n, 1.0 / n)
    work = np.empty(2 * n)
    it = _L().oracle_hits(n, _p(op), _p(oc), _p(ip), _p(ic), _p(a), _p(h), float(eps), int(max_iter),
                          _p(work))
    return a, h, int(it)


def update(n_cols, row_begin, row_end, row_cap, col, val, upd_rows, del_ptr, del_cols, ins_ptr,
           ins_cols, ins_vals=None, outdeg=None):
    """In-place update of (row_end, col, val, outdeg) numpy arrays.  Returns (code, fail_idx)."""
    for a in (row_end, col, outdeg):
        assert a is None or (a.dtype == np.int32 and a.flags["C_CONTIGUOUS"])
    rb, cap = _i32(row_begin), _i32(row_cap)
    n = rb.size
    vb = 0 if val is None else val.dtype.itemsize
    iv = None if ins_vals is None else np.ascontiguousarray(ins_vals, val.dtype)
    ur, dp_, dc, ip, ic = (_i32(a) for a in (upd_rows, del_ptr, del_cols, ins_ptr, ins_cols))
    st = np.zeros(2, np.int32)
    _L().oracle_update(n, int(n_cols), _p(rb), _p(row_end), _p(cap), _p(col), _p(val), vb,
                       ur.size, _p(ur), _p(dp_), _p(dc), _p(ip), _p(ic), _p(iv), _p(outdeg),
                       _p(st))
    return int(st[0]), int(st[1])


def partition(row_begin, P, b_nnz, b_row, row_end=None, align=1):
    rb, re = _i32(row_begin), _i32(row_end)
    n = _n_rows(rb, re)
    s = np.empty(P + 1, np.int64)
    _L().oracle_partition(n, _p(rb), _p(re), int(b_nnz), int(b_row), int(P), int(align), _p(s))
    return s


def csr_build(n_rows, rows, cols, vals=None, dedup=False):
    """Edge list -> (row_ptr, col, val) (stable (row, col) order)."""
    r, c = _i32(rows), _i32(cols)
    m = r.size
    rp = np.empty(n_rows + 1, np.int32)
    oc = np.empty(max(m, 1), np.int32)
    vb = 0 if vals is None else vals.dtype.itemsize
    vv = None if vals is None else np.ascontiguousarray(vals)
    ov = None if vals is None else np.empty(max(m, 1), vals.dtype)
    nnz = _L().oracle_csr_build(int(n_rows), m, _p(r), _p(c), _p(vv), vb, int(bool(dedup)),
                                _p(rp), _p(oc), _p(ov))
    return rp, oc[:nnz].copy(), (None if ov is None else ov[:nnz].copy())
