"""Seeded synthetic inputs shared by the oracle tests, the GPU tests and bench.py.

This module holds NO arithmetic of the method (no binning, no SpMV, no PageRank,
no update); it only draws matrices, vectors and change lists.  Every random
number comes from a counter-based hash (splitmix64 of (seed, stream, index)),
written with integer tensor ops so the same draw is produced on CPU and on GPU.

Generators (recipes in DESIGN.md §"Inputs"):

* ``rmat_edges`` / ``rmat_csr`` -- Graph500 R-MAT (a,b,c,d) = (0.57, 0.19, 0.19,
  0.05), edge factor 16, no noise, seeded random vertex permutation, duplicate
  edges removed, self-loops kept.  Shapes match the paper's power-law graphs
  (Table I; configs C1/C2/C4 of BASELINE.json).
* ``powerlaw_csr`` -- rows with truncated discrete power-law lengths and
  power-law column popularity (web-Google-like / LiveJournal-like, C3).
* ``boundary_csr`` -- one row per length in {0,1,2,3,4,5,8,9,...,2^k+1}: every
  bin edge of §III-A is exercised.
* ``values`` / ``vector`` -- U(-1,1) floats or integers in [-8, 8].
* ``insert_batches`` -- C5 edge-insertion batches encoded as per-row change
  lists "in CSR format", plus ``with_slack`` (P:334 reserved space).
"""
from __future__ import annotations

import numpy as np
import torch

_M64 = (1 << 64) - 1


def _s64(v: int) -> int:
    """Python int (mod 2^64) -> signed int64 value with the same bits."""
    v &= _M64
    return v - (1 << 64) if v >= (1 << 63) else v


_G = _s64(0x9E3779B97F4A7C15)
_C1 = _s64(0xBF58476D1CE4E5B9)
_C2 = _s64(0x94D049BB133111EB)


def _srl(x: torch.Tensor, k: int) -> torch.Tensor:
    """Logical right shift of int64 bit patterns."""
    return (x >> k) & ((1 << (64 - k)) - 1)


def _mix(z: torch.Tensor) -> torch.Tensor:
    z = z + _G
    z = (z ^ _srl(z, 30)) * _C1
    z = (z ^ _srl(z, 27)) * _C2
    return z ^ _srl(z, 31)


def _mix_int(v: int) -> int:
    z = (v + 0x9E3779B97F4A7C15) & _M64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & _M64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & _M64
    return z ^ (z >> 31)


def hash64(seed: int, stream: int, idx: torch.Tensor) -> torch.Tensor:
    """splitmix64(key(seed, stream) + idx) as int64 bit patterns."""
    key = _s64(_mix_int(_mix_int(seed & _M64) ^ ((stream * 0x100000001B3) & _M64)))
    return _mix(idx.to(torch.int64) + key)


def uniform53(h: torch.Tensor) -> torch.Tensor:
    """Top 53 bits of the hash as a float64 in [0, 1) (exact on every device)."""
    return _srl(h, 11).to(torch.float64) * (2.0 ** -53)


def _dev(device):
    return torch.device(device) if device is not None else torch.device("cpu")


# --------------------------------------------------------------------------- R-MAT
RMAT_ABCD = (0.57, 0.19, 0.19, 0.05)
_STREAM_LEVEL = 1000
_STREAM_PERM = 7
_STREAM_VAL = 11
_STREAM_X = 13


def rmat_perm(scale: int, seed: int, device=None) -> torch.Tensor:
    """Random vertex relabelling: new_id[v] (stable sort of per-vertex hashes)."""
    dev = _dev(device)
    n = 1 << scale
    v = torch.arange(n, device=dev, dtype=torch.int64)
    keys = _srl(hash64(seed, _STREAM_PERM, v), 1)  # non-negative for a signed sort
    order = torch.sort(keys, stable=True).indices
    new_id = torch.empty(n, dtype=torch.int64, device=dev)
    new_id[order] = v
    return new_id


def rmat_edges(scale: int, edge_factor: int = 16, seed: int = 1, device=None,
               first_edge: int = 0, n_edges: int | None = None, new_id=None,
               chunk: int = 1 << 25):
    """Raw (src, dst) R-MAT edges [first_edge, first_edge + n_edges) as int64 tensors
    (duplicates included), relabelled with ``rmat_perm``."""
    dev = _dev(device)
    n_edges = (edge_factor << scale) if n_edges is None else n_edges
    a, b, c, _ = RMAT_ABCD
    ta = int(a * 2 ** 53)
    tab = int((a + b) * 2 ** 53)
    tabc = int((a + b + c) * 2 ** 53)
    if new_id is None:
        new_id = rmat_perm(scale, seed, dev)
    srcs, dsts = [], []
    for e0 in range(first_edge, first_edge + n_edges, chunk):
        e = torch.arange(e0, min(e0 + chunk, first_edge + n_edges), device=dev, dtype=torch.int64)
        src = torch.zeros_like(e)
        dst = torch.zeros_like(e)
        for lvl in range(scale):
            u = _srl(hash64(seed, _STREAM_LEVEL + lvl, e), 11)
            right = ((u >= ta) & (u < tab)) | (u >= tabc)
            down = u >= tab
            bit = 1 << (scale - 1 - lvl)
            src += down.to(torch.int64) * bit
            dst += right.to(torch.int64) * bit
        srcs.append(new_id[src])
        dsts.append(new_id[dst])
    return torch.cat(srcs), torch.cat(dsts)


def csr_from_edges(n_rows: int, rows: torch.Tensor, cols: torch.Tensor, n_cols: int | None = None):
    """(row, col) pairs -> deduplicated CSR (row_ptr int32[n+1], col int32[nnz]) in (row, col)
    order.  Input construction only (P:30 CSR definition)."""
    n_cols = n_rows if n_cols is None else n_cols
    key = rows.to(torch.int64) * n_cols + cols.to(torch.int64)
    key = torch.unique(key, sorted=True)
    r = key // n_cols
    c = (key - r * n_cols).to(torch.int32)
    counts = torch.bincount(r, minlength=n_rows)
    row_ptr = torch.zeros(n_rows + 1, dtype=torch.int64, device=key.device)
    row_ptr[1:] = torch.cumsum(counts, 0)
    assert int(row_ptr[-1]) < 2 ** 31, "int32 row_ptr"
    return row_ptr.to(torch.int32), c


def rmat_csr(scale: int, edge_factor: int = 16, seed: int | None = None, device=None,
             transpose: bool = False):
    """R-MAT CSR.  transpose=False: rows = sources (out-links, the SpMV matrix);
    transpose=True: rows = destinations (the in-link pattern used by PageRank)."""
    seed = scale if seed is None else seed
    n = 1 << scale
    s, d = rmat_edges(scale, edge_factor, seed, device)
    if transpose:
        s, d = d, s
    return csr_from_edges(n, s, d)


# --------------------------------------------------------------------------- values
def values(nnz: int, seed: int, dtype=torch.float64, device=None, integer: bool = False,
           stream: int = _STREAM_VAL) -> torch.Tensor:
    """U(-1, 1) (or integers in [-8, 8] when integer=True) indexed by position."""
    dev = _dev(device)
    h = hash64(seed, stream, torch.arange(nnz, device=dev, dtype=torch.int64))
    if integer:
        v = (_srl(h, 1) % 17 - 8).to(torch.float64)
    else:
        v = uniform53(h) * 2.0 - 1.0
    return v.to(dtype)


def vector(n: int, seed: int, dtype=torch.float64, device=None, integer: bool = False):
    return values(n, seed, dtype, device, integer, stream=_STREAM_X)


# --------------------------------------------------------------------------- power law
def _powerlaw_cdf(gamma: float, kmin: int, kmax: int) -> np.ndarray:
    k = np.arange(kmin, kmax + 1, dtype=np.float64)
    p = k ** (-gamma)
    cdf = np.cumsum(p)  # sequential numpy sum: identical table for every device
    return cdf / cdf[-1]


def powerlaw_csr(n: int, gamma: float, kmin: int, kmax: int, seed: int, device=None,
                 col_skew: float = 3.0):
    """Row r draws a length d_r from P(k) ~ k^-gamma on [kmin, kmax]; its columns are drawn
    with popularity rank floor(n * u^col_skew) (a power-law in-degree), mapped through a random
    vertex permutation; repeated columns inside a row are dropped."""
    dev = _dev(device)
    cdf = torch.from_numpy(_powerlaw_cdf(gamma, kmin, kmax)).to(dev)
    r = torch.arange(n, device=dev, dtype=torch.int64)
    u = uniform53(hash64(seed, 21, r))
    deg = torch.searchsorted(cdf, u, right=True).clamp_max(kmax - kmin) + kmin
    m = int(deg.sum())
    rows = torch.repeat_interleave(r, deg)
    e = torch.arange(m, device=dev, dtype=torch.int64)
    uc = uniform53(hash64(seed, 23, e))
    rank = torch.clamp((uc ** col_skew * n).to(torch.int64), max=n - 1)
    perm_keys = _srl(hash64(seed, 25, r), 1)
    order = torch.sort(perm_keys, stable=True).indices  # rank -> vertex
    cols = order[rank]
    row_perm = torch.sort(_srl(hash64(seed, 27, r), 1), stable=True).indices
    return csr_from_edges(n, row_perm[rows], cols)


WEB_GOOGLE = dict(n=900_000, gamma=2.84, kmin=3, kmax=5000)
LIVEJOURNAL = dict(n=4_850_000, gamma=3.05, kmin=8, kmax=9186)


# --------------------------------------------------------------------------- boundary
def boundary_lengths(max_pow: int = 17):
    lens = [0, 1, 2, 3, 4]
    for k in range(2, max_pow + 1):
        lens += [1 << k, (1 << k) + 1]
    return sorted(set(lens))


def boundary_csr(lengths, n_cols: int, seed: int, device=None):
    """One row per requested length; columns uniform (repeats allowed -- a CSR row may hold
    the same column twice only in dynamic graphs; here columns are drawn distinct per row
    when the row is shorter than n_cols)."""
    dev = _dev(device)
    lengths = torch.as_tensor(lengths, dtype=torch.int64, device=dev)
    row_ptr = torch.zeros(lengths.numel() + 1, dtype=torch.int64, device=dev)
    row_ptr[1:] = torch.cumsum(lengths, 0)
    m = int(row_ptr[-1])
    e = torch.arange(m, device=dev, dtype=torch.int64)
    rows = torch.repeat_interleave(torch.arange(lengths.numel(), device=dev), lengths)
    pos = e - row_ptr[rows]
    off = _srl(hash64(seed, 31, rows), 1) % n_cols
    cols = ((off + pos * 7919) % n_cols).to(torch.int32)  # distinct while len <= n_cols
    return row_ptr.to(torch.int32), cols


# --------------------------------------------------------------------------- dynamic
def with_slack(row_ptr: torch.Tensor, col: torch.Tensor, val: torch.Tensor | None = None,
               min_slack: int = 4, frac: int = 4):
    """Standard CSR -> 4-array CSR with reserved space at the end of every row:
    cap_r = len_r + max(min_slack, ceil(len_r / frac)).  Returns
    (row_begin, row_end, row_cap, col, val) with entries past row_end set to -1 / 0."""
    rp = row_ptr.to(torch.int64)
    n = rp.numel() - 1
    ln = rp[1:] - rp[:-1]
    cap = ln + torch.clamp((ln + frac - 1) // frac, min=min_slack)
    rb = torch.zeros(n + 1, dtype=torch.int64, device=rp.device)
    rb[1:] = torch.cumsum(cap, 0)
    total = int(rb[-1])
    assert total < 2 ** 31
    rows = torch.repeat_interleave(torch.arange(n, device=rp.device), ln)
    dst = rb[rows] + (torch.arange(rp[-1], device=rp.device) - rp[rows])
    col2 = torch.full((max(total, 1),), -1, dtype=torch.int32, device=rp.device)
    col2[dst] = col
    val2 = None
    if val is not None:
        val2 = torch.zeros(max(total, 1), dtype=val.dtype, device=rp.device)
        val2[dst] = val
    return (rb[:-1].to(torch.int32).contiguous(), (rb[:-1] + ln).to(torch.int32),
            cap.to(torch.int32), col2, val2)


def encode_changes(n_rows: int, ins_rows: np.ndarray, ins_cols: np.ndarray,
                   del_rows: np.ndarray | None = None, del_cols: np.ndarray | None = None):
    """Change lists "in CSR format": strictly increasing upd_rows; per row a sorted
    delete list and a sorted insert list.  Host numpy int32 arrays."""
    ins_rows = np.asarray(ins_rows, np.int64)
    ins_cols = np.asarray(ins_cols, np.int64)
    if del_rows is None:
        del_rows = np.zeros(0, np.int64)
        del_cols = np.zeros(0, np.int64)
    del_rows = np.asarray(del_rows, np.int64)
    del_cols = np.asarray(del_cols, np.int64)
    upd = np.unique(np.concatenate([ins_rows, del_rows]))
    oi = np.lexsort((ins_cols, ins_rows))
    od = np.lexsort((del_cols, del_rows))
    ins_rows, ins_cols = ins_rows[oi], ins_cols[oi]
    del_rows, del_cols = del_rows[od], del_cols[od]
    ins_ptr = np.searchsorted(ins_rows, upd, side="left")
    ins_ptr = np.append(ins_ptr, ins_rows.size)
    del_ptr = np.searchsorted(del_rows, upd, side="left")
    del_ptr = np.append(del_ptr, del_rows.size)
    return dict(upd_rows=upd.astype(np.int32), ins_ptr=ins_ptr.astype(np.int32),
                ins_cols=ins_cols.astype(np.int32), del_ptr=del_ptr.astype(np.int32),
                del_cols=del_cols.astype(np.int32))


def insert_batches(scale: int, n_batches: int, batch_edges: int, existing_keys, base_seed: int = 3000,
                   graph_seed: int | None = None, device=None):
    """C5: batch b draws ``batch_edges`` R-MAT edges (same generator and vertex permutation as the
    base graph, edge seed base_seed + 1 + b), keeps in-link orientation (row = destination), drops
    edges already present (base graph or earlier batches) and in-batch duplicates, and encodes
    the survivors as insert-only change lists.  existing_keys: sorted int64 row*n+col keys of
    the base in-link graph (numpy or tensor).  Filtering runs on ``device``.  Yields
    (changes dict of host int32 numpy arrays, n_inserted)."""
    graph_seed = scale if graph_seed is None else graph_seed
    dev = _dev(device)
    n = 1 << scale
    new_id = rmat_perm(scale, graph_seed, dev)
    keys = torch.as_tensor(existing_keys, dtype=torch.int64).to(dev)
    for b in range(n_batches):
        src, dst = rmat_edges(scale, 16, base_seed + 1 + b, dev, n_edges=batch_edges, new_id=new_id)
        k = torch.unique(dst.to(torch.int64) * n + src.to(torch.int64), sorted=True)
        pos = torch.searchsorted(keys, k)
        present = keys[torch.clamp(pos, max=max(keys.numel() - 1, 0))] == k if keys.numel() else \
            torch.zeros_like(k, dtype=torch.bool)
        present &= pos < keys.numel()
        k = k[~present]
        keys = torch.sort(torch.cat([keys, k])).values
        kh = k.cpu().numpy()
        ch = encode_changes(n, kh // n, kh % n)
        yield ch, int(kh.size)


def mixed_batches(row_ptr: np.ndarray, col: np.ndarray, n_cols: int, frac_rows: float,
                  seed: int, n_epochs: int):
    """Paper-shaped epochs: choose frac_rows of the rows; scanning each chosen row's
    columns, either delete that column or add another (uniform, not in the row), each with
    probability 1/2.  Host-side numpy; yields change dicts for successive epochs applied to a
    running copy of the graph."""
    rp = np.asarray(row_ptr, np.int64)
    cols = [np.asarray(col[rp[i]:rp[i + 1]], np.int64) for i in range(rp.size - 1)]
    n = rp.size - 1
    for ep in range(n_epochs):
        t = torch.arange(n, dtype=torch.int64)
        pick = (uniform53(hash64(seed + ep, 41, t)).numpy() < frac_rows).nonzero()[0]
        ir, ic, dr, dc = [], [], [], []
        for r in pick:
            cur = cols[r]
            if cur.size == 0:
                continue
            idx = torch.arange(cur.size, dtype=torch.int64) + int(r) * 4096
            coin = uniform53(hash64(seed + ep, 43, idx)).numpy() < 0.5
            cand = (_srl(hash64(seed + ep, 45, idx), 1) % n_cols).numpy()
            present = set(cur.tolist())
            dels = cur[coin]
            adds = []
            for c in cand[~coin]:
                if c not in present:
                    present.add(int(c))
                    adds.append(int(c))
            dels = np.unique(dels)
            adds = np.unique(np.asarray(adds, np.int64))
            dr += [r] * dels.size
            dc += dels.tolist()
            ir += [r] * adds.size
            ic += adds.tolist()
            keep = np.setdiff1d(cur, dels, assume_unique=False)
            cols[r] = np.concatenate([cur[np.isin(cur, keep)], adds])
        yield encode_changes(n, np.asarray(ir), np.asarray(ic), np.asarray(dr), np.asarray(dc))


def mixed_epoch(row_begin: torch.Tensor, row_end: torch.Tensor, col: torch.Tensor, n_cols: int,
                frac_rows: float, seed: int):
    """Paper-shaped change list (reading R3) generated on the graph's device from the
    CURRENT live entries of a slack CSR: rows are picked with probability frac_rows; scanning
    a picked row's columns, each column is deleted or "another column" (uniform, not already
    in the row, not a duplicate) is added, each with probability 1/2.  Returns the change
    dict (host int32 numpy arrays, "in CSR format")."""
    dev = row_begin.device
    n = row_begin.numel()
    rid = torch.arange(n, device=dev, dtype=torch.int64)
    pick = uniform53(hash64(seed, 41, rid)) < frac_rows
    ln = (row_end - row_begin).long()
    lnp = torch.where(pick, ln, torch.zeros_like(ln))
    rows = torch.repeat_interleave(rid, lnp)
    start = torch.repeat_interleave(row_begin.long(), lnp)
    first = torch.zeros(n + 1, dtype=torch.int64, device=dev)
    first[1:] = torch.cumsum(lnp, 0)
    pos = torch.arange(rows.numel(), device=dev, dtype=torch.int64) - first[rows]
    cols = col[(start + pos)].long()
    key_e = rows * (1 << 32) + pos
    coin = uniform53(hash64(seed, 43, key_e)) < 0.5
    del_r, del_c = rows[coin], cols[coin]
    add_r = rows[~coin]
    add_c = _srl(hash64(seed, 45, key_e[~coin]), 1) % n_cols
    # drop adds already in the row (live entries) and duplicate adds
    live_r = torch.repeat_interleave(rid, ln)
    lfirst = torch.zeros(n + 1, dtype=torch.int64, device=dev)
    lfirst[1:] = torch.cumsum(ln, 0)
    lpos = torch.arange(live_r.numel(), device=dev, dtype=torch.int64) - lfirst[live_r]
    live_c = col[(torch.repeat_interleave(row_begin.long(), ln) + lpos)].long()
    live_keys = torch.sort(live_r * n_cols + live_c).values
    ak = torch.unique(add_r * n_cols + add_c)
    p = torch.searchsorted(live_keys, ak)
    present = (p < live_keys.numel()) & (live_keys[torch.clamp(p, max=max(live_keys.numel() - 1, 0))] == ak)
    ak = ak[~present]
    dk = torch.unique(del_r * n_cols + del_c)
    akh, dkh = ak.cpu().numpy(), dk.cpu().numpy()
    return encode_changes(n, akh // n_cols, akh % n_cols, dkh // n_cols, dkh % n_cols)
