"""Pins for oracle O7 (dynamic update, §VII), O8 (partition) and O1 (CSR build).

Update: apply-then-sort equals the CSR rebuilt (numpy, independently) from the updated edge
multiset; rejected batches leave everything bitwise unchanged; outdeg equals the column
bincount of the live entries.  Partition: brute-force split points.  CSR build: scipy.
"""
import numpy as np
import pytest
import scipy.sparse as sp
import torch

import oracle
import synth


def live_edges(rb, re, col):
    rows = np.concatenate([np.full(re[i] - rb[i], i) for i in range(rb.size)]).astype(np.int64)
    cols = np.concatenate([col[rb[i]:re[i]] for i in range(rb.size)]).astype(np.int64)
    return rows, cols


def sorted_multiset(rows, cols):
    k = np.sort(rows * (1 << 32) + cols)
    return k


def base_graph(scale=10, frac=4):
    rp, ci = synth.rmat_csr(scale, transpose=True)
    v = synth.values(ci.numel(), 5)
    rb, re, cap, c2, v2 = synth.with_slack(rp, ci, v, frac=frac)
    n = rp.numel() - 1
    return n, rb.numpy(), re.numpy().copy(), cap.numpy(), c2.numpy().copy(), v2.numpy().copy()


def test_insert_only_equals_rebuild():
    n, rb, re, cap, col, val = base_graph(12)
    r0, c0 = live_edges(rb, re, col)
    od = np.bincount(c0, minlength=n).astype(np.int32)
    keys = np.sort(r0 * n + c0)
    ch, m = next(synth.insert_batches(12, 1, 1024, keys))
    ins_vals = synth.values(ch["ins_cols"].size, 77).numpy()
    code, idx = oracle.update(n, rb, re, cap, col, val, ch["upd_rows"], None, None, ch["ins_ptr"],
                              ch["ins_cols"], ins_vals, od)
    assert code == oracle.OK and idx == -1
    r1, c1 = live_edges(rb, re, col)
    ir = np.repeat(ch["upd_rows"], np.diff(ch["ins_ptr"])).astype(np.int64)
    exp = sorted_multiset(np.concatenate([r0, ir]), np.concatenate([c0, ch["ins_cols"]]))
    assert np.array_equal(sorted_multiset(r1, c1), exp)
    assert np.array_equal(od, np.bincount(c1, minlength=n))
    # inserted values land right after the kept entries, in list order
    for i, r in enumerate(ch["upd_rows"][:50]):
        k = ch["ins_ptr"][i + 1] - ch["ins_ptr"][i]
        assert np.array_equal(col[re[r] - k:re[r]], ch["ins_cols"][ch["ins_ptr"][i]:ch["ins_ptr"][i + 1]])
        assert np.array_equal(val[re[r] - k:re[r]], ins_vals[ch["ins_ptr"][i]:ch["ins_ptr"][i + 1]])


def test_mixed_delete_insert_equals_rebuild():
    n, rb, re, cap, col, val = base_graph(frac=1)  # paper-shaped epochs need ~2x slack
    rp = np.zeros(n + 1, np.int64)
    rp[1:] = np.cumsum(re - rb)
    packed = np.concatenate([col[rb[i]:re[i]] for i in range(n)])
    ch = next(synth.mixed_batches(rp, packed, n, 0.1, 5, 1))
    r0, c0 = live_edges(rb, re, col)
    od = np.bincount(c0, minlength=n).astype(np.int32)
    code, _ = oracle.update(n, rb, re, cap, col, None, ch["upd_rows"], ch["del_ptr"],
                            ch["del_cols"], ch["ins_ptr"], ch["ins_cols"], None, od)
    assert code == oracle.OK
    dr = np.repeat(ch["upd_rows"], np.diff(ch["del_ptr"])).astype(np.int64)
    ir = np.repeat(ch["upd_rows"], np.diff(ch["ins_ptr"])).astype(np.int64)
    base = r0 * n + c0
    dk = dr * n + ch["del_cols"]
    keep = ~np.isin(base, dk)
    expk = np.sort(np.concatenate([base[keep], ir * n + ch["ins_cols"]]))
    r1, c1 = live_edges(rb, re, col)
    assert np.array_equal(np.sort(r1 * n + c1), expk)
    assert np.array_equal(od, np.bincount(c1, minlength=n))
    assert ch["del_cols"].size > 0 and ch["ins_cols"].size > 0


def test_capacity_rejects_whole_batch_unchanged():
    n, rb, re, cap, col, val = base_graph()
    od = np.bincount(np.concatenate([col[rb[i]:re[i]] for i in range(n)]), minlength=n).astype(np.int32)
    snap = [a.copy() for a in (re, col, val, od)]
    # row 3: fine; row 7: overflow by one
    free7 = int(cap[7] - (re[7] - rb[7]))
    ins_cols = np.concatenate([[1], np.arange(free7 + 1) % n]).astype(np.int32)
    ins_ptr = np.array([0, 1, 1 + free7 + 1], np.int32)
    code, idx = oracle.update(n, rb, re, cap, col, val, np.array([3, 7], np.int32), None, None,
                              ins_ptr, ins_cols, None, od)
    assert code == oracle.ERR_CAPACITY and idx == 1
    for a, b in zip((re, col, val, od), snap):
        assert np.array_equal(a, b)


def test_invalid_lists_rejected():
    n, rb, re, cap, col, val = base_graph()
    snap = [a.copy() for a in (re, col)]
    ip = np.array([0, 1, 2], np.int32)
    code, idx = oracle.update(n, rb, re, cap, col, None, np.array([5, 5], np.int32), None, None, ip,
                              np.array([1, 2], np.int32))
    assert (code, idx) == (oracle.ERR_INVALID_VALUE, 1)
    code, idx = oracle.update(n, rb, re, cap, col, None, np.array([5, 6], np.int32),
                              np.array([0, 0, 2], np.int32), np.array([9, 3], np.int32), ip,
                              np.array([1, 2], np.int32))
    assert (code, idx) == (oracle.ERR_INVALID_VALUE, 1)
    code, idx = oracle.update(n, rb, re, cap, col, None, np.array([5, 6], np.int32), None, None, ip,
                              np.array([1, n], np.int32))
    assert (code, idx) == (oracle.ERR_INVALID_VALUE, 1)
    for a, b in zip((re, col), snap):
        assert np.array_equal(a, b)


@pytest.mark.parametrize("P", [1, 2, 3, 8])
def test_partition_bruteforce(P):
    rp, _ = synth.rmat_csr(12)
    rp = rp.numpy()
    n = rp.size - 1
    s = oracle.partition(rp, P, 4, 36)
    cost = 4 * np.diff(rp).astype(np.int64) + 36
    pref = np.concatenate([[0], np.cumsum(cost)])
    total = int(pref[-1])
    assert s[0] == 0 and s[P] == n
    for k in range(1, P):
        t = -(-k * total // P)
        brute = min(r for r in range(n + 1) if pref[r] >= t)
        assert s[k] == brute
    assert np.all(np.diff(s) >= 0)
    assert np.all(np.diff(pref[s]) <= -(-total // P) + cost.max())
    # reading R7: split points rounded up to a multiple of `align`, clamped to n
    for align in (32, 1024, 5000):
        sa = oracle.partition(rp, P, 4, 36, align=align)
        assert sa[0] == 0 and sa[P] == n
        for k in range(1, P):
            assert sa[k] == min(n, -(-int(s[k]) // align) * align)


def test_csr_build_vs_scipy():
    rng = np.random.default_rng(4)
    r = rng.integers(0, 100, 3000)
    c = rng.integers(0, 80, 3000)
    v = rng.uniform(-1, 1, 3000)
    rp, ci, vv = oracle.csr_build(100, r, c, v, dedup=False)
    S = sp.coo_matrix((v, (r, c)), shape=(100, 80)).tocsr()
    S.sum_duplicates()
    # summing the duplicates of our build must reproduce scipy's summed CSR
    mine = sp.csr_matrix((vv, ci, rp), shape=(100, 80))
    mine.sum_duplicates()
    assert np.array_equal(mine.indptr, S.indptr) and np.array_equal(mine.indices, S.indices)
    assert np.allclose(mine.data, S.data, rtol=1e-14)
    rp2, ci2, _ = oracle.csr_build(100, r, c, None, dedup=True)
    assert np.array_equal(rp2, S.indptr) and np.array_equal(ci2, S.indices)
