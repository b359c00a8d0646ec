"""Pins for the oracle's RWR (Eq. 8, reading R5) and HITS (Eq. 5-7, P:299-317,
reading R6): closed forms, a dense linear solve, dense eigenvectors, networkx."""
import os

import networkx as nx
import numpy as np
import pytest

import oracle

C = 0.85
GOLD = os.path.join(os.path.dirname(__file__), "golden", "rwr_two_cycle.txt")


def inlink(n, edges):
    e = np.array(edges, np.int64).reshape(-1, 2)
    u, v = e[:, 0], e[:, 1]
    o = np.lexsort((u, v))
    rp = np.zeros(n + 1, np.int32)
    rp[1:] = np.cumsum(np.bincount(v[o], minlength=n))
    return rp, u[o].astype(np.int32), np.bincount(u, minlength=n).astype(np.int32)


def outlink(n, edges):
    e = np.array(edges, np.int64).reshape(-1, 2)
    u, v = e[:, 0], e[:, 1]
    o = np.lexsort((v, u))
    rp = np.zeros(n + 1, np.int32)
    rp[1:] = np.cumsum(np.bincount(u[o], minlength=n))
    return rp, v[o].astype(np.int32)


def rand_graph(n, seed, maxdeg=5, no_dangling=True):
    rng = np.random.default_rng(seed)
    edges = set()
    for u in range(n):
        k = rng.integers(1 if no_dangling else 0, maxdeg + 1)
        for v in rng.choice(n, size=k, replace=False):
            if int(v) != u:
                edges.add((u, int(v)))
    return sorted(edges)


def test_rwr_two_cycle_golden():
    vals = dict(l.split() for l in open(GOLD) if l.strip() and not l.startswith("#"))
    rp, c, od = inlink(2, [(0, 1), (1, 0)])
    r, it, _ = oracle.rwr(rp, c, od, restart=0, c=C, eps=1e-15)
    assert r[0] == pytest.approx(float(vals["a"]), rel=1e-14)
    assert r[1] == pytest.approx(float(vals["b"]), rel=1e-14)


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_rwr_equals_linear_solve(seed):
    n = 40
    edges = rand_graph(n, seed, no_dangling=False)
    rp, c, od = inlink(n, edges)
    W = np.zeros((n, n))
    for u, v in edges:
        W[v, u] = 1.0 / od[u]
    i = seed % n
    e = np.zeros(n)
    e[i] = 1.0
    exact = np.linalg.solve(np.eye(n) - C * W, (1 - C) * e)
    r, it, d2 = oracle.rwr(rp, c, od, restart=i, c=C, eps=1e-14)
    assert np.allclose(r, exact, rtol=1e-10, atol=1e-15)


def test_rwr_mass_and_step():
    n = 60
    edges = rand_graph(n, 7)  # no dangling vertices: W is column-stochastic
    rp, c, od = inlink(n, edges)
    r = np.random.default_rng(0).random(n)
    r /= r.sum()
    rn, d2 = oracle.rwr_step(rp, c, od, r, C, 5)
    assert rn.sum() == pytest.approx(1.0, rel=1e-14)  # c*1 + (1-c)
    assert d2 == pytest.approx(float(((rn - r) ** 2).sum()), rel=1e-12)


def test_hits_star_closed_form():
    k = 7
    edges = [(0, j) for j in range(1, k + 1)]
    op, oc = outlink(k + 1, edges)
    ip, ic, _ = inlink(k + 1, edges)
    a, h, it = oracle.hits(op, oc, ip, ic, eps=1e-14)
    assert a[0] == 0.0 and np.allclose(a[1:], 1 / np.sqrt(k), rtol=1e-14)
    assert h[0] == pytest.approx(1.0, rel=1e-15) and np.all(h[1:] == 0.0)


@pytest.mark.parametrize("seed", [4, 5])
def test_hits_principal_eigenvectors(seed):
    n = 50
    edges = rand_graph(n, seed)
    A = np.zeros((n, n))
    for u, v in edges:
        A[u, v] = 1.0
    op, oc = outlink(n, edges)
    ip, ic, _ = inlink(n, edges)
    a, h, it = oracle.hits(op, oc, ip, ic, eps=1e-13, max_iter=100000)
    wa, va = np.linalg.eigh(A.T @ A)
    wh, vh = np.linalg.eigh(A @ A.T)
    ea = np.abs(va[:, -1])
    eh = np.abs(vh[:, -1])
    assert wa[-1] - wa[-2] > 1e-3  # unique principal direction
    assert np.allclose(a, ea, atol=1e-9)
    assert np.allclose(h, eh, atol=1e-9)
    # networkx agrees up to normalisation (it uses L1 sums)
    G = nx.DiGraph(edges)
    G.add_nodes_from(range(n))
    hn, an = nx.hits(G, max_iter=100000, tol=1e-14)
    an = np.array([an[i] for i in range(n)])
    hn = np.array([hn[i] for i in range(n)])
    assert np.allclose(a, an / np.linalg.norm(an), atol=1e-7)
    assert np.allclose(h, hn / np.linalg.norm(hn), atol=1e-7)
