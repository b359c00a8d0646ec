"""Pins for oracle O6/O6' (PageRank step and loop, Alg. 5).

Closed forms (cycle, complete digraph, a->b golden fixture), the mass invariant of reading
Q11, networkx.pagerank on graphs without dangling vertices, and the fixed-point residual.
"""
import os

import networkx as nx
import numpy as np
import pytest

import oracle
import synth

D = 0.85
GOLD = os.path.join(os.path.dirname(__file__), "golden", "pagerank_two_vertex.txt")


def inlink_csr(n, edges):
    """edges u->v  ->  in-link pattern CSR (row v lists sources u) + outdeg (independent numpy)."""
    e = np.array(edges, np.int64).reshape(-1, 2)
    u, v = e[:, 0], e[:, 1]
    order = np.lexsort((u, v))
    u, v = u[order], v[order]
    rp = np.zeros(n + 1, np.int32)
    rp[1:] = np.cumsum(np.bincount(v, minlength=n))
    outdeg = np.bincount(u, minlength=n).astype(np.int32)
    return rp, u.astype(np.int32), outdeg


def test_cycle_uniform():
    n = 17
    rp, c, od = inlink_csr(n, [(i, (i + 1) % n) for i in range(n)])
    x, it, _ = oracle.pagerank(rp, c, od)
    assert it == 1
    assert np.allclose(x, 1.0 / n, rtol=2e-16, atol=0)


def test_complete_digraph_uniform():
    n = 9
    rp, c, od = inlink_csr(n, [(i, j) for i in range(n) for j in range(n) if i != j])
    x, it, _ = oracle.pagerank(rp, c, od)
    assert np.allclose(x, 1.0 / n, rtol=4e-16, atol=0)


def test_two_vertex_golden():
    vals = dict(l.split() for l in open(GOLD) if l.strip() and not l.startswith("#"))
    rp, c, od = inlink_csr(2, [(0, 1)])
    x, it, _ = oracle.pagerank(rp, c, od, eps=1e-15)
    assert x[0] == pytest.approx(float(vals["a"]), rel=1e-15)
    assert x[1] == pytest.approx(float(vals["b"]), rel=1e-15)


def test_mass_invariant_per_step():
    # Q11: sum x' = (1-d) + d * sum_{outdeg_u > 0} x_u  (dangling mass dropped)
    rp, ci = synth.rmat_csr(12, transpose=True)
    rp, ci = rp.numpy(), ci.numpy()
    n = rp.size - 1
    od = np.bincount(ci, minlength=n).astype(np.int32)
    x = synth.vector(n, 8).numpy() * 0.5 + 0.5
    x /= x.sum()
    xn, d2 = oracle.pagerank_step(rp, ci, od, x, (1 - D) / n, D)
    expect = (1 - D) + D * x[od > 0].sum()
    assert xn.sum() == pytest.approx(expect, rel=n * 2.3e-16)
    assert d2 == pytest.approx(float(((xn - x) ** 2).sum()), rel=1e-12)


@pytest.mark.parametrize("seed", [1, 2])
def test_networkx_no_dangling(seed):
    rng = np.random.default_rng(seed)
    n = 50
    edges = set()
    for u in range(n):  # every vertex has >= 1 out-link: no dangling vertices
        for v in rng.choice(n, size=rng.integers(1, 6), replace=False):
            edges.add((u, int(v)))
    G = nx.DiGraph()
    G.add_nodes_from(range(n))
    G.add_edges_from(edges)
    ref = nx.pagerank(G, alpha=D, tol=1e-15, max_iter=10000)
    rp, c, od = inlink_csr(n, sorted(edges))
    x, it, _ = oracle.pagerank(rp, c, od, eps=1e-14)
    for v in range(n):
        assert x[v] == pytest.approx(ref[v], rel=1e-10)


def test_fixed_point_residual_and_warm_start():
    rp, ci = synth.rmat_csr(11, transpose=True)
    rp, ci = rp.numpy(), ci.numpy()
    n = rp.size - 1
    od = np.bincount(ci, minlength=n).astype(np.int32)
    x, it, d2 = oracle.pagerank(rp, ci, od, eps=1e-6)
    assert np.sqrt(d2) <= 1e-6 and it > 3
    # residual r = x - ((1-d)/n + d * P (x/outdeg)) ~ contraction * last step
    xs = np.where(od > 0, x / np.maximum(od, 1), 0.0)
    y = np.add.reduceat(np.append(xs[ci], 0.0), rp[:-1])[:n] * (np.diff(rp) > 0)
    res = x - ((1 - D) / n + D * y)
    assert np.linalg.norm(res) <= 1e-6
    # warm start from the converged vector: one step suffices
    x2, it2, _ = oracle.pagerank(rp, ci, od, x0=x, eps=1e-6)
    assert it2 == 1
