"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle.

Bins and updates: bit-exact.  SpMV on integer-valued data: bit-exact (every summation
order is exact).  SpMV on U(-1,1) data: |y - y_ref| <= 1e-12 * (|A||x|)_r in fp64 and
1e-5 * (|A||x|)_r in fp32 (north_star; reading Q16); rows with den == 0 must match bitwise
(+0.0 for empty rows).  PageRank: step-wise at the fp64 bar, loop iteration count within
+-1 of the oracle (reading Q18).
"""
import os

import numpy as np
import pytest
import torch

import oracle
import synth

pytestmark = pytest.mark.gpu

TOL = {torch.float64: 1e-12, torch.float32: 1e-5}


def check_spmv(y_gpu, y_ref, den, dtype, exact=False):
    y_gpu = np.asarray(y_gpu, dtype=np.float64)
    y_ref = np.asarray(y_ref, dtype=np.float64)
    if exact:
        assert np.array_equal(y_gpu, y_ref), np.flatnonzero(y_gpu != y_ref)[:10]
        return
    zero = den == 0
    assert np.array_equal(y_gpu[zero], y_ref[zero])
    assert not np.any(np.signbit(y_gpu[zero]) != np.signbit(y_ref[zero]))
    err = np.abs(y_gpu - y_ref)
    bad = err > TOL[dtype] * den
    assert not bad.any(), (np.flatnonzero(bad)[:10], err[bad][:5], den[bad][:5])


MAPPINGS = ["window", "alg2"]  # SpMV mapping of bins 0..5 (acsr_bin / acsr_bin_ex ACSR_BIN_SHORT_ALG2)


def run_csr(acsr, rp, ci, val, x, dev, row_end=None, short_rows="window"):
    rbd = rp.to(dev)
    red = None if row_end is None else row_end.to(dev)
    m = acsr.ACSRMatrix(rbd, ci.to(dev), None if val is None else val.to(dev),
                        n_cols=x.numel(), row_end=red, nnz_max=max(ci.numel(), 1), short_rows=short_rows)
    y = m.spmv(x.to(dev))
    torch.cuda.synchronize()
    return m, y.cpu()


# ------------------------------------------------------------------------------ bins
@pytest.mark.parametrize("scale", [10, 14, 17])
def test_bins_bitwise_rmat(acsr, cuda, scale):
    rp, ci = synth.rmat_csr(scale)
    m, _ = run_csr(acsr, rp, ci, None, torch.ones(rp.numel() - 1, dtype=torch.float64), cuda)
    br, off = oracle.bins(rp.numpy())
    assert np.array_equal(m.bin_offsets.cpu().numpy(), off)
    assert np.array_equal(m.bin_rows.cpu().numpy(), br)


@pytest.mark.parametrize("env", ["ACSR_BIN_SS=1", "ACSR_BIN_FUSED=1", "ACSR_PDL=0", "ACSR_XPREFETCH=0"])
def test_bins_alternative_launch_paths(cuda, env):
    """The opt-in binning launch paths (scan + scatter in one launch; one cooperative
    launch) and PDL off give the same bins and plan: bitwise bins vs the oracle and an SpMV
    on integer data bitwise, in a fresh process (the knobs are read once per process)."""
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    code = (
        "import sys; sys.path.insert(0, %r)\n"
        "import numpy as np, torch, oracle, synth\n"
        "import paper_conf_sc_ashariseps14_b200 as acsr\n"
        "for sc in (12, 17):\n"
        "    rp, ci = synth.rmat_csr(sc)\n"
        "    val = synth.values(ci.numel(), 3, integer=True); x = synth.vector(rp.numel() - 1, 4, integer=True)\n"
        "    m = acsr.ACSRMatrix(rp.cuda(), ci.cuda(), val.cuda())\n"
        "    y = m.spmv(x.cuda()).cpu().numpy()\n"
        "    br, off = oracle.bins(rp.numpy())\n"
        "    assert np.array_equal(m.bin_rows.cpu().numpy(), br) and np.array_equal(m.bin_offsets.cpu().numpy(), off)\n"
        "    y_ref, _ = oracle.spmv(rp.numpy(), ci.numpy(), val.numpy(), x.numpy())\n"
        "    assert np.array_equal(y, y_ref)\n"
        "print('alt-path ok')\n" % root)
    k, v = env.split("=")
    out = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, timeout=300,
                         env=dict(os.environ, **{k: v}))
    assert out.returncode == 0 and "alt-path ok" in out.stdout, out.stdout[-2000:] + out.stderr[-2000:]


def test_update_global_search_path(cuda):
    """The hub-row update path with the delete list searched in global memory
    (ACSR_UPD_SMEM=0, the fallback when shared memory cannot be reserved) passes the
    bitwise update tests too (fresh pytest process: the knob is read once)."""
    import subprocess
    import sys
    out = subprocess.run([sys.executable, "-m", "pytest", os.path.abspath(__file__), "-q", "-x", "-m", "gpu",
                          "-k", "update_long_row_cta_path or paper_epoch_update_bitwise or update_mixed_bitwise"],
                         capture_output=True, text=True, timeout=600, env=dict(os.environ, ACSR_UPD_SMEM="0"),
                         cwd=os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    assert out.returncode == 0 and " passed" in out.stdout, out.stdout[-2000:] + out.stderr[-2000:]


def test_bins_boundary_and_slack(acsr, cuda):
    lens = synth.boundary_lengths(17)
    rp, ci = synth.boundary_csr(lens * 3, 1 << 18, 5)
    rb, re, cap, c2, _ = synth.with_slack(rp, ci)
    br, off = oracle.bins(rb.numpy(), re.numpy())
    out = acsr.acsr_bin(rb.to(cuda), re.to(cuda), nnz_max=c2.numel())
    torch.cuda.synchronize()
    assert np.array_equal(out[1].cpu().numpy(), off)
    assert np.array_equal(out[0].cpu().numpy(), br)


@pytest.mark.parametrize("n", [0, 1, 4095, 4096, 4097, 70000])
def test_bins_edge_sizes(acsr, cuda, n):
    g = torch.Generator().manual_seed(n)
    ln = torch.randint(0, 40, (n,), generator=g) * (torch.rand(n, generator=g) < 0.5)
    if n:
        ln[n // 2] = 5000  # one heavy row
    rp = torch.zeros(n + 1, dtype=torch.int64)
    rp[1:] = torch.cumsum(ln, 0)
    rp = rp.to(torch.int32)
    br, bo, ws = acsr.acsr_bin(rp.to(cuda), None, nnz_max=int(rp[-1]))
    torch.cuda.synchronize()
    br_ref, off_ref = oracle.bins(rp.numpy())
    assert np.array_equal(bo.cpu().numpy(), off_ref)
    assert np.array_equal(br.cpu().numpy(), br_ref)


# ------------------------------------------------------------------------------ SpMV exact
@pytest.mark.parametrize("mapping", MAPPINGS)
@pytest.mark.parametrize("dtype", [torch.float64, torch.float32])
def test_spmv_integer_bitwise_rmat14(acsr, cuda, dtype, mapping):
    rp, ci = synth.rmat_csr(14)
    n = rp.numel() - 1
    val = synth.values(ci.numel(), 1014, dtype, integer=True)
    x = synth.vector(n, 2014, dtype, integer=True)
    _, y = run_csr(acsr, rp, ci, val, x, cuda, short_rows=mapping)
    y_ref, den = oracle.spmv(rp.numpy(), ci.numpy(), val.numpy(), x.numpy())
    check_spmv(y.numpy(), y_ref, den, dtype, exact=True)


@pytest.mark.parametrize("mapping", MAPPINGS)
@pytest.mark.parametrize("dtype", [torch.float64, torch.float32])
def test_spmv_integer_bitwise_boundary(acsr, cuda, dtype, mapping):
    # one row per bin edge up to 2^17+1 nnz: every mapping (sub-warp widths 1..32, warp,
    # split rows with many chunks) is exercised; integer data makes every order exact.
    lens = synth.boundary_lengths(17)
    rp, ci = synth.boundary_csr(lens, 1 << 18, 3)
    val = synth.values(ci.numel(), 7, dtype, integer=True)
    x = synth.vector(1 << 18, 8, dtype, integer=True)
    _, y = run_csr(acsr, rp, ci, val, x, cuda, short_rows=mapping)
    y_ref, den = oracle.spmv(rp.numpy(), ci.numpy(), val.numpy(), x.numpy())
    check_spmv(y.numpy(), y_ref, den, dtype, exact=True)


def test_identity_permutation_pattern(acsr, cuda):
    n = 100_000
    x = synth.vector(n, 5)
    rp = torch.arange(n + 1, dtype=torch.int32)
    _, y = run_csr(acsr, rp, torch.arange(n, dtype=torch.int32), torch.ones(n, dtype=torch.float64), x, cuda)
    assert torch.equal(y, x)
    perm = torch.randperm(n, generator=torch.Generator().manual_seed(1)).to(torch.int32)
    _, y = run_csr(acsr, rp, perm, None, x, cuda)
    assert torch.equal(y, x[perm.long()])


# ------------------------------------------------------------------------------ SpMV float
@pytest.mark.parametrize("mapping", MAPPINGS)
@pytest.mark.parametrize("dtype", [torch.float64, torch.float32])
@pytest.mark.parametrize("scale", [14, 16])
def test_spmv_float_rmat(acsr, cuda, dtype, scale, mapping):
    rp, ci = synth.rmat_csr(scale)
    n = rp.numel() - 1
    val = synth.values(ci.numel(), 1014, dtype)
    x = synth.vector(n, 2014, dtype)
    _, y = run_csr(acsr, rp, ci, val, x, cuda, short_rows=mapping)
    y_ref, den = oracle.spmv(rp.numpy(), ci.numpy(), val.numpy(), x.numpy())
    check_spmv(y.numpy(), y_ref, den, dtype)


@pytest.mark.parametrize("mapping", MAPPINGS)
@pytest.mark.parametrize("dtype", [torch.float64, torch.float32])
def test_spmv_float_boundary(acsr, cuda, dtype, mapping):
    lens = synth.boundary_lengths(17)
    rp, ci = synth.boundary_csr(lens, 1 << 18, 9)
    val = synth.values(ci.numel(), 10, dtype)
    x = synth.vector(1 << 18, 11, dtype)
    _, y = run_csr(acsr, rp, ci, val, x, cuda, short_rows=mapping)
    y_ref, den = oracle.spmv(rp.numpy(), ci.numpy(), val.numpy(), x.numpy())
    check_spmv(y.numpy(), y_ref, den, dtype)


@pytest.mark.parametrize("dtype,L", [(torch.float64, 100_000), (torch.float32, 1_000_000)])
def test_adversarial_long_equal_row(acsr, cuda, dtype, L):
    # 0.1 repeated: sequential fp64 misses 1e-12 at 1e5 terms, sequential fp32 misses 1e-5
    # at 1e6 terms; the chunked tree must not.
    rp = torch.tensor([0, L, L], dtype=torch.int32)
    ci = torch.zeros(L, dtype=torch.int32)
    val = torch.full((L,), 0.1, dtype=dtype)
    x = torch.ones(1, dtype=dtype)
    _, y = run_csr(acsr, rp, ci, val, x, cuda)
    y_ref, den = oracle.spmv(rp.numpy(), ci.numpy(), val.numpy(), x.numpy())
    check_spmv(y.numpy(), y_ref, den, dtype)


@pytest.mark.parametrize("mapping", MAPPINGS)
def test_powerlaw_webgoogle_like(acsr, cuda, mapping):
    rp, ci = synth.powerlaw_csr(seed=3, **dict(synth.WEB_GOOGLE, n=200_000))
    n = rp.numel() - 1
    val = synth.values(ci.numel(), 4)
    x = synth.vector(n, 5)
    _, y = run_csr(acsr, rp, ci, val, x, cuda, short_rows=mapping)
    y_ref, den = oracle.spmv(rp.numpy(), ci.numpy(), val.numpy(), x.numpy())
    check_spmv(y.numpy(), y_ref, den, torch.float64)


@pytest.mark.parametrize("dtype", [torch.float64, torch.float32])
def test_window_rows_are_in_order_sums(acsr, cuda, dtype):
    """Short-row windows: a row with <= 32 non-zeros is summed by one lane in element
    order from rounded products, i.e. exactly the oracle's plain sequential loop (O4',
    compiled without FMA contraction; fp32 accumulated in double, rounded once) -- so
    those rows must match oracle.spmv_plain BIT FOR BIT, and a row's result must not
    depend on its neighbours (lengths of other rows changed -> same bits)."""
    rp, ci = synth.rmat_csr(16)
    n = rp.numel() - 1
    val = synth.values(ci.numel(), 31, dtype)
    x = synth.vector(n, 32, dtype)
    _, y = run_csr(acsr, rp, ci, val, x, cuda)
    y_plain = oracle.spmv_plain(rp.numpy(), ci.numpy(), val.numpy(), x.numpy())
    ln = (rp[1:] - rp[:-1]).numpy()
    short = ln <= 32
    assert short.sum() > n // 2
    assert np.array_equal(y.numpy()[short].view(np.uint8), y_plain[short].view(np.uint8))
    # drop the last non-zero of every third row: the other rows keep their bits
    rb, re = rp[:-1].clone(), rp[1:].clone()
    cut = (torch.arange(n) % 3 == 0) & (re > rb)
    re[cut] -= 1
    _, y2 = run_csr(acsr, rb, ci, val, x, cuda, row_end=re)
    keep = ~cut.numpy()
    assert np.array_equal(y2.numpy()[keep].view(np.uint8), y.numpy()[keep].view(np.uint8))


@pytest.mark.parametrize("mapping", MAPPINGS)
def test_slack_csr_equals_standard_and_determinism(acsr, cuda, mapping):
    rp, ci = synth.rmat_csr(15)
    n = rp.numel() - 1
    val = synth.values(ci.numel(), 1)
    x = synth.vector(n, 2)
    m, y1 = run_csr(acsr, rp, ci, val, x, cuda, short_rows=mapping)
    y2 = m.spmv(x.to(cuda)).cpu()
    assert torch.equal(y1, y2)  # run-to-run bitwise
    rb, re, cap, c2, v2 = synth.with_slack(rp, ci, val)
    _, y3 = run_csr(acsr, rb, c2, v2, x, cuda, row_end=re, short_rows=mapping)
    y_ref, den = oracle.spmv(rp.numpy(), ci.numpy(), val.numpy(), x.numpy())
    check_spmv(y3.numpy(), y_ref, den, torch.float64)


def test_empty_and_all_empty(acsr, cuda):
    rp = torch.zeros(1, dtype=torch.int32)
    m, y = run_csr(acsr, rp, torch.zeros(0, dtype=torch.int32), torch.zeros(0, dtype=torch.float64),
                   torch.ones(3, dtype=torch.float64), cuda)
    assert y.numel() == 0
    rp = torch.zeros(5001, dtype=torch.int32)
    m, y = run_csr(acsr, rp, torch.zeros(0, dtype=torch.int32), torch.zeros(0, dtype=torch.float64),
                   torch.ones(3, dtype=torch.float64), cuda)
    assert torch.equal(y, torch.zeros(5000, dtype=torch.float64))
    assert not torch.signbit(y).any()


@pytest.mark.parametrize("mapping", MAPPINGS)
@pytest.mark.parametrize("n", [1, 31, 33, 4097, 70001])
def test_spmv_ragged_sizes(acsr, cuda, n, mapping):
    """Row counts that end inside a 32-row window / a 1024-row tile, with a mix of
    empty, short (1..32), bin-6 (33..64), warp (65..1024) and split (> 1024) rows;
    integer data, so every mapping must match the oracle bit for bit."""
    g = torch.Generator().manual_seed(n)
    kind = torch.randint(0, 10, (n,), generator=g)
    ln = torch.where(kind < 3, torch.zeros(n, dtype=torch.int64),
                     torch.where(kind < 8, torch.randint(1, 33, (n,), generator=g),
                                 torch.where(kind < 9, torch.randint(33, 65, (n,), generator=g),
                                             torch.randint(65, 1025, (n,), generator=g))))
    if n > 100:
        ln[n // 3] = 5000
        ln[-1] = 17  # a short row in the ragged last window
    rp = torch.zeros(n + 1, dtype=torch.int64)
    rp[1:] = torch.cumsum(ln, 0)
    nnz = int(rp[-1])
    n_cols = 50_000
    ci = torch.randint(0, n_cols, (nnz,), generator=g).to(torch.int32)
    rp = rp.to(torch.int32)
    val = synth.values(nnz, n, torch.float64, integer=True)
    x = synth.vector(n_cols, n + 1, torch.float64, integer=True)
    _, y = run_csr(acsr, rp, ci, val, x, cuda, short_rows=mapping)
    y_ref, den = oracle.spmv(rp.numpy(), ci.numpy(), val.numpy(), x.numpy())
    check_spmv(y.numpy(), y_ref, den, torch.float64, exact=True)


def full_parity(rp, ci, val, x, y):
    """Every row of y (host numpy) against the oracle on the whole matrix (Dot2, O4)."""
    y_ref, den = oracle.spmv(rp.cpu().numpy(), ci.cpu().numpy(), val.cpu().numpy(), x.cpu().numpy())
    check_spmv(y, y_ref, den, val.dtype)


@pytest.mark.parametrize("dtype", [torch.float64, torch.float32])
def test_full_size_rmat20_every_row(acsr, cuda, dtype):
    """C2 at BASELINE size, in the launch configuration bench.py times: bins bitwise, and
    EVERY row against the oracle element by element."""
    rp, ci = synth.rmat_csr(20, device=cuda)
    n = rp.numel() - 1
    val = synth.values(ci.numel(), 1014, dtype, device=cuda)
    x = synth.vector(n, 2014, dtype, device=cuda)
    m = acsr.ACSRMatrix(rp, ci, val)
    y = m.spmv(x).cpu().numpy()
    br, off = oracle.bins(rp.cpu().numpy())
    assert np.array_equal(m.bin_offsets.cpu().numpy(), off)
    assert np.array_equal(m.bin_rows.cpu().numpy(), br)
    full_parity(rp, ci, val, x, y)


@pytest.mark.parametrize("shape", ["WEB_GOOGLE", "LIVEJOURNAL"])
def test_full_size_powerlaw_every_row(acsr, cuda, shape):
    """C3 shapes at full size (0.9 M / 4.85 M rows): bins bitwise + every row."""
    rp, ci = synth.powerlaw_csr(seed=3, device=cuda, **getattr(synth, shape))
    n = rp.numel() - 1
    val = synth.values(ci.numel(), 4, device=cuda)
    x = synth.vector(n, 5, device=cuda)
    m = acsr.ACSRMatrix(rp, ci, val)
    y = m.spmv(x).cpu().numpy()
    br, off = oracle.bins(rp.cpu().numpy())
    assert np.array_equal(m.bin_rows.cpu().numpy(), br)
    full_parity(rp, ci, val, x, y)


def test_c1_rmat14_single_spmv(acsr, cuda):
    """C1 exactly as BASELINE.json configs[0] names it: R-MAT s14 fp64, one SpMV, every
    row against the oracle."""
    rp, ci = synth.rmat_csr(14)
    val = synth.values(ci.numel(), 1014)
    x = synth.vector(rp.numel() - 1, 2014)
    br, bo, ws = acsr.acsr_bin(rp.to(cuda), None, nnz_max=ci.numel(), col_idx=ci.to(cuda), n_cols=x.numel())
    y = acsr.acsr_spmv(rp.to(cuda), ci.to(cuda), val.to(cuda), x.to(cuda), br, bo, ws).cpu().numpy()
    y_ref, den = oracle.spmv(rp.numpy(), ci.numpy(), val.numpy(), x.numpy())
    check_spmv(y, y_ref, den, torch.float64)


# ------------------------------------------------------------------------------ PageRank
def _inlink(scale, dev):
    rp, ci = synth.rmat_csr(scale, transpose=True)
    n = rp.numel() - 1
    od = torch.bincount(ci.long(), minlength=n).to(torch.int32)
    return rp, ci, od, n


def test_pagerank_step_parity(acsr, cuda):
    rp, ci, od, n = _inlink(14, cuda)
    x = synth.vector(n, 3).abs() / n
    m = acsr.ACSRMatrix(rp.to(cuda), ci.to(cuda))
    xs = acsr.acsr_pagerank_scale(x.to(cuda), od.to(cuda))
    xn = torch.empty(n, dtype=torch.float64, device=cuda)
    xsn = torch.empty_like(xn)
    d2 = torch.zeros(1, dtype=torch.float64, device=cuda)
    acsr.acsr_pagerank_step(m.row_begin, m.col_idx, m.bin_rows, m.bin_offsets, m.plan_ws, xs,
                            x.to(cuda), od.to(cuda), xn, xsn, d2, 0.85, 0.15 / n)
    xn_ref, d2_ref = oracle.pagerank_step(rp.numpy(), ci.numpy(), od.numpy(), x.numpy(), 0.15 / n, 0.85)
    # den of the step = teleport + d * sum xs  (all terms >= 0)
    xs_h = np.where(od.numpy() > 0, x.numpy() / np.maximum(od.numpy(), 1), 0.0)
    _, den = oracle.spmv(rp.numpy(), ci.numpy(), None, xs_h)
    bound = 1e-12 * (0.15 / n + 0.85 * den) + 2.3e-16 * np.abs(xn_ref)
    assert np.all(np.abs(xn.cpu().numpy() - xn_ref) <= bound)
    xsn_ref = np.where(od.numpy() > 0, xn_ref / np.maximum(od.numpy(), 1), 0.0)
    assert np.allclose(xsn.cpu().numpy(), xsn_ref, rtol=1e-12, atol=0)
    assert float(d2.item()) == pytest.approx(d2_ref, rel=1e-9)
    # deterministic Delta^2 and x_new across runs
    xn2 = torch.empty_like(xn)
    d22 = torch.zeros_like(d2)
    acsr.acsr_pagerank_step(m.row_begin, m.col_idx, m.bin_rows, m.bin_offsets, m.plan_ws, xs,
                            x.to(cuda), od.to(cuda), xn2, xsn, d22, 0.85, 0.15 / n)
    assert torch.equal(xn, xn2) and torch.equal(d2, d22)


@pytest.mark.parametrize("scale", [16, 20])
def test_pagerank_converged_parity(acsr, cuda, scale):
    rp, ci, od, n = _inlink(scale, cuda)
    m = acsr.ACSRMatrix(rp.to(cuda), ci.to(cuda))
    x, it, d2 = acsr.pagerank(m, od.to(cuda), eps=1e-6)
    x_ref, it_ref, _ = oracle.pagerank(rp.numpy(), ci.numpy(), od.numpy(), eps=1e-6)
    assert abs(it - it_ref) <= 1
    if it == it_ref:
        xr = x_ref
    else:
        xr, _, _ = oracle.pagerank(rp.numpy(), ci.numpy(), od.numpy(), eps=0.0, max_iter=it)
    assert np.all(np.abs(x.cpu().numpy() - xr) <= 1e-11 * xr + 1e-18)


def _oracle_pagerank_step_parallel(rph, cih, odh, xh, teleport, d, threads=None):
    """The oracle step (O6) over every row, computed in row blocks by host threads (the
    ctypes call releases the GIL; the step is row-independent, so blocks change no bit).
    Each block passes the row offsets of its rows and the FULL col / outdeg / x arrays
    (gathers use global ids).  Returns x' for all rows."""
    from concurrent.futures import ThreadPoolExecutor
    n = rph.size - 1
    threads = threads or max(1, min(32, os.cpu_count() or 1))
    cuts = np.linspace(0, n, 4 * threads + 1).astype(np.int64)
    out = np.empty(n, np.float64)

    def block(i):
        r0, r1 = int(cuts[i]), int(cuts[i + 1])
        if r1 > r0:
            xn, _ = oracle.pagerank_step(rph[r0:r1 + 1], cih, odh, xh, teleport, d)
            out[r0:r1] = xn

    with ThreadPoolExecutor(threads) as ex:
        list(ex.map(block, range(cuts.size - 1)))
    return out


def test_pagerank_s26_first_steps_every_row(acsr, cuda):
    """C4 at BASELINE size (R-MAT s26 in-link pattern: 67 M rows, ~1.06 B nnz), in the
    launch configuration bench.py times (one fused acsr_pagerank_step per iteration from
    the cold start): bins bitwise, and for each of the first three steps EVERY row against
    the oracle step taken from the same iterate ("at s26, check parity on the
    first 3 PageRank steps in full"), plus x'/outdeg bitwise and Delta^2."""
    rp, ci = synth.rmat_csr(26, device=cuda, transpose=True)
    n = rp.numel() - 1
    od = torch.bincount(ci.long(), minlength=n).to(torch.int32)
    m = acsr.ACSRMatrix(rp, ci)
    rph = rp.cpu().numpy()
    br, off = oracle.bins(rph)
    assert np.array_equal(m.bin_offsets.cpu().numpy(), off)
    assert np.array_equal(m.bin_rows.cpu().numpy(), br)
    del br
    cih = ci.cpu().numpy()
    odh = od.cpu().numpy()
    teleport = (1.0 - 0.85) / n
    x = torch.full((n,), 1.0 / n, dtype=torch.float64, device=cuda)
    xs = acsr.acsr_pagerank_scale(x, od)
    xn, xsn = torch.empty_like(x), torch.empty_like(x)
    d2 = torch.zeros(1, dtype=torch.float64, device=cuda)
    for step in range(3):
        acsr.acsr_pagerank_step(m.row_begin, m.col_idx, m.bin_rows, m.bin_offsets, m.plan_ws, xs, x, od,
                                xn, xsn, d2, 0.85, teleport, n)
        xh = x.cpu().numpy()
        ref = _oracle_pagerank_step_parallel(rph, cih, odh, xh, teleport, 0.85)
        got = xn.cpu().numpy()
        # step bar (fp64 O5): |err| <= 1e-12 * (teleport + d * sum |xs|) = 1e-12 * ref (all >= 0)
        bad = np.abs(got - ref) > 1e-12 * ref
        assert not bad.any(), (step, np.flatnonzero(bad)[:10], np.max(np.abs(got - ref) / ref))
        # the scaled vector the next step gathers is x'/outdeg (IEEE division): bitwise
        xs_ref = np.where(odh > 0, got / np.maximum(odh, 1), 0.0)
        assert np.array_equal(xsn.cpu().numpy(), xs_ref), step
        # Delta^2 = sum (x' - x)^2 (exact fixed point on the GPU; compared to the oracle rows)
        assert float(d2.item()) == pytest.approx(float(np.sum((ref - xh) ** 2)), rel=1e-9)
        x, xn = xn, x
        xs, xsn = xsn, xs


def test_pagerank_closed_forms(acsr, cuda):
    # directed cycle -> uniform 1/n after one step
    n = 10007
    rp = torch.arange(n + 1, dtype=torch.int32)
    ci = ((torch.arange(n) - 1) % n).to(torch.int32)  # in-link of v is v-1
    od = torch.ones(n, dtype=torch.int32)
    m = acsr.ACSRMatrix(rp.to(cuda), ci.to(cuda))
    x, it, _ = acsr.pagerank(m, od.to(cuda))
    assert it == 1 and torch.allclose(x.cpu(), torch.full((n,), 1.0 / n, dtype=torch.float64), rtol=2e-16, atol=0)
    # a -> b (b dangling): (1-d)/2 and (1-d)(1+d)/2 (tests/golden/pagerank_two_vertex.txt)
    m = acsr.ACSRMatrix(torch.tensor([0, 0, 1], dtype=torch.int32, device=cuda),
                        torch.tensor([0], dtype=torch.int32, device=cuda))
    x, it, _ = acsr.pagerank(m, torch.tensor([1, 0], dtype=torch.int32, device=cuda), eps=1e-15)
    assert x[0].item() == pytest.approx(0.075, rel=1e-15)
    assert x[1].item() == pytest.approx(0.13875, rel=1e-15)


# ------------------------------------------------------------------------------ update
def _slack_graph(scale, frac=4, dtype=torch.float64):
    rp, ci = synth.rmat_csr(scale, transpose=True)
    val = synth.values(ci.numel(), 5, dtype)
    rb, re, cap, c2, v2 = synth.with_slack(rp, ci, val, frac=frac)
    n = rp.numel() - 1
    od = torch.bincount(ci.long(), minlength=n).to(torch.int32)
    return n, rb, re, cap, c2, v2, od, rp, ci


def _dev_changes(ch, dev):
    return {k: torch.from_numpy(v).to(dev) for k, v in ch.items()}


@pytest.mark.parametrize("dtype", [torch.float64, torch.float32])
def test_update_insert_bitwise(acsr, cuda, dtype):
    n, rb, re, cap, col, val, od, rp, ci = _slack_graph(14, dtype=dtype)
    keys = np.sort(np.repeat(np.arange(n), np.diff(rp.numpy())).astype(np.int64) * n + ci.numpy())
    ch, _ = next(synth.insert_batches(14, 1, 4096, keys))
    iv = synth.values(ch["ins_cols"].size, 99, dtype)
    # oracle on host copies
    re_h, col_h, val_h, od_h = re.numpy().copy(), col.numpy().copy(), val.numpy().copy(), od.numpy().copy()
    code, idx = oracle.update(n, rb.numpy(), re_h, cap.numpy(), col_h, val_h, ch["upd_rows"], None, None,
                              ch["ins_ptr"], ch["ins_cols"], iv.numpy(), od_h)
    assert code == 0
    m = acsr.ACSRMatrix(rb.to(cuda), col.to(cuda), val.to(cuda), row_end=re.to(cuda), row_cap=cap.to(cuda),
                        nnz_max=col.numel())
    odd = od.to(cuda)
    st = m.update(_dev_changes(ch, cuda), outdeg=odd, ins_vals=iv.to(cuda))
    torch.cuda.synchronize()
    assert st.cpu().tolist() == [0, -1]
    re_g = m.row_end.cpu().numpy()
    assert np.array_equal(re_g, re_h)
    col_g, val_g = m.col_idx.cpu().numpy(), m.values.cpu().numpy()
    live = np.concatenate([np.arange(b, e) for b, e in zip(rb.numpy(), re_h)])
    assert np.array_equal(col_g[live], col_h[live])
    assert np.array_equal(val_g[live].view(np.uint8), val_h[live].view(np.uint8))
    assert np.array_equal(odd.cpu().numpy(), od_h)
    # re-bin + SpMV on the updated slack CSR vs the oracle
    m.rebin()
    x = synth.vector(n, 6, dtype)
    y = m.spmv(x.to(cuda)).cpu().numpy()
    br, off = oracle.bins(rb.numpy(), re_h)
    assert np.array_equal(m.bin_rows.cpu().numpy(), br)
    y_ref, den = oracle.spmv(rb.numpy(), col_h, val_h, x.numpy(), row_end=re_h)
    check_spmv(y, y_ref, den, dtype)


def test_update_graph_replay_bitwise(acsr, cuda):
    """C5 through one captured CUDA graph (acsr_update_edges_dev with the batch size on the
    device -> acsr_bin -> acsr_pagerank_scale -> acsr_spmv), replayed for three insert
    batches of different sizes: the pattern slack CSR, outdeg, bins and y equal the oracle
    applied batch by batch; a device count above the capacity rejects the batch whole."""
    n, rb, re, cap, col, _, od, rp, ci = _slack_graph(14, frac=1)
    keys = np.sort(np.repeat(np.arange(n), np.diff(rp.numpy())).astype(np.int64) * n + ci.numpy())
    batches = [ch for ch, _ in synth.insert_batches(14, 3, 4096, keys)]
    m = acsr.ACSRMatrix(rb.to(cuda), col.to(cuda), None, row_end=re.to(cuda), row_cap=cap.to(cuda),
                        nnz_max=col.numel())
    odd = od.to(cuda)
    x = (synth.vector(n, 7).abs() + 0.5).to(cuda)
    xs, y = torch.empty_like(x), torch.empty_like(x)
    g = acsr.UpdateGraph(m, odd, x, xs, y, max_upd=6000, max_ins=6000)
    re_h, col_h, od_h = re.numpy().copy(), col.numpy().copy(), od.numpy().copy()
    for ch in batches:
        code, _ = oracle.update(n, rb.numpy(), re_h, cap.numpy(), col_h, None, ch["upd_rows"], None, None,
                                ch["ins_ptr"], ch["ins_cols"], None, od_h)
        assert code == 0
        st = g.replay({k: torch.from_numpy(v).pin_memory() for k, v in ch.items()})
        torch.cuda.synchronize()
        assert st.cpu().tolist() == [0, -1]
        assert np.array_equal(m.row_end.cpu().numpy(), re_h)
        live = np.concatenate([np.arange(b, e) for b, e in zip(rb.numpy(), re_h)])
        assert np.array_equal(m.col_idx.cpu().numpy()[live], col_h[live])
        assert np.array_equal(odd.cpu().numpy(), od_h)
        br, off = oracle.bins(rb.numpy(), re_h)
        assert np.array_equal(m.bin_rows.cpu().numpy(), br)
        xs_ref = np.where(od_h > 0, x.cpu().numpy() / np.maximum(od_h, 1), 0.0)
        y_ref, den = oracle.spmv(rb.numpy(), col_h, None, xs_ref, row_end=re_h)
        check_spmv(y.cpu().numpy(), y_ref, den, torch.float64)
    # the same three batches replayed back to back with NO synchronisation in between
    # (the pinned batch size must not be overwritten before its copy ran)
    m2 = acsr.ACSRMatrix(rb.to(cuda), col.to(cuda), None, row_end=re.to(cuda), row_cap=cap.to(cuda),
                         nnz_max=col.numel())
    odd2 = od.to(cuda)
    y2 = torch.empty_like(x)
    g2 = acsr.UpdateGraph(m2, odd2, x, torch.empty_like(x), y2, max_upd=6000, max_ins=6000)
    for ch in batches:
        g2.replay({k: torch.from_numpy(v).pin_memory() for k, v in ch.items()})
    torch.cuda.synchronize()
    assert g2.status.cpu().tolist() == [0, -1]
    assert np.array_equal(m2.row_end.cpu().numpy(), re_h)
    assert np.array_equal(m2.col_idx.cpu().numpy()[live], col_h[live])
    assert np.array_equal(odd2.cpu().numpy(), od_h) and torch.equal(y2, y)
    # a device batch size beyond the capacity buffers: rejected, nothing modified
    before = m.col_idx.clone(), m.row_end.clone()
    g.n_host[0] = 7000
    g.n_dev.copy_(g.n_host)
    g.graph.replay()
    torch.cuda.synchronize()
    assert g.status.cpu().tolist() == [acsr.ACSR_ERR_INVALID_VALUE, 0]
    assert torch.equal(m.col_idx, before[0]) and torch.equal(m.row_end, before[1])


def test_update_mixed_bitwise(acsr, cuda):
    n, rb, re, cap, col, val, od, rp, ci = _slack_graph(12, frac=1)
    ch = next(synth.mixed_batches(rp.numpy(), ci.numpy(), n, 0.1, 5, 1))
    re_h, col_h, od_h = re.numpy().copy(), col.numpy().copy(), od.numpy().copy()
    code, _ = oracle.update(n, rb.numpy(), re_h, cap.numpy(), col_h, None, ch["upd_rows"], ch["del_ptr"],
                            ch["del_cols"], ch["ins_ptr"], ch["ins_cols"], None, od_h)
    assert code == 0
    m = acsr.ACSRMatrix(rb.to(cuda), col.to(cuda), None, row_end=re.to(cuda), row_cap=cap.to(cuda),
                        nnz_max=col.numel())
    odd = od.to(cuda)
    st = m.update(_dev_changes(ch, cuda), outdeg=odd)
    torch.cuda.synchronize()
    assert st.cpu().tolist() == [0, -1]
    assert np.array_equal(m.row_end.cpu().numpy(), re_h)
    live = np.concatenate([np.arange(b, e) for b, e in zip(rb.numpy(), re_h)])
    assert np.array_equal(m.col_idx.cpu().numpy()[live], col_h[live])
    assert np.array_equal(odd.cpu().numpy(), od_h)


def test_update_rejections_leave_matrix_unchanged(acsr, cuda):
    n, rb, re, cap, col, val, od, rp, ci = _slack_graph(10)
    m = acsr.ACSRMatrix(rb.to(cuda), col.to(cuda), val.to(cuda), row_end=re.to(cuda), row_cap=cap.to(cuda),
                        nnz_max=col.numel())
    odd = od.to(cuda)
    snap = [t.clone() for t in (m.row_end, m.col_idx, m.values, odd)]
    free7 = int(cap[7] - (re[7] - rb[7]))
    cases = [
        (dict(upd_rows=[3, 7], ins_ptr=[0, 1, free7 + 2], ins_cols=[1] + [2] * (free7 + 1)), [3, 1]),
        (dict(upd_rows=[5, 5], ins_ptr=[0, 1, 2], ins_cols=[1, 2]), [1, 1]),
        (dict(upd_rows=[5, 6], ins_ptr=[0, 1, 2], ins_cols=[1, n]), [1, 1]),
        (dict(upd_rows=[5, 6], ins_ptr=[0, 1, 2], ins_cols=[1, 2], del_ptr=[0, 0, 2], del_cols=[9, 3]), [1, 1]),
    ]
    for ch, expect in cases:
        chd = {k: torch.tensor(v, dtype=torch.int32, device=cuda) for k, v in ch.items()}
        st = m.update(chd, outdeg=odd)
        torch.cuda.synchronize()
        assert st.cpu().tolist() == expect
        for a, b in zip((m.row_end, m.col_idx, m.values, odd), snap):
            assert torch.equal(a, b)


def test_understated_nnz_max_is_loud(acsr, cuda):
    """An nnz_max smaller than the stored entries overflows the plan's work list: the plan
    is marked invalid, acsr_plan_status raises ACSR_ERR_CAPACITY, the SpMV writes NaN to
    every row (never stale data) and a device-side PageRank loop stops with
    ctrl[0] = ACSR_CTRL_PLAN_ERROR and Delta^2 = NaN (no silent failure)."""
    n, L = 64, 20000
    rp = torch.arange(n + 1, dtype=torch.int32) * L
    ci = (torch.arange(n * L) % n).to(torch.int32)
    x = torch.ones(n, dtype=torch.float64, device=cuda)
    m = acsr.ACSRMatrix(rp.to(cuda), ci.to(cuda), None, nnz_max=1000)
    with pytest.raises(acsr.ACSRError, match="ACSR_ERR_CAPACITY"):
        m.plan_status()
    y = torch.zeros(n, dtype=torch.float64, device=cuda)
    m.spmv(x, y)
    assert torch.isnan(y).all()
    od = torch.full((n,), L, dtype=torch.int32, device=cuda)
    with pytest.raises(acsr.ACSRError, match="ACSR_ERR_CAPACITY"):
        acsr.pagerank(m, od)
    xs = acsr.acsr_pagerank_scale(x / n, od)
    xn, xsn = torch.zeros_like(x), torch.zeros_like(x)
    d2 = torch.zeros(1, dtype=torch.float64, device=cuda)
    ctrl = torch.zeros(2, dtype=torch.int32, device=cuda)
    acsr.acsr_pagerank_step(m.row_begin, m.col_idx, m.bin_rows, m.bin_offsets, m.plan_ws, xs, x / n, od, xn, xsn,
                            d2, ctrl=ctrl, eps2=1.0)
    assert int(ctrl[0]) == acsr.ACSR_CTRL_PLAN_ERROR and torch.isnan(d2).all() and torch.isnan(xn).all()
    # the same matrix with a correct bound is fine
    m2 = acsr.ACSRMatrix(rp.to(cuda), ci.to(cuda), None)
    m2.plan_status()
    assert torch.equal(m2.spmv(x), torch.full((n,), float(L), dtype=torch.float64, device=cuda))


def test_argument_errors(acsr, cuda):
    with pytest.raises(TypeError):
        acsr.acsr_bin(torch.zeros(3, dtype=torch.int32), None, nnz_max=0)  # CPU tensor
    rp = torch.zeros(3, dtype=torch.int32, device=cuda)
    with pytest.raises(acsr.ACSRError) as e:
        acsr.acsr_bin(rp, None, nnz_max=0, plan_ws=torch.empty(8, dtype=torch.uint8, device=cuda))
    assert e.value.code == acsr.ACSR_ERR_WORKSPACE


@pytest.mark.parametrize("shift_c,shift_v", [(1, 1), (2, 0), (3, 3), (1, 0)])
def test_spmv_unaligned_views(acsr, cuda, shift_c, shift_v):
    # col/val given as offset views: the 128-bit load phase (or the scalar fallback when
    # col and val phases disagree) must not change results beyond the fp64 bar.
    rp, ci = synth.rmat_csr(13)
    n = rp.numel() - 1
    val = synth.values(ci.numel(), 21)
    x = synth.vector(n, 22)
    cbuf = torch.zeros(ci.numel() + 4, dtype=torch.int32, device=cuda)
    vbuf = torch.zeros(ci.numel() + 4, dtype=torch.float64, device=cuda)
    cv = cbuf[shift_c:shift_c + ci.numel()]
    vv = vbuf[shift_v:shift_v + ci.numel()]
    cv.copy_(ci.to(cuda))
    vv.copy_(val.to(cuda))
    m = acsr.ACSRMatrix(rp.to(cuda), cv, vv)
    y = m.spmv(x.to(cuda)).cpu().numpy()
    y_ref, den = oracle.spmv(rp.numpy(), ci.numpy(), val.numpy(), x.numpy())
    check_spmv(y, y_ref, den, torch.float64)


@pytest.mark.parametrize("dtype", [torch.float64, torch.float32])
@pytest.mark.parametrize("shift_x", [0, 1, 3])
def test_spmv_x_prefetch_views(acsr, cuda, dtype, shift_x):
    # x given as an offset view (the L2 bulk prefetch of x is clipped inward to 16-byte
    # bounds) and with the prefetch disabled by size (x of one column): results are the
    # same bits as with an aligned x (bitwise on integer data)
    rp, ci = synth.rmat_csr(13)
    n = rp.numel() - 1
    val = synth.values(ci.numel(), 31, dtype, integer=True)
    x = synth.vector(n, 32, dtype, integer=True)
    xbuf = torch.zeros(n + 4, dtype=dtype, device=cuda)
    xv = xbuf[shift_x:shift_x + n]
    xv.copy_(x.to(cuda))
    m = acsr.ACSRMatrix(rp.to(cuda), ci.to(cuda), val.to(cuda))
    y = m.spmv(xv).cpu().numpy()
    y_ref, den = oracle.spmv(rp.numpy(), ci.numpy(), val.numpy(), x.numpy())
    check_spmv(y, y_ref, den, dtype, exact=True)
    # one column: every row sums val * x[0]
    rp1 = torch.tensor([0, 3, 3, 5], dtype=torch.int32)
    ci1 = torch.zeros(5, dtype=torch.int32)
    v1 = torch.tensor([1, -2, 4, 3, 5], dtype=dtype)
    x1 = torch.tensor([2], dtype=dtype)
    m1 = acsr.ACSRMatrix(rp1.to(cuda), ci1.to(cuda), v1.to(cuda), n_cols=1)
    assert m1.spmv(x1.to(cuda)).cpu().tolist() == [6.0, 0.0, 16.0]


def test_dist_pagerank_single_rank_cuda(acsr, cuda):
    # the partitioned driver (dist.py) on one rank runs the same fused CUDA step: it must
    # reproduce the single-GPU loop bitwise and the oracle within the converged bar
    from paper_conf_sc_ashariseps14_b200 import dist as pdist
    rp, ci, od, n = _inlink(14, cuda)
    splits = pdist.partition_rows(np.diff(rp.numpy()), 1)
    pr = pdist.DistPageRank(rp.to(cuda), ci.to(cuda), od.to(cuda), splits, n)
    x, it, d2 = pr.run(eps=1e-6)
    m = acsr.ACSRMatrix(rp.to(cuda), ci.to(cuda))
    x1, it1, d21 = acsr.pagerank(m, od.to(cuda), eps=1e-6)
    assert it == it1 and torch.equal(x, x1)
    x_ref, it_ref, _ = oracle.pagerank(rp.numpy(), ci.numpy(), od.numpy(), eps=1e-6)
    assert abs(it - it_ref) <= 1


def test_capacity_reject_then_grow_and_retry(acsr, cuda):
    # reading R4: a CAPACITY rejection leaves the matrix unchanged; acsr_relayout (via
    # ACSRMatrix.grow) adds slack; the same batch then applies bit-for-bit like the oracle
    n, rb, re, cap, col, val, od, rp, ci = _slack_graph(11)
    m = acsr.ACSRMatrix(rb.to(cuda), col.to(cuda), val.to(cuda), row_end=re.to(cuda), row_cap=cap.to(cuda),
                        nnz_max=col.numel())
    odd = od.to(cuda)
    r = 9
    free = int(cap[r] - (re[r] - rb[r]))
    ins = np.arange(free + 3, dtype=np.int32) % n
    ch = {"upd_rows": torch.tensor([r], dtype=torch.int32, device=cuda),
          "ins_ptr": torch.tensor([0, ins.size], dtype=torch.int32, device=cuda),
          "ins_cols": torch.from_numpy(ins).to(cuda)}
    st = m.update(ch, outdeg=odd)
    assert st.cpu().tolist() == [3, 0]
    live_before = [m.col_idx[m.row_begin[i]:m.row_end[i]].cpu() for i in range(0, n, 97)]
    m.grow()
    live_after = [m.col_idx[m.row_begin[i]:m.row_end[i]].cpu() for i in range(0, n, 97)]
    assert all(torch.equal(a, b) for a, b in zip(live_before, live_after))
    st = m.update(ch, outdeg=odd)
    torch.cuda.synchronize()
    assert st.cpu().tolist() == [0, -1]
    got = m.col_idx[m.row_begin[r]:m.row_end[r]].cpu().numpy()
    exp = np.concatenate([col.numpy()[rb[r]:re[r]], ins])
    assert np.array_equal(got, exp)
    assert int(odd.sum()) == int(od.sum()) + ins.size
    m.rebin()
    x = synth.vector(n, 3)
    y = m.spmv(x.to(cuda)).cpu().numpy()
    y_ref, den = oracle.spmv(m.row_begin.cpu().numpy(), m.col_idx.cpu().numpy(), m.values.cpu().numpy(),
                             x.numpy(), row_end=m.row_end.cpu().numpy())
    check_spmv(y, y_ref, den, torch.float64)


# ------------------------------------------------------------------------------ RWR / HITS
def test_rwr_parity(acsr, cuda):
    rp, ci, od, n = _inlink(14, cuda)
    i = int(np.argmax(od.numpy()))  # restart at a hub
    m = acsr.ACSRMatrix(rp.to(cuda), ci.to(cuda))
    r, it, d2 = acsr.rwr(m, od.to(cuda), i, c=0.85, eps=1e-6)
    r_ref, it_ref, _ = oracle.rwr(rp.numpy(), ci.numpy(), od.numpy(), i, c=0.85, eps=1e-6)
    assert abs(it - it_ref) <= 1
    if it != it_ref:
        r_ref, _, _ = oracle.rwr(rp.numpy(), ci.numpy(), od.numpy(), i, c=0.85, eps=0.0, max_iter=it)
    assert np.all(np.abs(r.cpu().numpy() - r_ref) <= 1e-11 * r_ref + 1e-18)
    # one step from the same iterate meets the fp64 step bar
    rr = synth.vector(n, 9).abs().numpy()
    rs = torch.where(od > 0, torch.from_numpy(rr) / od.clamp(min=1), torch.zeros(n, dtype=torch.float64))
    rn, rsn = torch.empty(n, dtype=torch.float64, device=cuda), torch.empty(n, dtype=torch.float64, device=cuda)
    d2 = torch.zeros(1, dtype=torch.float64, device=cuda)
    acsr.acsr_pagerank_step(m.row_begin, m.col_idx, m.bin_rows, m.bin_offsets, m.plan_ws, rs.to(cuda),
                            torch.from_numpy(rr).to(cuda), od.to(cuda), rn, rsn, d2, 0.85, 0.0, n,
                            restart=i, restart_weight=0.15)
    rn_ref, d2_ref = oracle.rwr_step(rp.numpy(), ci.numpy(), od.numpy(), rr, 0.85, i)
    _, den = oracle.spmv(rp.numpy(), ci.numpy(), None, rs.numpy())
    assert np.all(np.abs(rn.cpu().numpy() - rn_ref) <= 1e-12 * 0.85 * den + 2.3e-16 * np.abs(rn_ref))
    assert float(d2.item()) == pytest.approx(d2_ref, rel=1e-9)


@pytest.mark.parametrize("scale", [12, 16])
def test_hits_parity(acsr, cuda, scale):
    rp, ci = synth.rmat_csr(scale)  # rows = sources: the adjacency A of Eq. 5-6
    n = rp.numel() - 1
    a, h, it = acsr.hits(rp.to(cuda), ci.to(cuda), eps=1e-6)
    rpT, ciT = synth.rmat_csr(scale, transpose=True)
    a_ref, h_ref, it_ref = oracle.hits(rp.numpy(), ci.numpy(), rpT.numpy(), ciT.numpy(), eps=1e-6)
    assert abs(it - it_ref) <= 1
    if it != it_ref:
        a_ref, h_ref, _ = oracle.hits(rp.numpy(), ci.numpy(), rpT.numpy(), ciT.numpy(), eps=0.0, max_iter=it)
    assert np.allclose(a.cpu().numpy(), a_ref, rtol=1e-9, atol=1e-15)
    assert np.allclose(h.cpu().numpy(), h_ref, rtol=1e-9, atol=1e-15)
    # device-side stop test: enqueueing 8 iterations per host check (steps after convergence
    # are no-ops) gives the iterate of a host test after every iteration, bitwise
    a1, h1, it1 = acsr.hits(rp.to(cuda), ci.to(cuda), eps=1e-6, check_every=1)
    assert it1 == it and torch.equal(a1, a) and torch.equal(h1, h)


@pytest.mark.parametrize("scale", [12, 16])
def test_hits_one_step_parity(acsr, cuda, scale):
    """One HITS step (Eq. 5-7 + reading R6) from the same non-normalised iterate: the block
    SpMV + acsr_hits_normalize against oracle.hits_step.  Bar (derived): y = [A^T h; A a]
    has non-negative terms, so the SpMV bar 1e-12 * den is 1e-12 relative per entry; each
    side's norm carries at most a gamma_n sequential error (n u relative on the squared
    sum), so a', h' agree to (1e-12 + 2 n u) relative.  Distances to a far iterate to 1e-9."""
    rp, ci = synth.rmat_csr(scale)
    rpT, ciT = synth.rmat_csr(scale, transpose=True)
    n = rp.numel() - 1
    a = synth.vector(n, 71).abs().numpy()
    h = synth.vector(n, 72).abs().numpy()
    a_ref, h_ref, d2_ref = oracle.hits_step(rp.numpy(), ci.numpy(), rpT.numpy(), ciT.numpy(), a, h)
    bp, bc = acsr.hits_matrix(rp.to(cuda), ci.to(cuda), n)
    B = acsr.ACSRMatrix(bp, bc, None, n_cols=2 * n)
    v = torch.from_numpy(np.concatenate([a, h])).to(cuda)
    y = B.spmv(v)
    vn = torch.empty_like(v)
    d2 = torch.zeros(2, dtype=torch.float64, device=cuda)
    ws = torch.empty(acsr.acsr_hits_workspace_bytes(n), dtype=torch.uint8, device=cuda)
    acsr.acsr_hits_normalize(y, v, vn, d2, ws)
    got = vn.cpu().numpy()
    tol = 1e-12 + 2 * n * 2.0 ** -53
    for g, r in ((got[:n], a_ref), (got[n:], h_ref)):
        assert np.all(np.abs(g - r) <= tol * r + 1e-300)
        assert np.array_equal(g == 0.0, r == 0.0)
    assert d2.cpu().numpy() == pytest.approx(d2_ref, rel=1e-9)


@pytest.mark.parametrize("scale", [14, 20])
def test_degree_relabel_pagerank_equivalent(acsr, cuda, scale):
    # P A P^T relabelling (degree order, acsr_degree_relabel on the device) is a pure
    # renumbering: PR'[perm[v]] == PR[v] within the Q18 bar, iteration count +-1
    rp, ci, od, n = _inlink(scale, cuda)
    rp2, ci2, od2, perm = acsr.degree_relabel(rp.to(cuda), ci.to(cuda), od.to(cuda))
    assert torch.all(od2[:-1] >= od2[1:])
    m = acsr.ACSRMatrix(rp2, ci2)
    x2, it2, _ = acsr.pagerank(m, od2, eps=1e-6)
    x_ref, it_ref, _ = oracle.pagerank(rp.numpy(), ci.numpy(), od.numpy(), eps=1e-6)
    assert abs(it2 - it_ref) <= 1
    if it2 != it_ref:
        x_ref, _, _ = oracle.pagerank(rp.numpy(), ci.numpy(), od.numpy(), eps=0.0, max_iter=it2)
    back = x2[perm].cpu().numpy()
    assert np.all(np.abs(back - x_ref) <= 1e-11 * x_ref + 1e-18)


@pytest.mark.parametrize("sort_rows", [False, True])
@pytest.mark.parametrize("scale", [12, 17])
def test_degree_relabel_structure_bitwise(acsr, cuda, scale, sort_rows):
    """acsr_degree_relabel against its definition, on the host (integer data, bitwise):
    order = vertices by decreasing out-degree, ties by increasing id (numpy stable sort);
    perm = its inverse; new row perm[u] = old row u with every column c replaced by perm[c],
    in the same order; outdeg' = outdeg[order].  Includes rows longer than the 1024-entry
    threshold of the CTA copy path at s17."""
    rp, ci, od, n = _inlink(scale, cuda)
    rp2, c2, od2, perm = acsr.acsr_degree_relabel(rp.to(cuda), ci.to(cuda), od.to(cuda), sort_rows=sort_rows)
    rph, cih, odh = rp.numpy(), ci.numpy(), od.numpy()
    order = np.argsort(-odh.astype(np.int64), kind="stable")
    pr = np.empty(n, np.int64)
    pr[order] = np.arange(n)
    assert np.array_equal(perm.cpu().numpy(), pr)
    assert np.array_equal(od2.cpu().numpy(), odh[order])
    ln = np.diff(rph)
    rp_ref = np.zeros(n + 1, np.int64)
    rp_ref[1:] = np.cumsum(ln[order])
    assert np.array_equal(rp2.cpu().numpy(), rp_ref)
    starts = np.repeat(rph[:-1][order] - rp_ref[:-1], ln[order])
    src = np.arange(cih.size) + starts  # old position of every new entry
    ref = pr[cih[src]]
    if sort_rows:  # each row's columns ascending (numpy lexsort by (row, col))
        rows = np.repeat(np.arange(n), ln[order])
        ref = ref[np.lexsort((ref, rows))]
    assert np.array_equal(c2.cpu().numpy(), ref)
    if scale == 17:
        assert ln.max() > 1024


def test_paper_epoch_update_bitwise(acsr, cuda):
    # P:337 paper-shaped epoch generated on the device from the live graph (synth.mixed_epoch)
    n, rb, re, cap, col, val, od, rp, ci = _slack_graph(14, frac=1)
    m = acsr.ACSRMatrix(rb.to(cuda), col.to(cuda), None, row_end=re.to(cuda), row_cap=cap.to(cuda),
                        nnz_max=col.numel())
    odd = od.to(cuda)
    re_h, col_h, od_h = re.numpy().copy(), col.numpy().copy(), od.numpy().copy()
    for ep in range(3):
        ch = synth.mixed_epoch(m.row_begin, m.row_end, m.col_idx, n, 0.1, 77 + ep)
        code, _ = oracle.update(n, rb.numpy(), re_h, cap.numpy(), col_h, None, ch["upd_rows"], ch["del_ptr"],
                                ch["del_cols"], ch["ins_ptr"], ch["ins_cols"], None, od_h)
        st = m.update(_dev_changes(ch, cuda), outdeg=odd)
        torch.cuda.synchronize()
        assert st.cpu().tolist() == [code, -1 if code == 0 else st.cpu().tolist()[1]]
        if code != 0:
            break
        assert np.array_equal(m.row_end.cpu().numpy(), re_h)
        live = np.concatenate([np.arange(b, e) for b, e in zip(rb.numpy(), re_h)])
        assert np.array_equal(m.col_idx.cpu().numpy()[live], col_h[live])
        assert np.array_equal(odd.cpu().numpy(), od_h)


def _live(rb, re):
    """Indices of the stored entries of a slack CSR (vectorised)."""
    ln = (re - rb).astype(np.int64)
    return np.repeat(rb.astype(np.int64) - np.concatenate([[0], np.cumsum(ln)[:-1]]), ln) + np.arange(int(ln.sum()))


def test_c5_full_size_batches_bitwise(acsr, cuda):
    """C5 at BASELINE size in the bench's configuration (R-MAT s20 in-link pattern, slack
    cap = len + max(4, ceil(len/4)), 16,384-edge insert batches from the same R-MAT, seeds
    3000 + b): two batches through acsr_update_edges -> acsr_bin -> acsr_spmv; col, row_end,
    outdeg and bins bitwise against the oracle (O7, O3) after each batch, y = A xs at the fp64
    bar; then one paper-shaped mixed epoch (N2) bitwise."""
    S = 20
    rp, ci = synth.rmat_csr(S, transpose=True)
    n = rp.numel() - 1
    od = torch.bincount(ci.long(), minlength=n).to(torch.int32)
    rb, re, cap, col, _ = synth.with_slack(rp, ci)
    keys = np.sort(np.repeat(np.arange(n), np.diff(rp.numpy())).astype(np.int64) * n + ci.numpy())
    m = acsr.ACSRMatrix(rb.to(cuda), col.to(cuda), None, row_end=re.to(cuda), row_cap=cap.to(cuda),
                        nnz_max=col.numel())
    odd = od.to(cuda)
    rb_h, cap_h = rb.numpy(), cap.numpy()
    re_h, col_h, od_h = re.numpy().copy(), col.numpy().copy(), od.numpy().copy()
    x = (synth.vector(n, 7).abs() + 0.5)
    for ch, _ in synth.insert_batches(S, 2, 16384, keys):
        code, _ = oracle.update(n, rb_h, re_h, cap_h, col_h, None, ch["upd_rows"], None, None, ch["ins_ptr"],
                                ch["ins_cols"], None, od_h)
        st = m.update(_dev_changes(ch, cuda), outdeg=odd)
        torch.cuda.synchronize()
        assert st.cpu().tolist() == [code, -1 if code == 0 else st.cpu().tolist()[1]]
        if code != 0:  # capacity: both sides rejected the whole batch, nothing changed
            continue
        assert np.array_equal(m.row_end.cpu().numpy(), re_h)
        live = _live(rb_h, re_h)
        assert np.array_equal(m.col_idx.cpu().numpy()[live], col_h[live])
        assert np.array_equal(odd.cpu().numpy(), od_h)
        m.rebin()
        m.plan_status()
        br, off = oracle.bins(rb_h, re_h)
        assert np.array_equal(m.bin_rows.cpu().numpy(), br) and np.array_equal(m.bin_offsets.cpu().numpy(), off)
        xs = np.where(od_h > 0, x.numpy() / np.maximum(od_h, 1), 0.0)
        y = m.spmv(torch.from_numpy(xs).to(cuda)).cpu().numpy()
        y_ref, den = oracle.spmv(rb_h, col_h, None, xs, row_end=re_h)
        check_spmv(y, y_ref, den, torch.float64)
    ch = synth.mixed_epoch(m.row_begin, m.row_end, m.col_idx, n, 0.1, 91)
    code, _ = oracle.update(n, rb_h, re_h, cap_h, col_h, None, ch["upd_rows"], ch["del_ptr"], ch["del_cols"],
                            ch["ins_ptr"], ch["ins_cols"], None, od_h)
    st = m.update(_dev_changes(ch, cuda), outdeg=odd)
    torch.cuda.synchronize()
    assert int(st[0]) == code
    if code == 0:
        assert np.array_equal(m.row_end.cpu().numpy(), re_h)
        live = _live(rb_h, re_h)
        assert np.array_equal(m.col_idx.cpu().numpy()[live], col_h[live])
        assert np.array_equal(odd.cpu().numpy(), od_h)


def test_update_long_row_cta_path(acsr, cuda):
    # hub rows (> 2048 entries) with deletes take the CTA-per-row validate/compact path
    lens = [3, 10000, 5, 40000, 0, 2049]
    rp, ci = synth.boundary_csr(lens, 1 << 17, 11)
    val = synth.values(ci.numel(), 12)
    rb, re, cap, col, v2 = synth.with_slack(rp, ci, val)
    n = len(lens)
    od = torch.bincount(ci.long(), minlength=1 << 17).to(torch.int32)
    rng = np.random.default_rng(3)
    upd = np.array([1, 2, 3, 5], np.int32)
    dels, inss = [], []
    for r in upd:
        cur = ci.numpy()[rp[r]:rp[r + 1]]
        dels.append(np.unique(rng.choice(cur, size=len(cur) // 2)))
        inss.append(rng.integers(0, 1 << 17, size=min(len(cur) // 5, 40)).astype(np.int32))
    ch = {"upd_rows": upd,
          "del_ptr": np.concatenate([[0], np.cumsum([d.size for d in dels])]).astype(np.int32),
          "del_cols": np.concatenate(dels).astype(np.int32),
          "ins_ptr": np.concatenate([[0], np.cumsum([a.size for a in inss])]).astype(np.int32),
          "ins_cols": np.concatenate(inss).astype(np.int32)}
    re_h, col_h, v_h, od_h = re.numpy().copy(), col.numpy().copy(), v2.numpy().copy(), od.numpy().copy()
    code, _ = oracle.update(1 << 17, rb.numpy(), re_h, cap.numpy(), col_h, v_h, ch["upd_rows"], ch["del_ptr"],
                            ch["del_cols"], ch["ins_ptr"], ch["ins_cols"], None, od_h)
    assert code == 0
    m = acsr.ACSRMatrix(rb.to(cuda), col.to(cuda), v2.to(cuda), n_cols=1 << 17, row_end=re.to(cuda),
                        row_cap=cap.to(cuda), nnz_max=col.numel())
    odd = od.to(cuda)
    st = m.update(_dev_changes(ch, cuda), outdeg=odd)
    torch.cuda.synchronize()
    assert st.cpu().tolist() == [0, -1]
    assert np.array_equal(m.row_end.cpu().numpy(), re_h)
    live = np.concatenate([np.arange(b, e) for b, e in zip(rb.numpy(), re_h)])
    assert np.array_equal(m.col_idx.cpu().numpy()[live], col_h[live])
    assert np.array_equal(m.values.cpu().numpy()[live].view(np.uint8), v_h[live].view(np.uint8))
    assert np.array_equal(odd.cpu().numpy(), od_h)
    # a long-row capacity failure is reported at its index, nothing applied
    snap = [t.clone() for t in (m.row_end, m.col_idx, odd)]
    r = 3
    free = int(m.row_cap[r] - (m.row_end[r] - m.row_begin[r]))
    bad = {"upd_rows": np.array([0, r], np.int32), "del_ptr": np.array([0, 0, 1], np.int32),
           "del_cols": np.array([int(m.col_idx[m.row_begin[r]])], np.int32),
           "ins_ptr": np.array([0, 1, 1 + free + 2], np.int32),
           "ins_cols": np.arange(free + 3, dtype=np.int32)}
    st = m.update(_dev_changes(bad, cuda), outdeg=odd)
    torch.cuda.synchronize()
    assert st.cpu().tolist() == [3, 1]
    for a, b in zip((m.row_end, m.col_idx, odd), snap):
        assert torch.equal(a, b)


def test_property_random_csr_spmv_and_updates(acsr, cuda):
    """Property test (hypothesis, derandomized): random CSR shapes -- row lengths drawn from
    a mixture that hits every mapping (empty, window, Alg. 2 / warp per row, split rows),
    random columns, random n_cols, fp64 and fp32, integer and float values -- bins bitwise,
    SpMV bitwise on integer data and at the O5 bar on float data; then a random insert /
    delete batch on the slack copy, bitwise against O7."""
    from hypothesis import given, settings, strategies as st, HealthCheck

    @settings(max_examples=150, derandomize=True, deadline=None,
              suppress_health_check=[HealthCheck.too_slow, HealthCheck.data_too_large])
    @given(st.integers(1, 700), st.integers(1, 5000), st.integers(0, 2 ** 31 - 1), st.booleans(), st.booleans())
    def check(n, n_cols, seed, f32, integer):
        rng = np.random.default_rng(seed)
        kind = rng.integers(0, 5, n)
        ln = np.where(kind == 0, 0, np.where(kind == 1, rng.integers(1, 33, n),
                      np.where(kind == 2, rng.integers(33, 1025, n),
                               np.where(kind == 3, rng.integers(1025, 3000, n), rng.integers(1, 9, n)))))
        ln = np.minimum(ln, 20000)
        rp = np.zeros(n + 1, np.int64)
        rp[1:] = np.cumsum(ln)
        nnz = int(rp[-1])
        ci = rng.integers(0, n_cols, nnz).astype(np.int32)
        dt = np.float32 if f32 else np.float64
        if integer:
            val = rng.integers(-8, 9, nnz).astype(dt)
            x = rng.integers(-8, 9, n_cols).astype(dt)
        else:
            val = rng.uniform(-1, 1, nnz).astype(dt)
            x = rng.uniform(-1, 1, n_cols).astype(dt)
        rpt = torch.from_numpy(rp.astype(np.int32))
        m, y = run_csr(acsr, rpt, torch.from_numpy(ci), torch.from_numpy(val), torch.from_numpy(x), cuda)
        br, off = oracle.bins(rp.astype(np.int32))
        assert np.array_equal(m.bin_rows.cpu().numpy(), br) and np.array_equal(m.bin_offsets.cpu().numpy(), off)
        y_ref, den = oracle.spmv(rp.astype(np.int32), ci, val, x)
        check_spmv(y.numpy(), y_ref, den, torch.float32 if f32 else torch.float64, exact=integer)
        # a random mixed update batch on the slack copy: O7 bitwise
        rb, re, cap, c2, v2 = synth.with_slack(rpt, torch.from_numpy(ci), torch.from_numpy(val))
        rows = np.unique(rng.integers(0, n, max(1, n // 4))).astype(np.int32)
        dptr, dcol, iptr, icol = [0], [], [0], []
        for r in rows:
            cols_r = c2.numpy()[rb[r]:re[r]]
            k = int(rng.integers(0, min(len(cols_r), 6) + 1))
            dcol += sorted(rng.choice(cols_r, k, replace=False).tolist()) if k else []
            dptr.append(len(dcol))
            icol += rng.integers(0, n_cols, int(rng.integers(0, 5))).tolist()
            iptr.append(len(icol))
        ch = {"upd_rows": rows, "del_ptr": np.array(dptr, np.int32), "del_cols": np.array(dcol, np.int32),
              "ins_ptr": np.array(iptr, np.int32), "ins_cols": np.array(icol, np.int32)}
        iv = rng.uniform(-1, 1, len(icol)).astype(dt)
        re_h, c_h, v_h = re.numpy().copy(), c2.numpy().copy(), v2.numpy().copy()
        code, idx = oracle.update(n_cols, rb.numpy(), re_h, cap.numpy(), c_h, v_h, rows, ch["del_ptr"], ch["del_cols"],
                                  ch["ins_ptr"], ch["ins_cols"], iv)
        mu = acsr.ACSRMatrix(rb.to(cuda), c2.to(cuda), v2.to(cuda), n_cols=n_cols, row_end=re.to(cuda),
                             row_cap=cap.to(cuda), nnz_max=c2.numel())
        stt = mu.update({k: torch.from_numpy(v).to(cuda) for k, v in ch.items()}, ins_vals=torch.from_numpy(iv).to(cuda))
        torch.cuda.synchronize()
        assert stt.cpu().tolist() == [code, idx]
        assert np.array_equal(mu.row_end.cpu().numpy(), re_h)
        live = _live(rb.numpy(), re_h)
        assert np.array_equal(mu.col_idx.cpu().numpy()[live], c_h[live])
        assert np.array_equal(mu.values.cpu().numpy()[live].view(np.uint8), v_h[live].view(np.uint8))

    check()


def test_property_multi_tile_spmv(acsr, cuda):
    """Property test (hypothesis, derandomized) over MANY tiles: 1025 .. 120000 rows, so plans
    hold full and ragged tiles, the 4x smaller units of the tail tiles (ACSR_TAIL_DIV) next
    to ordinary ones, windows that straddle long rows, and split rows anywhere in the list;
    bins bitwise, SpMV bitwise on integer data and at the O5 bar on float data."""
    from hypothesis import given, settings, strategies as st, HealthCheck

    @settings(max_examples=60, derandomize=True, deadline=None,
              suppress_health_check=[HealthCheck.too_slow, HealthCheck.data_too_large])
    @given(st.integers(1025, 120000), st.integers(1, 200000), st.integers(0, 2 ** 31 - 1), st.booleans(), st.booleans())
    def check(n, n_cols, seed, f32, integer):
        rng = np.random.default_rng(seed)
        u = rng.random(n)
        ln = np.where(u < 0.15, 0, np.where(u < 0.75, rng.integers(1, 33, n),
                      np.where(u < 0.97, rng.integers(33, 1025, n),
                               np.where(u < 0.995, rng.integers(1, 5, n), rng.integers(1025, 5000, n)))))
        rp = np.zeros(n + 1, np.int64)
        rp[1:] = np.cumsum(ln)
        nnz = int(rp[-1])
        ci = rng.integers(0, n_cols, nnz).astype(np.int32)
        dt = np.float32 if f32 else np.float64
        if integer:
            val = rng.integers(-8, 9, nnz).astype(dt)
            x = rng.integers(-8, 9, n_cols).astype(dt)
        else:
            val = rng.uniform(-1, 1, nnz).astype(dt)
            x = rng.uniform(-1, 1, n_cols).astype(dt)
        rpt = torch.from_numpy(rp.astype(np.int32))
        m, y = run_csr(acsr, rpt, torch.from_numpy(ci), torch.from_numpy(val), torch.from_numpy(x), cuda)
        br, off = oracle.bins(rp.astype(np.int32))
        assert np.array_equal(m.bin_rows.cpu().numpy(), br) and np.array_equal(m.bin_offsets.cpu().numpy(), off)
        y_ref, den = oracle.spmv(rp.astype(np.int32), ci, val, x)
        check_spmv(y.numpy(), y_ref, den, torch.float32 if f32 else torch.float64, exact=integer)

    check()


def test_c_abi_from_plain_c(cuda):
    # the boundary is usable without Python: compile tests/c/capi_smoke.c against
    # include/acsr.h and libacsr.so and run it
    import os
    import subprocess
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    lib = os.path.join(root, "paper_conf_sc_ashariseps14_b200", "lib")
    exe = os.path.join(lib, "capi_smoke")
    subprocess.check_call(["nvcc", "-Wno-deprecated-gpu-targets", "-o", exe, os.path.join(root, "tests", "c", "capi_smoke.c"),
                           "-L" + lib, "-lacsr", "-Xlinker", "-rpath=" + lib])
    out = subprocess.run([exe], capture_output=True, text=True, timeout=120)
    assert out.returncode == 0, out.stdout + out.stderr
    assert "capi_smoke OK" in out.stdout


def test_spmv_from_host_e2e(acsr, cuda):
    rp, ci = synth.rmat_csr(13)
    val = synth.values(ci.numel(), 3)
    x = synth.vector(rp.numel() - 1, 4)
    y = acsr.spmv_from_host(rp.pin_memory(), ci.pin_memory(), val.pin_memory(), x.pin_memory(), device=cuda)
    y_ref, den = oracle.spmv(rp.numpy(), ci.numpy(), val.numpy(), x.numpy())
    check_spmv(y.numpy(), y_ref, den, torch.float64)


def test_spmv_from_host_two_streams(acsr, cuda):
    """The double-buffered end-to-end pattern bench.py times: calls alternating between two
    streams, each with its own pinned output, overlap in flight; every result equals the
    one-stream call bit for bit (and the oracle at the fp64 bar)."""
    rp, ci = synth.rmat_csr(15)
    val = synth.values(ci.numel(), 5)
    x = synth.vector(rp.numel() - 1, 6)
    h = [t.pin_memory() for t in (rp, ci, val, x)]
    y1 = acsr.spmv_from_host(*h, device=cuda)
    sts = [torch.cuda.Stream(device=cuda) for _ in range(2)]
    outs = [torch.empty_like(x).pin_memory() for _ in range(6)]
    for k in range(6):
        acsr.spmv_from_host(*h, outs[k], device=cuda, stream=sts[k % 2])
    torch.cuda.synchronize()
    for o in outs:
        assert torch.equal(o, y1)
    y_ref, den = oracle.spmv(rp.numpy(), ci.numpy(), val.numpy(), x.numpy())
    check_spmv(y1.numpy(), y_ref, den, torch.float64)


def _two_ranks(scale, world=2, **kw):
    import socket
    import sys
    import torch.multiprocessing as mp
    sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
    import _dist_gpu_worker
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_dist_gpu_worker.worker, args=(r, world, port, scale, q), kwargs=kw)
             for r in range(world)]
    for p in procs:
        p.start()
    full, it, d2 = q.get(timeout=300)
    for p in procs:
        p.join(60)
        assert p.exitcode == 0
    return full, it, d2


def test_dist_pagerank_two_ranks_one_gpu(cuda):
    # the partitioned driver with two ranks sharing the GPU (gloo for the exchange): CUDA
    # step + column renumbering + padded all-gather + Delta^2 all-reduce vs the oracle
    full, it, _ = _two_ranks(14)
    rp, ci, od, n = _inlink(14, cuda)
    x_ref, it_ref, _ = oracle.pagerank(rp.numpy(), ci.numpy(), od.numpy(), eps=1e-6)
    assert abs(it - it_ref) <= 1
    if it != it_ref:
        x_ref, _, _ = oracle.pagerank(rp.numpy(), ci.numpy(), od.numpy(), eps=0.0, max_iter=it)
    assert np.all(np.abs(full - x_ref) <= 1e-11 * x_ref + 1e-18)


@pytest.mark.parametrize("compact", [True, False])
def test_dist_pagerank_acsr_comm_two_ranks(cuda, compact):
    """The library-owned exchange (acsr_comm: NCCL all-gather of the xs slices + exact
    global Delta^2 inside acsr_pagerank_step) with two ranks, here sharing one GPU (NCCL
    over its socket transport; see the worker).  Same iterate, iteration count and
    Delta^2 bits as the torch.distributed exchange, and the oracle bar."""
    full_a, it_a, d2_a = _two_ranks(14, exchange="acsr", compact=compact, check_every=4)
    full_t, it_t, d2_t = _two_ranks(14, exchange="torch", compact=compact)
    assert it_a == it_t
    assert np.array_equal(full_a, full_t)
    # the library adds exact fixed-point partials: the single-GPU Delta^2 of the last step
    rp, ci, od, n = _inlink(14, cuda)
    x_ref, it_ref, _ = oracle.pagerank(rp.numpy(), ci.numpy(), od.numpy(), eps=1e-6)
    assert abs(it_a - it_ref) <= 1
    if it_a != it_ref:
        x_ref, _, _ = oracle.pagerank(rp.numpy(), ci.numpy(), od.numpy(), eps=0.0, max_iter=it_a)
    assert np.all(np.abs(full_a - x_ref) <= 1e-11 * x_ref + 1e-18)
    assert d2_a == pytest.approx(d2_t, rel=1e-12)


def test_acsr_partition_equals_oracle(acsr, cuda):
    """acsr_partition (O8 on the device: CUB prefix + binary search) = oracle.partition bitwise."""
    for scale, P, bn, br, al in ((14, 2, 4, 36, 1), (16, 3, 12, 16, 32), (17, 8, 4, 36, 1), (10, 1, 4, 36, 1),
                                 (15, 5, 12, 16, 1024)):
        rp, ci = synth.rmat_csr(scale, transpose=True)
        got = acsr.acsr_partition(rp.to(cuda), P, bn, br, align=al).cpu().numpy()
        assert np.array_equal(got, oracle.partition(rp.numpy(), P, bn, br, align=al)), (scale, P)
    rb, re, cap, c2, _ = synth.with_slack(*synth.rmat_csr(12))
    got = acsr.acsr_partition(rb.to(cuda), 4, 4, 36, row_end=re.to(cuda)).cpu().numpy()
    assert np.array_equal(got, oracle.partition(rb.numpy(), 4, 4, 36, row_end=re.numpy()))
    empty = acsr.acsr_partition(torch.zeros(1, dtype=torch.int32, device=cuda), 3, 4, 36).cpu().numpy()
    assert np.array_equal(empty, [0, 0, 0, 0])


def test_partition_and_relabel_edge_cases(acsr, cuda):
    """acsr_partition with more ranks than rows and on empty rows; acsr_degree_relabel on a
    one-vertex graph, on a graph without edges (all ties -> identity) and on an empty graph;
    argument errors of the multi-GPU calls."""
    rp = torch.tensor([0, 5, 5, 9], dtype=torch.int32)
    for P in (1, 2, 3, 8):
        got = acsr.acsr_partition(rp.to(cuda), P, 4, 36).cpu().numpy()
        assert np.array_equal(got, oracle.partition(rp.numpy(), P, 4, 36)), P
        assert got[0] == 0 and got[-1] == 3 and np.all(np.diff(got) >= 0)
    one = acsr.acsr_degree_relabel(torch.tensor([0, 1], dtype=torch.int32, device=cuda),
                                   torch.tensor([0], dtype=torch.int32, device=cuda),
                                   torch.tensor([1], dtype=torch.int32, device=cuda))
    assert one[3].cpu().tolist() == [0] and one[1].cpu().tolist() == [0] and one[0].cpu().tolist() == [0, 1]
    n = 1000
    rp2, c2, od2, perm = acsr.acsr_degree_relabel(torch.zeros(n + 1, dtype=torch.int32, device=cuda),
                                                  torch.zeros(0, dtype=torch.int32, device=cuda),
                                                  torch.zeros(n, dtype=torch.int32, device=cuda))
    assert torch.equal(perm.cpu(), torch.arange(n, dtype=torch.int32)) and int(rp2[-1]) == 0
    e = acsr.acsr_degree_relabel(torch.zeros(1, dtype=torch.int32, device=cuda), None,
                                 torch.zeros(0, dtype=torch.int32, device=cuda))
    assert e[0].cpu().tolist() == [0]
    with pytest.raises(acsr.ACSRError, match="INVALID_VALUE"):
        acsr.AcsrComm(2, 5, acsr.AcsrComm.unique_id())
    with pytest.raises(ValueError):
        acsr.AcsrComm(1, 0, b"short")


def test_grow_layout_matches_reading_r4(acsr, cuda):
    """acsr_grow_layout = reading R4 written out on the host: cap' = max(cap + max(m, ceil(cap/f)),
    len + max(m, ceil(len/f))), begin' = exclusive prefix, total = sum (bitwise, integers)."""
    n, rb, re, cap, col, _, od, rp, ci = _slack_graph(13)
    for m_, f in ((8, 2), (4, 4), (1, 1)):
        nb, nc, tot = acsr.acsr_grow_layout(rb.to(cuda), re.to(cuda), cap.to(cuda), m_, f)
        ln = (re - rb).numpy().astype(np.int64)
        c = cap.numpy().astype(np.int64)
        ref = np.maximum(c + np.maximum(m_, -(-c // f)), ln + np.maximum(m_, -(-ln // f)))
        pre = np.concatenate([[0], np.cumsum(ref)[:-1]])
        assert np.array_equal(nc.cpu().numpy(), ref) and np.array_equal(nb.cpu().numpy(), pre)
        assert tot == int(ref.sum())


@pytest.mark.parametrize("P", [2, 3])
def test_exchange_layout_matches_definition(acsr, cuda, P):
    """acsr_exchange_layout + acsr_permute_graph = the compact layout's definition written out
    on the host: pos[v] = owner(v) * Lx + rank among the owner's non-dangling
    vertices (P * Lx for dangling v), local order = non-dangling rows first, stable, and the
    permuted local CSR with renumbered columns -- bitwise, for every rank."""
    from paper_conf_sc_ashariseps14_b200 import dist as pdist
    rp, ci, od, n = _inlink(14, cuda)
    splits = pdist.partition_rows(np.diff(rp.numpy()), P)
    nd = (od.numpy() > 0)
    counts = [int(nd[splits[k]:splits[k + 1]].sum()) for k in range(P)]
    Lx = max(1, max(counts))
    owner = np.searchsorted(splits[1:-1], np.arange(n), side="right")
    ex = np.cumsum(nd) - nd
    pos_ref = np.where(nd, owner * Lx + ex - ex[splits[owner]], P * Lx)
    sp = torch.as_tensor(splits, dtype=torch.int64, device=cuda)
    for rank in range(P):
        pos, order, cnt, lx = acsr.acsr_exchange_layout(torch.from_numpy(nd.astype(np.uint8)).to(cuda), sp, rank)
        assert cnt == counts and lx == Lx
        assert np.array_equal(pos.cpu().numpy(), pos_ref)
        lo, hi = int(splits[rank]), int(splits[rank + 1])
        ndl = nd[lo:hi]
        order_ref = np.concatenate([np.flatnonzero(ndl), np.flatnonzero(~ndl)])
        assert np.array_equal(order.cpu().numpy(), order_ref)
        rpl = (rp[lo:hi + 1] - rp[lo]).to(torch.int32)
        cil = ci[int(rp[lo]):int(rp[hi])]
        rp2, c2 = acsr.acsr_permute_graph(rpl.to(cuda), cil.to(cuda), order, col_map=pos)
        ln = np.diff(rpl.numpy())[order_ref]
        assert np.array_equal(rp2.cpu().numpy(), np.concatenate([[0], np.cumsum(ln)]))
        ref = np.concatenate([pos_ref[cil.numpy()[rpl[r]:rpl[r + 1]]] for r in order_ref]) if ln.sum() else np.zeros(0)
        assert np.array_equal(c2.cpu().numpy(), ref)


def test_single_rank_acsr_comm_step_equals_pagerank(acsr, cuda):
    """acsr_pagerank_step with a one-rank acsr_comm (exchange + global Delta^2 in the
    library) gives the single-GPU loop's iterate, iteration count and Delta^2 bitwise."""
    from paper_conf_sc_ashariseps14_b200 import dist as pdist
    rp, ci, od, n = _inlink(15, cuda)
    m = acsr.ACSRMatrix(rp.to(cuda), ci.to(cuda))
    x1, it1, d21 = acsr.pagerank(m, od.to(cuda), eps=1e-6)
    pr = pdist.DistPageRank(rp.to(cuda), ci.to(cuda), od.to(cuda), np.array([0, n]), n, exchange="acsr")
    assert pr.comm.query() == (1, 0)
    x2, it2, d22 = pr.run(eps=1e-6)
    assert it1 == it2 and torch.equal(x1, x2) and d21 == d22
    pr.comm.close()


@pytest.mark.parametrize("dtype", ["float64", "float32"])
def test_dist_spmv_row_split_bitwise(acsr, cuda, dtype):
    """N4 (P:345 row split): one SpMV row-split over three ranks sharing the GPU equals the
    one-GPU acsr_spmv bit for bit (local col/val keep their global 16-byte phase), and the
    oracle bar."""
    import socket
    import sys
    import torch.multiprocessing as mp
    sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
    import _dist_gpu_worker
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_dist_gpu_worker.spmv_worker, args=(r, 3, port, 16, dtype, q)) for r in range(3)]
    for p in procs:
        p.start()
    y_split = q.get(timeout=300)
    for p in procs:
        p.join(60)
        assert p.exitcode == 0
    dt = getattr(torch, dtype)
    rp, ci = synth.rmat_csr(16, device=cuda)
    val = synth.values(ci.numel(), 1014, dt, cuda)
    x = synth.vector(rp.numel() - 1, 2014, dt, cuda)
    y1 = acsr.ACSRMatrix(rp, ci, val).spmv(x).cpu().numpy()
    assert np.array_equal(y_split, y1)
    y_ref, den = oracle.spmv(rp.cpu().numpy(), ci.cpu().numpy(), val.cpu().numpy(), x.cpu().numpy())
    check_spmv(y_split, y_ref, den, dt)


@pytest.mark.parametrize("compact", [True, False])
def test_peer_exchange_two_ranks_one_gpu(cuda, compact):
    # N1: the exchange fused into the step over peer memory (two processes sharing the GPU,
    # CUDA IPC mappings, in-kernel P2P stores + release/acquire flags, exact Delta^2
    # partials).  Same partition and layout as the collective all-gather path -> the same
    # bits (iterate, iteration count, Delta^2); every rank's replicated xs identical
    # (checked in the worker); and the oracle bar.
    full_p, it_p, d2_p = _two_ranks(14, exchange="peer", compact=compact)
    full_c, it_c, d2_c = _two_ranks(14, exchange="torch", compact=compact)
    assert it_p == it_c and np.array_equal(full_p, full_c)
    # Delta^2: the collective path all-reduces two rounded doubles, the peer path adds the
    # exact fixed-point partials and rounds once -> equal up to that one rounding
    assert abs(d2_p - d2_c) <= 4e-16 * d2_c
    full_8, it_8, d2_8 = _two_ranks(14, exchange="peer", compact=compact, check_every=8)
    assert it_8 == it_p and d2_8 == d2_p and np.array_equal(full_8, full_p)
    rp, ci, od, n = _inlink(14, cuda)
    x_ref, it_ref, _ = oracle.pagerank(rp.numpy(), ci.numpy(), od.numpy(), eps=1e-6)
    assert abs(it_p - it_ref) <= 1
    if it_p != it_ref:
        x_ref, _, _ = oracle.pagerank(rp.numpy(), ci.numpy(), od.numpy(), eps=0.0, max_iter=it_p)
    assert np.all(np.abs(full_p - x_ref) <= 1e-11 * x_ref + 1e-18)


def test_peer_exchange_three_ranks_one_gpu(cuda):
    # three ranks: every fused step stores its slice into two remote regions (the
    # out-of-line remote loop with the self-skip); same bits as the collective path
    full_p, it_p, _ = _two_ranks(13, world=3, exchange="peer", compact=True, check_every=4)
    full_c, it_c, _ = _two_ranks(13, world=3, exchange="torch", compact=True)
    assert it_p == it_c and np.array_equal(full_p, full_c)
    rp, ci, od, n = _inlink(13, cuda)
    x_ref, it_ref, _ = oracle.pagerank(rp.numpy(), ci.numpy(), od.numpy(), eps=1e-6)
    assert abs(it_p - it_ref) <= 1
    if it_p != it_ref:
        x_ref, _, _ = oracle.pagerank(rp.numpy(), ci.numpy(), od.numpy(), eps=0.0, max_iter=it_p)
    assert np.all(np.abs(full_p - x_ref) <= 1e-11 * x_ref + 1e-18)


def test_peer_exchange_single_rank_equals_pagerank(acsr, cuda):
    # one rank: the peer path (push to itself, flags, Delta^2 via the partial) gives the
    # single-GPU pagerank() bits, and a second run on the same acsr_peer (push count
    # continues, buffer parity flips) gives them again
    from paper_conf_sc_ashariseps14_b200 import dist as pdist
    rp, ci, od, n = _inlink(15, cuda)
    m = acsr.ACSRMatrix(rp.to(cuda), ci.to(cuda))
    x1, it1, d1 = acsr.pagerank(m, od.to(cuda), eps=1e-6, check_every=1)
    pr = pdist.DistPageRank(rp.to(cuda), ci.to(cuda), od.to(cuda), np.array([0, n]), n, exchange="peer")
    for _ in range(2):
        xp, itp, dp = pr.run(eps=1e-6)
        assert itp == it1 and dp == d1 and torch.equal(xp, x1)
    x3, it3, d3 = pr.run(eps=1e-6, check_every=8)
    assert it3 == it1 and d3 == d1 and torch.equal(x3, x1)
    pushes, err, _ = pr.peer.query()
    assert err == 0 and pushes == 3 * (it1 + 1)
    # the replicated xs is the scaled final iterate
    xs = pr.peer.read_xs()
    ref = acsr.acsr_pagerank_scale(x1, od.to(cuda))
    assert torch.equal(xs, ref)
    pr.peer.close()


def test_peer_wait_times_out_instead_of_hanging(cuda):
    """A rank that stops issuing pushes: the other rank's flag wait gives up after the
    bound (ACSR_PEER_TIMEOUT_MS = 300 here), sets the error word and the GPU stays usable."""
    import socket
    import sys
    import torch.multiprocessing as mp
    sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
    import _dist_gpu_worker
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_dist_gpu_worker.peer_timeout_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    pushes, err, waited = q.get(timeout=120)
    for p in procs:
        p.join(60)
        assert p.exitcode == 0
    assert err == 1 and pushes == 2 and waited < 30.0


def test_peer_argument_errors(acsr, cuda):
    with pytest.raises(acsr.ACSRError):
        acsr.AcsrPeer(9, 0, 10, 0, 5)  # more ranks than ACSR_PEER_MAX
    with pytest.raises(acsr.ACSRError):
        acsr.AcsrPeer(2, 0, 10, 8, 5)  # slice outside xs
    p = acsr.AcsrPeer(1, 0, 10, 0, 10)
    x = torch.ones(10, dtype=torch.float64, device=cuda)
    od = torch.ones(10, dtype=torch.int32, device=cuda)
    with pytest.raises(acsr.ACSRError):
        p.push(x, od)  # not opened
    p.open([p.handle_bytes()])
    with pytest.raises(acsr.ACSRError):
        p.push(x[:5], od[:5])  # fewer local rows than the slice
    p.push(x, od)
    assert torch.equal(p.read_xs(), x)
    p.close()


def test_device_side_convergence_identical(acsr, cuda):
    # enqueueing 8 steps between host checks (ctrl no-op steps after convergence) gives the
    # same iterate, iteration count and Delta^2 as a host test after every step
    rp, ci, od, n = _inlink(15, cuda)
    m = acsr.ACSRMatrix(rp.to(cuda), ci.to(cuda))
    x1, it1, d1 = acsr.pagerank(m, od.to(cuda), eps=1e-6, check_every=1)
    x8, it8, d8 = acsr.pagerank(m, od.to(cuda), eps=1e-6, check_every=8)
    assert it1 == it8 and d1 == d8 and torch.equal(x1, x8)
    r1, j1, _ = acsr.rwr(m, od.to(cuda), 3, check_every=1)
    r8, j8, _ = acsr.rwr(m, od.to(cuda), 3, check_every=8)
    assert j1 == j8 and torch.equal(r1, r8)
    # blocks of 8 steps replayed from one CUDA graph (PDL edges inside) -- same bits
    xg, itg, dg = acsr.pagerank(m, od.to(cuda), eps=1e-6, check_every=8, graph=True)
    xe, ite, de = acsr.pagerank(m, od.to(cuda), eps=1e-6, check_every=8, graph=False)
    assert itg == ite == it1 and dg == de and torch.equal(xg, xe) and torch.equal(xg, x1)
    # a tight eps forces several graph replays (and a ragged eager tail via max_iter)
    xg, itg, _ = acsr.pagerank(m, od.to(cuda), eps=1e-13, max_iter=43, graph=True)
    xe, ite, _ = acsr.pagerank(m, od.to(cuda), eps=1e-13, max_iter=43, graph=False)
    assert itg == ite and torch.equal(xg, xe)


def test_graph_captured_bin_spmv(acsr, cuda):
    """acsr_bin + acsr_spmv captured into a CUDA graph (the calls are stream-ordered and
    allocation-free, PDL edges included) and replayed: same bits as eager calls."""
    rp, ci = synth.rmat_csr(15)
    n = rp.numel() - 1
    val = synth.values(ci.numel(), 5).to(cuda)
    x = synth.vector(n, 6).to(cuda)
    m = acsr.ACSRMatrix(rp.to(cuda), ci.to(cuda), val)
    y_e = m.spmv(x).clone()
    y = torch.empty_like(y_e)
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        m.rebin()
        m.spmv(x, y)
    y.zero_()
    g.replay()
    torch.cuda.synchronize()
    assert torch.equal(y, y_e)
    x.mul_(-2.0)  # inputs updated in place -> the replay sees them
    g.replay()
    torch.cuda.synchronize()
    assert torch.equal(y, m.spmv(x))
