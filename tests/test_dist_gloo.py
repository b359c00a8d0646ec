"""Multi-process (world_size 2, gloo, CPU) test of the row-partitioned PageRank host logic:
partition, column renumbering into the padded all-gather layout, in-place all-gather of the
xs slices, all-reduce of Delta^2 and the Alg. 5 loop.  The per-rank local step is injected
(the CPU oracle on the local rows) -- the CUDA step itself is covered by tests -m gpu."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import synth
from paper_conf_sc_ashariseps14_b200 import dist as acsr_dist


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, scale, out, compact=True):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    rp, ci = synth.rmat_csr(scale, transpose=True)
    n = rp.numel() - 1
    od = torch.bincount(ci.long(), minlength=n).to(torch.int32)
    splits = acsr_dist.partition_rows(np.diff(rp.numpy()), world)
    lo, hi = int(splits[rank]), int(splits[rank + 1])
    rpl = (rp[lo:hi + 1] - rp[lo]).contiguous()
    cil = ci[int(rp[lo]):int(rp[hi])].contiguous()
    odl = od[lo:hi].contiguous()

    def step(xs, x, x_new, xs_next_slice, delta2):
        # the local CSR / outdeg as the object holds them (rows possibly reordered,
        # columns renumbered into the exchange layout)
        xn, d2 = oracle.pagerank_step(pr.row_ptr.numpy(), pr.col.numpy(), np.ones(xs.numel(), np.int32),
                                      xs.numpy(), pr.teleport, pr.damping)
        # oracle with outdeg = 1 gathers xs itself: y_v = sum xs_u  (xs already scaled)
        od_l = pr.outdeg
        x_new.copy_(torch.from_numpy(xn))
        xs_next_slice.copy_(torch.where(od_l > 0, x_new / od_l.clamp(min=1).double(), torch.zeros_like(x_new)))
        delta2.fill_(float(((x_new - x) ** 2).sum()))

    def scale(x, outdeg, outv):
        outv.copy_(torch.where(outdeg > 0, x / outdeg.clamp(min=1).double(), torch.zeros_like(x)))

    pr = acsr_dist.DistPageRank(rpl, cil, odl, splits, n, step_fn=step, scale_fn=scale,
                                device=torch.device("cpu"), compact=compact)
    x, it, d2 = pr.run(eps=1e-8)
    # exchange volume: the compact layout carries only the non-dangling vertices
    nb = torch.tensor([pr.exchange_bytes_per_rank(), pr.Lx, pr.L], dtype=torch.int64)
    xs_all = [torch.zeros(pr.L, dtype=torch.float64) for _ in range(world)]
    xp = torch.zeros(pr.L, dtype=torch.float64)
    xp[: x.numel()] = x
    dist.all_gather(xs_all, xp)
    if rank == 0:
        full = torch.cat([xs_all[k][: int(splits[k + 1] - splits[k])] for k in range(world)])
        out.put((full.numpy(), it, d2, splits, nb.tolist()))
    dist.destroy_process_group()


@pytest.mark.parametrize("compact", [True, False])
@pytest.mark.parametrize("world", [2])
def test_partitioned_pagerank_matches_single(world, compact):
    scale = 11
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, scale, q, compact)) for r in range(world)]
    for p in procs:
        p.start()
    full, it, d2, splits, (xbytes, Lx, L) = q.get(timeout=240)
    for p in procs:
        p.join(60)
        assert p.exitcode == 0
    rp, ci = synth.rmat_csr(scale, transpose=True)
    n = rp.numel() - 1
    od = torch.bincount(ci.long(), minlength=n).to(torch.int32).numpy()
    x_ref, it_ref, _ = oracle.pagerank(rp.numpy(), ci.numpy(), od, eps=1e-8)
    assert abs(it - it_ref) <= 1
    assert np.allclose(full, x_ref, rtol=1e-11, atol=1e-18)
    assert splits[0] == 0 and splits[-1] == n and np.all(np.diff(splits) > 0)
    if compact:
        # slot per non-dangling vertex only: the largest per-rank count of outdeg > 0
        nnd = max(int((od[splits[k]:splits[k + 1]] > 0).sum()) for k in range(world))
        assert Lx == nnd < L
        assert xbytes == (world - 1) * nnd * 8
    else:
        assert Lx == L


def test_partition_matches_oracle_rule():
    rp, _ = synth.rmat_csr(12)
    for P in (1, 2, 4, 8):
        s = acsr_dist.partition_rows(np.diff(rp.numpy()), P)
        assert np.array_equal(s, oracle.partition(rp.numpy(), P, 4, 36))


def test_renumber_roundtrip():
    splits = np.array([0, 5, 12, 20])
    L = acsr_dist.padded_layout(splits)
    col = torch.arange(20, dtype=torch.int32)
    c2 = acsr_dist.renumber_columns(col, splits, L)
    owner = c2 // L
    assert torch.equal(owner, torch.tensor([0] * 5 + [1] * 7 + [2] * 8))
    back = torch.tensor(splits[:-1])[owner.long()] + c2 % L
    assert torch.equal(back.to(torch.int32), col)


def test_permute_rows_roundtrip():
    rp, ci = synth.rmat_csr(9)
    n = rp.numel() - 1
    perm = torch.randperm(n, generator=torch.Generator().manual_seed(3))
    rp2, ci2 = acsr_dist.permute_rows(rp, ci, perm)
    for i in range(0, n, 7):
        r = int(perm[i])
        assert torch.equal(ci2[int(rp2[i]):int(rp2[i + 1])], ci[int(rp[r]):int(rp[r + 1])])
    assert int(rp2[-1]) == ci.numel()


def _spmv_worker(rank, world, port, out):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    rp, ci = synth.rmat_csr(12)
    n = rp.numel() - 1
    val = synth.values(ci.numel(), 7)
    x = synth.vector(n, 8)
    splits = acsr_dist.partition_rows(np.diff(rp.numpy()), world, b_nnz=12, b_row=16)

    def local(row_ptr, col, v, xx):
        y, _ = oracle.spmv(row_ptr.numpy(), col.numpy(), v.numpy(), xx.numpy())
        return torch.from_numpy(y)

    sp = acsr_dist.DistSpMV(rp, ci, val, splits, spmv_fn=local)
    # the local arrays keep the global 16-byte phase of their first element
    k0 = int(rp[int(splits[rank])])
    assert sp.col.data_ptr() % 16 == (ci.data_ptr() + 4 * k0) % 16
    assert sp.val.data_ptr() % 16 == (val.data_ptr() + 8 * k0) % 16
    y = sp.gather(sp.spmv(x))
    if rank == 0:
        out.put((y.numpy(), splits))
    dist.destroy_process_group()


def test_dist_spmv_row_split_gloo_ws2():
    """N4: one SpMV split by rows over two ranks (gloo, CPU; the oracle as the local SpMV):
    nnz-balanced split points equal the oracle's O8 partition, the gathered y equals the
    oracle on the whole matrix bit for bit."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_spmv_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    y, splits = q.get(timeout=120)
    for p in ps:
        p.join(60)
        assert p.exitcode == 0
    rp, ci = synth.rmat_csr(12)
    val = synth.values(ci.numel(), 7)
    x = synth.vector(rp.numel() - 1, 8)
    y_ref, _ = oracle.spmv(rp.numpy(), ci.numpy(), val.numpy(), x.numpy())
    assert np.array_equal(y, y_ref)
    assert np.array_equal(splits, oracle.partition(rp.numpy(), 2, 12, 16))
