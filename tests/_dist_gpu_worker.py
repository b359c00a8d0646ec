"""Worker for tests/test_gpu_parity.py::test_dist_pagerank_two_ranks_one_gpu (spawned)."""
import os

import numpy as np
import torch
import torch.distributed as dist


def worker(rank, world, port, scale, q, exchange="torch", compact=True, check_every=1):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    if exchange == "acsr":
        # the library's NCCL communicator with every rank on the SAME GPU: NCCL refuses two
        # ranks on one device of one host, so each rank claims its own host id (the ranks
        # then talk over NCCL's socket transport on loopback).  Test-only: on a real node
        # every rank has its own GPU and NCCL uses NVLink / NVSwitch.
        os.environ.update(NCCL_HOSTID=f"acsr-test-host-{rank}", NCCL_SOCKET_IFNAME="lo", NCCL_IB_DISABLE="1",
                          NCCL_P2P_DISABLE="1", NCCL_SHM_DISABLE="1", NCCL_NVLS_ENABLE="0")
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import synth
    from paper_conf_sc_ashariseps14_b200 import dist as pdist
    dev = torch.device("cuda:0")
    rp, ci = synth.rmat_csr(scale, transpose=True)
    n = rp.numel() - 1
    od = torch.bincount(ci.long(), minlength=n).to(torch.int32)
    splits = pdist.partition_rows(np.diff(rp.numpy()), world)
    lo, hi = int(splits[rank]), int(splits[rank + 1])
    rpl = (rp[lo:hi + 1] - rp[lo]).to(dev)
    cil = ci[int(rp[lo]):int(rp[hi])].to(dev)
    pr = pdist.DistPageRank(rpl, cil, od[lo:hi].to(dev), splits, n, exchange=exchange, compact=compact)
    if exchange == "peer":
        x, it, d2 = pr.run(eps=1e-6, check_every=check_every)
        # every rank's replicated xs after the last push is the same vector
        xs = pr.peer.read_xs()
        allx = [torch.zeros_like(xs.cpu()) for _ in range(world)]
        dist.all_gather(allx, xs.cpu())
        assert all(torch.equal(allx[0], a) for a in allx), "replicated xs differ across ranks"
        pr.peer.close()
    else:
        x, it, d2 = pr.run(eps=1e-6, check_every=check_every)
        if exchange == "acsr":
            pr.comm.close()
    parts = [torch.zeros(pr.L, dtype=torch.float64) for _ in range(world)]
    xp = torch.zeros(pr.L, dtype=torch.float64)
    xp[: x.numel()] = x.cpu()
    dist.all_gather(parts, xp)
    if rank == 0:
        full = torch.cat([parts[k][: int(splits[k + 1] - splits[k])] for k in range(world)])
        q.put((full.numpy(), it, d2))
    dist.destroy_process_group()


def spmv_worker(rank, world, port, scale, dtype_name, q):
    """N4: C2-shaped matrix row-split over `world` ranks sharing the GPU (gloo for the
    y gather); rank 0 returns the gathered y."""
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import synth
    from paper_conf_sc_ashariseps14_b200 import dist as pdist
    dev = torch.device("cuda:0")
    dtype = getattr(torch, dtype_name)
    rp, ci = synth.rmat_csr(scale, device=dev)
    n = rp.numel() - 1
    val = synth.values(ci.numel(), 1014, dtype, dev)
    x = synth.vector(n, 2014, dtype, dev)
    splits = pdist.partition_rows((rp[1:] - rp[:-1]).cpu().numpy(), world, b_nnz=4 + val.element_size(), b_row=16,
                                  align=32)
    sp = pdist.DistSpMV(rp, ci, val, splits)
    y = sp.spmv(x)
    y2 = sp.spmv(x)  # a second call on the same plan: identical
    assert torch.equal(y, y2)
    yall = sp.gather(y.cpu())
    if rank == 0:
        q.put(yall.numpy())
    dist.destroy_process_group()


def peer_timeout_worker(rank, world, port, q):
    """Rank 1 maps the regions and then stops issuing pushes; rank 0's push and steps must
    time out (ACSR_PEER_TIMEOUT_MS), set the error word and return, not hang."""
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), ACSR_PEER_TIMEOUT_MS="300")
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import time
    import paper_conf_sc_ashariseps14_b200 as acsr
    dev = torch.device("cuda:0")
    n = 1000
    peer = acsr.AcsrPeer(world, rank, 2 * n, rank * n, n)
    hs = [None] * world
    dist.all_gather_object(hs, peer.handle_bytes())
    peer.open(hs)
    if rank == 0:
        x = torch.full((n,), 1.0 / n, dtype=torch.float64, device=dev)
        od = torch.ones(n, dtype=torch.int32, device=dev)
        peer.push(x, od)          # waits only for pushes >= 0: passes
        peer.push(x, od)          # needs rank 1's first push: times out
        t0 = time.perf_counter()
        torch.cuda.synchronize()
        pushes, err, _ = peer.query()
        q.put((pushes, err, time.perf_counter() - t0))
    dist.barrier()
    peer.close()
    dist.destroy_process_group()
