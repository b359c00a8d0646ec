"""Run a few fused peer-exchange PageRank steps with P processes sharing one GPU (CUDA IPC),
for timing / ncu store-transaction counts of acsr_pagerank_step_peer.
  python tools/peer_steps.py [P] [scale] [steps]
Rank 0 prints one JSON line: ms per step (CUDA events over `steps` steps, after 2 warm-up
steps), the variant (ACSR_LIB_VARIANT) and the exchanged slice."""
import json
import os
import socket
import sys

import numpy as np
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def worker(rank, world, port, scale, steps):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import synth
    from paper_conf_sc_ashariseps14_b200 import dist as pdist
    dev = torch.device("cuda:0")
    torch.cuda.set_device(dev)
    rp, ci = synth.rmat_csr(scale, device=dev, transpose=True)
    n = rp.numel() - 1
    od = torch.bincount(ci.long(), minlength=n).to(torch.int32)
    splits = pdist.partition_rows(np.diff(rp.cpu().numpy()), world)
    lo, hi = int(splits[rank]), int(splits[rank + 1])
    rpl = (rp[lo:hi + 1] - rp[lo]).contiguous()
    cil = ci[int(rp[lo]):int(rp[hi])].clone()
    pr = pdist.DistPageRank(rpl, cil, od[lo:hi].clone(), splits, n, exchange="peer")
    pr.run(eps=0.0, max_iter=2, check_every=2)
    torch.cuda.synchronize()
    dist.barrier()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    x, it, d2 = pr.run(eps=0.0, max_iter=steps, check_every=steps)
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / steps
    t = torch.tensor([ms], dtype=torch.float64)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    if rank == 0:
        print(json.dumps({"P": world, "scale": scale, "steps": steps, "ms_per_step_max_rank": round(float(t), 4),
                          "variant": os.environ.get("ACSR_LIB_VARIANT", ""), "slice": pr.Lx, "n": n,
                          "delta2": d2}), flush=True)
    pr.peer.close()
    dist.destroy_process_group()


if __name__ == "__main__":
    P = int(sys.argv[1]) if len(sys.argv) > 1 else 2
    scale = int(sys.argv[2]) if len(sys.argv) > 2 else 20
    steps = int(sys.argv[3]) if len(sys.argv) > 3 else 10
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    mp.start_processes(worker, args=(P, port, scale, steps), nprocs=P, start_method="spawn")
