"""Does an event between acsr_bin and acsr_spmv cost the step its PDL overlap?  C2 step timed
(L2 flushed) with three events per step (bin | SpMV split) and with two (start, end)."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import synth
import paper_conf_sc_ashariseps14_b200 as acsr
dev = torch.device("cuda:0")
rp, ci = synth.rmat_csr(20, seed=20, device=dev)
n, nnz = rp.numel() - 1, ci.numel()
val = synth.values(nnz, 1014, torch.float64, dev); x = synth.vector(n, 2014, torch.float64, dev)
br = torch.empty(n, dtype=torch.int32, device=dev); bo = torch.empty(33, dtype=torch.int32, device=dev)
ws = torch.empty(acsr.acsr_bin_workspace_bytes(n, n, nnz), dtype=torch.uint8, device=dev)
y = torch.empty(n, dtype=torch.float64, device=dev)
flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
res = {}
for mode in ("three_events", "two_events", "three_events", "two_events"):
    ts = []
    for k in range(40):
        flush.zero_()
        e = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
        e[0].record()
        acsr.acsr_bin(rp, None, nnz, br, bo, ws, col_idx=ci, n_cols=n)
        if mode == "three_events":
            e[1].record()
        acsr.acsr_spmv(rp, ci, val, x, br, bo, ws, None, y)
        e[2].record()
        torch.cuda.synchronize()
        if k >= 5:
            ts.append(e[0].elapsed_time(e[2]))
    res.setdefault(mode, []).append(round(1e3 * float(np.mean(ts)), 2))
print(json.dumps(res))
