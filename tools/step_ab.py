"""C2 / web-Google-like / LiveJournal-like step (acsr_bin + acsr_spmv back to back, L2 flushed,
events at the step's ends only) for the loaded build (ACSR_LIB_VARIANT)."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import synth
import paper_conf_sc_ashariseps14_b200 as acsr
wl = sys.argv[1] if len(sys.argv) > 1 else "rmat20"
dev = torch.device("cuda:0")
if wl == "rmat20":
    rp, ci = synth.rmat_csr(20, seed=20, device=dev)
elif wl == "webgoogle":
    rp, ci = synth.powerlaw_csr(seed=3, device=dev, **synth.WEB_GOOGLE)
else:
    rp, ci = synth.powerlaw_csr(seed=4, device=dev, **synth.LIVEJOURNAL)
n, nnz = rp.numel() - 1, ci.numel()
val = synth.values(nnz, 1014, torch.float64, dev); x = synth.vector(n, 2014, torch.float64, dev)
br = torch.empty(n, dtype=torch.int32, device=dev); bo = torch.empty(33, dtype=torch.int32, device=dev)
ws = torch.empty(acsr.acsr_bin_workspace_bytes(n, n, nnz), dtype=torch.uint8, device=dev)
y = torch.empty(n, dtype=torch.float64, device=dev)
flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
ts = []
for k in range(45):
    flush.zero_()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    acsr.acsr_bin(rp, None, nnz, br, bo, ws, col_idx=ci, n_cols=n)
    acsr.acsr_spmv(rp, ci, val, x, br, bo, ws, None, y)
    e1.record()
    torch.cuda.synchronize()
    if k >= 5:
        ts.append(e0.elapsed_time(e1))
print(json.dumps({"variant": os.environ.get("ACSR_LIB_VARIANT", ""), "wl": wl, "step_us": round(1e3 * float(np.mean(ts)), 2),
                  "step_us_median": round(1e3 * float(np.median(ts)), 2)}))
