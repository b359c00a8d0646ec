"""Does column hotness cost gather rate?  x[idx] (torch.index_select, 8-byte elements, x = 8 MB
L2-resident after a warm-up) with idx = (a) the C2 matrix's own columns (power-law, R-MAT
in-degrees), (b) uniform random columns of the same count, (c) the C2 columns spread over R
replicas of x by position (hot lines served by R different addresses / L2 slices),
(d) the C2 columns sorted (maximal line reuse).  Prints one JSON line of median us."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import synth

dev = torch.device("cuda:0")
rp, ci = synth.rmat_csr(20, device=dev)
n, nnz = rp.numel() - 1, ci.numel()
col = ci.long()
g = torch.Generator(device=dev).manual_seed(7)
uni = torch.randint(0, n, (nnz,), device=dev, generator=g)
x = torch.randn(n, dtype=torch.float64, device=dev)
out = torch.empty(nnz, dtype=torch.float64, device=dev)
cases = {"c2_cols": (x, col), "uniform": (x, uni), "c2_sorted": (x, torch.sort(col).values)}
for R in (2, 4, 8):
    xr = x.repeat(R)
    rep = (torch.arange(nnz, device=dev) // 4096) % R
    cases["c2_cols_rep%d" % R] = (xr, col + rep * n)
    cases["uniform_rep%d" % R] = (xr, uni + rep * n)
res = {}
for name, (xx, idx) in cases.items():
    ts = []
    for i in range(25):
        torch.index_select(xx, 0, idx, out=out)  # x warm in L2
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        torch.index_select(xx, 0, idx, out=out)
        e1.record()
        torch.cuda.synchronize()
        if i >= 5:
            ts.append(e0.elapsed_time(e1) * 1e3)
    ts.sort()
    res[name] = round(ts[len(ts) // 2], 2)
print(json.dumps({"nnz": nnz, "n": n, "median_us": res}))
