"""Per-mapping SpMV efficiency: matrices whose rows all have length L (one bin), random
uniform columns over 2^20 columns (x L2-resident), ~8M nnz.  Prints one JSON line per L."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import synth
import paper_conf_sc_ashariseps14_b200 as acsr

dev = torch.device("cuda:0")
n_cols = 1 << 20
for L in [1, 2, 3, 4, 6, 8, 12, 16, 24, 32, 48, 64, 96, 128, 192, 256, 384, 512, 768, 1024, 1536, 4096, 16384]:
    n = max(1, (8 << 20) // L)
    rp = (torch.arange(n + 1, device=dev, dtype=torch.int64) * L).to(torch.int32)
    nnz = n * L
    ci = (synth._srl(synth.hash64(7, 3, torch.arange(nnz, device=dev)), 1) % n_cols).to(torch.int32)
    val = synth.values(nnz, 5, device=dev)
    x = synth.vector(n_cols, 6, device=dev)
    m = acsr.ACSRMatrix(rp, ci, val, n_cols=n_cols)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    ts = []
    for i in range(13):
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); m.spmv(x); e1.record(); torch.cuda.synchronize()
        if i >= 3: ts.append(e0.elapsed_time(e1))
    t = float(np.median(ts)) * 1e-3
    alg = 12 * nnz + 8 * n + 4 + 8 * n_cols + 8 * n
    print(json.dumps({"L": L, "n": n, "nnz": nnz, "t_us": round(t * 1e6, 2), "GBs": round(alg / t / 1e9, 1),
                      "Ggather_s": round(nnz / t / 1e9, 2), "env": {k: v for k, v in os.environ.items() if k.startswith("ACSR_")}}), flush=True)
