"""Time acsr_bin and acsr_spmv separately on one workload (CUDA events, L2 flushed
between reps).  Used for A/B runs of the env knobs; prints one JSON line."""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import synth
import paper_conf_sc_ashariseps14_b200 as acsr

def main():
    wl = sys.argv[1] if len(sys.argv) > 1 else "rmat20"
    reps = int(sys.argv[2]) if len(sys.argv) > 2 else 20
    dev = torch.device("cuda:0")
    dtype = torch.float32 if wl.endswith("_f32") else torch.float64
    if wl.startswith("rmat"):
        sc = int(wl[4:6])
        rp, ci = synth.rmat_csr(sc, device=dev)
    elif wl == "webgoogle":
        rp, ci = synth.powerlaw_csr(seed=3, device=dev, **synth.WEB_GOOGLE)
    else:
        rp, ci = synth.powerlaw_csr(seed=4, device=dev, **synth.LIVEJOURNAL)
    n, nnz = rp.numel() - 1, ci.numel()
    val = synth.values(nnz, 1014, dtype, dev); x = synth.vector(n, 2014, dtype, dev)
    colperm = os.environ.get("COLPERM") == "1"
    t_relabel = None
    if colperm:  # experiment: columns renumbered by decreasing frequency (x gathered through q)
        torch.cuda.synchronize(); t0 = time.perf_counter()
        cnt = torch.bincount(ci.long(), minlength=n)
        q = torch.sort(cnt, descending=True, stable=True).indices
        p = torch.empty_like(q); p[q] = torch.arange(n, device=dev)
        ci = p[ci.long()].to(torch.int32)
        torch.cuda.synchronize(); t_relabel = time.perf_counter() - t0
    m = acsr.ACSRMatrix(rp, ci, val, short_rows=os.environ.get("SHORT_ROWS", "window"))
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    tb, ts = [], []
    for i in range(reps + 3):
        flush.zero_()
        e = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
        e[0].record(); m.rebin(); e[1].record()
        y = m.spmv(x[q] if colperm else x)
        e[2].record()
        torch.cuda.synchronize()
        if i >= 3:
            tb.append(e[0].elapsed_time(e[1])); ts.append(e[1].elapsed_time(e[2]))
    sv = 8 if dtype == torch.float64 else 4
    n_c = int((torch.bincount(ci.long(), minlength=n) > 0).sum())
    alg = (sv + 4) * nnz + 8 * n + 4 + sv * n_c + sv * n
    print(json.dumps({"wl": wl, "env": {k: v for k, v in os.environ.items() if k.startswith("ACSR_") or k == "SHORT_ROWS"},
                      "t_bin_us": round(1e3 * float(np.median(tb)), 2), "t_spmv_us": round(1e3 * float(np.median(ts)), 2),
                      "t_spmv_min_us": round(1e3 * float(np.min(ts)), 2),
                      "t_spmv_mean_us": round(1e3 * float(np.mean(ts)), 2),
                      "spmv_GBs": round(alg / (np.median(ts) * 1e-3) / 1e9, 1), "nnz": nnz, "n": n,
                      "colperm": colperm, "t_relabel_s": t_relabel}))

main()
