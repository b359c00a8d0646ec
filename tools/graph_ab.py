"""Bin and SpMV device times with sub-tick resolution: K iterations of
(L2 flush; acsr_bin) and (L2 flush; acsr_spmv) captured in CUDA graphs and replayed
between two events, minus a graph of K flushes alone.  The box's event clock ticks
in ~2 us steps, so single-launch event pairs (tools/spmv_ab.py) are quantised; this
divides the tick by K.  Prints one JSON line."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import synth
import paper_conf_sc_ashariseps14_b200 as acsr


def main():
    wl = sys.argv[1] if len(sys.argv) > 1 else "rmat20"
    K = int(sys.argv[2]) if len(sys.argv) > 2 else 20
    dev = torch.device("cuda:0")
    dtype = torch.float32 if wl.endswith("_f32") else torch.float64
    if wl.startswith("rmat"):
        rp, ci = synth.rmat_csr(int(wl[4:6]), device=dev)
    elif wl == "webgoogle":
        rp, ci = synth.powerlaw_csr(seed=3, device=dev, **synth.WEB_GOOGLE)
    else:
        rp, ci = synth.powerlaw_csr(seed=4, device=dev, **synth.LIVEJOURNAL)
    n, nnz = rp.numel() - 1, ci.numel()
    val = synth.values(nnz, 1014, dtype, dev)
    x = synth.vector(n, 2014, dtype, dev)
    y = torch.empty(n, dtype=dtype, device=dev)
    m = acsr.ACSRMatrix(rp, ci, val)
    fmode = os.environ.get("GRAPH_AB_FLUSH", "write")  # write | write+read | none
    fw = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    fr = torch.zeros(64 << 20, dtype=torch.int32, device=dev)
    facc = torch.zeros((), dtype=torch.int64, device=dev)

    class _Flush:
        @staticmethod
        def zero_():
            if fmode != "none":
                fw.zero_()
            if fmode == "write+read":
                torch.sum(fr, dim=0, dtype=torch.int64, out=facc)
    flush = _Flush()
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):  # warm-up outside capture
        m.rebin(stream=s)
        m.spmv(x, y, stream=s)
    s.synchronize()

    def capture(body):
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            for _ in range(K):
                flush.zero_()
                body()
        return g

    cs = torch.cuda.current_stream
    graphs = {
        "flush": capture(lambda: None),
        "bin": capture(lambda: m.rebin(stream=cs())),
        "spmv": capture(lambda: m.spmv(x, y, stream=cs())),
        "step": capture(lambda: (m.rebin(stream=cs()), m.spmv(x, y, stream=cs()))),
    }
    res = {}
    for rep in range(7):
        for k, g in graphs.items():
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            g.replay()
            e1.record()
            torch.cuda.synchronize()
            if rep >= 2:
                res.setdefault(k, []).append(e0.elapsed_time(e1) * 1e3 / K)
    med = {k: sorted(v)[len(v) // 2] for k, v in res.items()}
    out = {"wl": wl, "n": n, "nnz": nnz, "K": K,
           "variant": os.environ.get("ACSR_LIB_VARIANT", ""),
           "env": {k: v for k, v in os.environ.items() if k.startswith("ACSR_") and k != "ACSR_LIB_VARIANT"},
           "flush_mode": fmode, "flush_us": round(med["flush"], 2)}
    for k in ("bin", "spmv", "step"):
        out["t_%s_us" % k] = round(med[k] - med["flush"], 2)
    print(json.dumps(out))


main()
