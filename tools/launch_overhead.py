"""GPU-side fixed cost per launch: K back-to-back launches captured in one CUDA graph
(so host/ctypes overhead is excluded), timed with CUDA events around the replay.
Compares the persistent SpMV kernel on tiny matrices with a minimal kernel.  Prints
one JSON line."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sc_ashariseps14_b200 as acsr

dev = torch.device("cuda:0")
K = 100


def graph_time(fn):
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        for _ in range(3):
            fn()
    torch.cuda.current_stream().wait_stream(s)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        for _ in range(K):
            fn()
    g.replay()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(5):
        g.replay()
    e1.record()
    torch.cuda.synchronize()
    return round(e0.elapsed_time(e1) * 1e3 / (5 * K), 2)


out = {}
for n in (1, 65536, 1 << 20):
    rp = torch.arange(n + 1, dtype=torch.int32, device=dev)
    ci = torch.arange(n, dtype=torch.int32, device=dev)
    m = acsr.ACSRMatrix(rp, ci, torch.ones(n, dtype=torch.float64, device=dev))
    x = torch.ones(n, dtype=torch.float64, device=dev)
    y = torch.empty_like(x)
    out[f"spmv_n{n}_us"] = graph_time(lambda: m.spmv(x, y))
    out[f"bin_n{n}_us"] = graph_time(lambda: m.rebin())
x1 = torch.ones(1, dtype=torch.float64, device=dev)
od = torch.ones(1, dtype=torch.int32, device=dev)
xs = torch.empty_like(x1)
out["tiny_kernel_us"] = graph_time(lambda: acsr.acsr_pagerank_scale(x1, od, xs))
out["pdl"] = os.environ.get("ACSR_PDL", "1")
print(json.dumps(out))
