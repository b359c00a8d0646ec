"""Per-unit timeline of one spmv_kernel launch (needs the ACSR_TIMELINE=1 variant:
ACSR_LIB_VARIANT=tl, built by tools/build_variants.sh tl).  L2 flushed before the launch,
as in bench.py.  Prints one JSON line: per-CTA span, entry -> first unit, unit durations
by kind (early / late half of the launch), warp occupancy over time (busy warps per SM in
1 us buckets), and the tail (time from the first warp running out of units to the CTA's
last unit end)."""
import ctypes, json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import synth
import paper_conf_sc_ashariseps14_b200 as acsr

wl = sys.argv[1] if len(sys.argv) > 1 else "rmat20"
dev = torch.device("cuda:0")
if wl.startswith("rmat"):
    rp, ci = synth.rmat_csr(int(wl[4:6]), device=dev)
elif wl == "webgoogle":
    rp, ci = synth.powerlaw_csr(seed=3, device=dev, **synth.WEB_GOOGLE)
else:
    rp, ci = synth.powerlaw_csr(seed=4, device=dev, **synth.LIVEJOURNAL)
n = rp.numel() - 1
val = synth.values(ci.numel(), 1014, torch.float64, dev)
x = synth.vector(n, 2014, torch.float64, dev)
m = acsr.ACSRMatrix(rp, ci, val)
flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
f = acsr._lib.acsr_debug_timeline
f.argtypes = [ctypes.c_void_p]
TL = 1 << 16
buf = np.zeros(2 * TL + 3072, dtype=np.uint64)
m.spmv(x)
torch.cuda.synchronize()
f(buf.ctypes.data)
res = []
for rep in range(5):
    flush.zero_()
    m.rebin()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(); m.spmv(x); e1.record()
    torch.cuda.synchronize()
    f(buf.ctypes.data)
    t = buf[:2 * TL].reshape(TL, 2)
    cta = buf[2 * TL:].reshape(1024, 3)
    used = t[:, 1] != 0
    MASK = (1 << 48) - 1
    st = (t[used, 0] & MASK).astype(np.int64)
    en = (t[used, 1] & MASK).astype(np.int64)
    sm = ((t[used, 0] >> 48) & 0xff).astype(np.int64)
    kind = ((t[used, 0] >> 56) & 0xf).astype(np.int64)
    ghz = 1.965e3  # cycles per us at the bench clock
    ncta = int((cta[:, 0] != 0).sum())
    g0 = cta[:ncta, 0].astype(np.int64)
    g2 = cta[:ncta, 2].astype(np.int64)
    span_g = (g2 - g0) / 1e3  # us, CTA entry -> exit (globaltimer)
    entry_skew = (g0 - g0.min()) / 1e3
    # per SM: last unit end, first "no more units" moment ~ the earliest end of a warp's last unit
    per_sm_end = np.zeros(256); per_sm_first_idle = np.full(256, np.inf)
    # a warp's last unit is not identified directly; approximate the tail by unit starts:
    last_start = np.zeros(256)
    for s_ in np.unique(sm):
        k = sm == s_
        per_sm_end[s_] = en[k].max() / ghz
        last_start[s_] = st[k].max() / ghz
    smu = np.unique(sm)
    ends = per_sm_end[smu]
    # busy warps per SM over time (1 us buckets)
    T = int(en.max() / ghz) + 2
    occ = np.zeros(T)
    for a_, b_ in zip(st / ghz, en / ghz):
        occ[int(a_):int(b_) + 1] += 1
    occ /= len(smu)
    dur = (en - st) / ghz
    half = np.median(st)
    kinds = ["window", "light_sub", "light_warp", "heavy", "empty"]
    out = {"wl": wl, "rep": rep, "event_us": round(e0.elapsed_time(e1) * 1e3, 2), "units": int(used.sum()),
           "ctas": ncta, "cta_span_us": [round(float(np.min(span_g)), 2), round(float(np.median(span_g)), 2), round(float(np.max(span_g)), 2)],
           "cta_entry_skew_us_max": round(float(entry_skew.max()), 2),
           "first_unit_start_us": round(float(st.min() / ghz), 2),
           "sm_last_unit_end_us": [round(float(ends.min()), 2), round(float(np.median(ends)), 2), round(float(ends.max()), 2)],
           "sm_last_unit_start_us": [round(float(last_start[smu].min()), 2), round(float(np.median(last_start[smu])), 2), round(float(last_start[smu].max()), 2)],
           "busy_warps_per_sm_by_us": [round(float(v), 1) for v in occ],
           "unit_us_by_kind": {kinds[k]: {"n": int((kind == k).sum()),
                                          "mean_early": round(float(dur[(kind == k) & (st <= half)].mean()), 2) if ((kind == k) & (st <= half)).any() else None,
                                          "mean_late": round(float(dur[(kind == k) & (st > half)].mean()), 2) if ((kind == k) & (st > half)).any() else None,
                                          "p95": round(float(np.percentile(dur[kind == k], 95)), 2) if (kind == k).any() else None}
                               for k in range(5)}}
    res.append(out)
print(json.dumps(res[-1]))
print(json.dumps({"wl": wl, "event_us_all": [r["event_us"] for r in res], "sm_last_unit_end_max": [r["sm_last_unit_end_us"][2] for r in res]}))
