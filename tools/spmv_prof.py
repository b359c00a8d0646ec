"""Warp-cycle breakdown of spmv_kernel by mapping (needs the ACSR_PROF=1 variant:
ACSR_LIB_VARIANT=prof, built by tools/build_variants.sh prof).  Prints one JSON line:
per unit type (window / light_sub / light_warp / heavy / empty) total warp-cycles, units,
cycles per unit, and the window sub-phases, per launch, plus the kernel time."""
import ctypes, json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import synth
import paper_conf_sc_ashariseps14_b200 as acsr

wl = sys.argv[1] if len(sys.argv) > 1 else "rmat20"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 10
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
f = acsr._lib.acsr_debug_prof
f.argtypes = [ctypes.c_void_p, ctypes.c_int]
buf = (ctypes.c_ulonglong * 16)()
m.spmv(x)
f(buf, 1)
ts = []
for _ in range(reps):
    flush.zero_()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(); m.spmv(x); e1.record()
    torch.cuda.synchronize()
    ts.append(e0.elapsed_time(e1))
f(buf, 0)
v = [int(buf[i]) for i in range(16)]
L = max(1, v[15])
names = ["window", "light_sub", "light_warp", "heavy", "empty"]
warps = 148 * 32
tot_unit = sum(v[:5])
out = {"wl": wl, "launches": L, "spmv_ms_median": float(np.median(ts)),
       "warp_cycles_per_launch": {nm: v[i] / L for i, nm in enumerate(names)},
       "units_per_launch": {nm: v[10 + i] / L for i, nm in enumerate(names)},
       "cycles_per_unit": {nm: (v[i] / v[10 + i] if v[10 + i] else None) for i, nm in enumerate(names)},
       "share_of_unit_time": {nm: round(v[i] / max(1, tot_unit), 4) for i, nm in enumerate(names)},
       "window_phases_per_launch": {"bounds_wait": v[5] / L, "loads_gathers": v[6] / L, "in_order_sums": v[7] / L},
       "entry_to_first_unit_per_warp": v[8] / L / warps, "last_unit_to_exit_per_warp": v[9] / L / warps,
       "unit_cycles_per_warp": tot_unit / L / warps}
print(json.dumps(out))
