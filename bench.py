#!/usr/bin/env python
"""bench.py -- ACSR hot path on B200, one JSON line (driver contract).

Step = one pass of the whole ACSR path over one synthetic matrix already resident in
HBM: acsr_bin (row lengths -> bins -> work map, Alg. 1) + acsr_spmv (bin-specific
kernels, Alg. 2-4).  Default workload = BASELINE.json configs[1]: R-MAT scale 20, edge
factor 16, fp64 (C2).  `value` = GFLOP/s = 2*nnz per step / device time of the step
(bin included: the per-update cost of the dynamic-graph setting).
L2 is flushed (256 MiB write) between timed steps, outside the step's events.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl acsr|reference]
                  [--workload rmat20|rmat20_f32|webgoogle|livejournal|rmat20_split|pagerank|
                              pagerank_dist|dynamic|dynamic_mixed|hits|rwr]

With N > 1 (torchrun) the default workload is the SAME C2 matrix row-split across the
ranks (§VIII, reading Q19: contiguous nnz-balanced row ranges from acsr_partition,
every rank bins its rows and runs acsr_spmv on them; y stays distributed) -- one problem
at every N (strong scaling), the time is the max over ranks.  `--replicas` restores the
old independent-matrix-per-rank mode.  Every default line also carries a `pagerank_dist`
record: C4 (R-MAT s26 in-link PageRank) row-partitioned over the N ranks with the
library-owned NCCL exchange (acsr_comm) and with the fused peer-memory exchange, against
SURVEY §8(e)'s bound max(T1/P, T_comm).  `--impl reference` times the CPU oracle (plain
sequential C) on the same workload (rank 0 only).
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402

FALLBACK_HBM = 6650.0


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured"
    return FALLBACK_HBM, "fallback"


class L2Flush:
    """The L2 flush between timed steps: a 256 MiB write (larger than the 126 MB L2).
    ACSR_BENCH_FLUSH=write+read adds a 256 MiB read of a second buffer after the write, so
    the step starts with a clean L2 (the write leaves ~126 MB of dirty lines whose
    write-back otherwise lands inside the next timed step).  Graph-capturable."""

    def __init__(self, dev, mode=None):
        self.mode = mode or os.environ.get("ACSR_BENCH_FLUSH", "write")
        assert self.mode in ("write", "write+read"), self.mode
        self.w = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
        if self.mode == "write+read":
            self.r = torch.zeros(64 << 20, dtype=torch.int32, device=dev)
            self.acc = torch.zeros((), dtype=torch.int64, device=dev)

    def zero_(self):  # the name the call sites used for the plain write flush
        self.w.zero_()
        if self.mode == "write+read":
            torch.sum(self.r, dim=0, dtype=torch.int64, out=self.acc)

    @staticmethod
    def describe(mode=None):
        mode = mode or os.environ.get("ACSR_BENCH_FLUSH", "write")
        return ("flushed: 256 MiB write" + (" + 256 MiB read (clean L2)" if mode == "write+read" else "")
                + " between timed steps (outside the step events)")


class Clocks:
    """Sample SM clocks + throttle reasons DURING the timed region.

    NVML (pynvml) is polled from a thread every ~2 ms, so even a few-ms timed region
    gets samples; `nvidia-smi -lms 100` is the fallback when NVML is unavailable.  The
    sampler is started (and its first sample awaited) before the timed region."""

    REASONS = (("hw_slowdown", "nvmlClocksEventReasonHwSlowdown"),
               ("hw_thermal_slowdown", "nvmlClocksEventReasonHwThermalSlowdown"),
               ("sw_thermal_slowdown", "nvmlClocksEventReasonSwThermalSlowdown"),
               ("sw_power_cap", "nvmlClocksEventReasonSwPowerCap"))
    Q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.proc = None
        self.lines = []
        self.samples = []  # (sm_mhz, max_mhz, reasons bitmask)
        self.stop = threading.Event()
        self.nv = None

    def _nvml_handle(self):
        import pynvml
        pynvml.nvmlInit()
        idx = self.index
        vis = os.environ.get("CUDA_VISIBLE_DEVICES", "")
        ids = [v.strip() for v in vis.split(",") if v.strip()]
        if ids and idx < len(ids):
            if ids[idx].isdigit():
                idx = int(ids[idx])
            else:
                return pynvml, pynvml.nvmlDeviceGetHandleByUUID(ids[idx])
        return pynvml, pynvml.nvmlDeviceGetHandleByIndex(idx)

    def _poll(self):
        nv, h = self.nv
        mx = nv.nvmlDeviceGetMaxClockInfo(h, nv.NVML_CLOCK_SM)
        while True:
            try:
                sm = nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM)
                rs = nv.nvmlDeviceGetCurrentClocksEventReasons(h)
                self.samples.append((float(sm), float(mx), int(rs)))
            except Exception:
                pass
            if self.stop.wait(0.002):
                break

    def __enter__(self):
        try:
            self.nv = self._nvml_handle()
            self.t = threading.Thread(target=self._poll, daemon=True)
            self.t.start()
            t0 = time.perf_counter()
            while not self.samples and time.perf_counter() - t0 < 2.0:
                time.sleep(0.001)
            self.n0 = len(self.samples)
            return self
        except Exception:
            self.nv = None
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def __exit__(self, *a):
        if self.nv is not None:
            self.n1 = len(self.samples)
            self.stop.set()
            self.t.join(1.0)
            return
        if self.proc:
            time.sleep(0.25)
            self.proc.terminate()
            try:
                self.proc.wait(2)
            except Exception:
                self.proc.kill()

    def summary(self):
        if self.nv is not None:
            nv = self.nv[0]
            # samples taken while the timed region ran (plus the one awaited before it)
            s = self.samples[max(0, self.n0 - 1):self.n1] or self.samples[-1:]
            reasons = sorted({name for name, attr in self.REASONS
                              for (_, _, rs) in s if rs & getattr(nv, attr, 0)})
            return {"sm_mhz": float(np.median([v[0] for v in s])) if s else None,
                    "sm_max_mhz": max(v[1] for v in s) if s else None,
                    "reasons": reasons, "samples": len(s), "source": "nvml, 2 ms poll"}
        sm, mx, reasons = [], 0.0, set()
        names = [r[0] for r in self.REASONS]
        for l in self.lines:
            f = [x.strip() for x in l.split(",")]
            if len(f) < 6:
                continue
            try:
                sm.append(float(f[0]))
                mx = max(mx, float(f[1]))
            except ValueError:
                continue
            for n, v in zip(names, f[2:6]):
                if v.lower().startswith("active"):
                    reasons.add(n)
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": mx or None,
                "reasons": sorted(reasons), "samples": len(sm), "source": "nvidia-smi -lms 100"}


# ------------------------------------------------------------------------------ workloads
def make_workload(name, dev, rank):
    seed_shift = 1000 * rank
    dtype = torch.float32 if name.endswith("_f32") else torch.float64
    if name.startswith("rmat20"):
        rp, ci = synth.rmat_csr(20, seed=20 + seed_shift, device=dev)
        label = f"rmat20_ef16_{'f32' if dtype == torch.float32 else 'f64'}"
    elif name == "webgoogle":
        rp, ci = synth.powerlaw_csr(seed=3 + seed_shift, device=dev, **synth.WEB_GOOGLE)
        label = "webgoogle_like_f64"
    elif name == "livejournal":
        rp, ci = synth.powerlaw_csr(seed=4 + seed_shift, device=dev, **synth.LIVEJOURNAL)
        label = "livejournal_like_f64"
    else:
        raise SystemExit(f"unknown workload {name}")
    n = rp.numel() - 1
    val = synth.values(ci.numel(), 1014 + seed_shift, dtype, dev)
    x = synth.vector(n, 2014 + seed_shift, dtype, dev)
    return label, dtype, rp, ci, val, x


def bin_stats(rp, bin_offsets, heavy_chunk=1024):
    """The B200 analogue of the paper's Table V: rows per bin
    (from acsr_bin's bin_offsets), non-empty bins, rows split across warps (> 1024 nnz)
    and their chunks."""
    off = bin_offsets.cpu().numpy().astype(np.int64)
    cnt = np.diff(off)
    ln = (rp[1:] - rp[:-1]).to(torch.int64)
    heavy = ln[ln > heavy_chunk]
    return {"rows_per_bin": {int(b): int(c) for b, c in enumerate(cnt) if c},
            "nonempty_bins": int((cnt[1:] > 0).sum()),
            "split_rows": int(heavy.numel()),
            "split_chunks": int(((heavy + heavy_chunk - 1) // heavy_chunk).sum()) if heavy.numel() else 0,
            "split_nnz_share": round(float(heavy.sum()) / max(1, int(ln.sum())), 4)}


def read_stream_gbs(dev, gib=2, reps=5):
    """Read-only streaming bandwidth measured in the same job (quote the
    roofline against the spec, the measured copy and a read-only stream): a 2 GiB fp32
    reduction (torch.sum, far larger than L2), best of `reps`."""
    buf = torch.ones((gib << 30) // 4, dtype=torch.float32, device=dev)
    buf.sum()
    torch.cuda.synchronize()
    best = 0.0
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        buf.sum()
        e1.record()
        torch.cuda.synchronize()
        best = max(best, buf.numel() * 4 / (e0.elapsed_time(e1) * 1e-3) / 1e9)
    del buf
    torch.cuda.empty_cache()
    return best


HBM_SPEC_GBS = 8000.0  # B200 HBM3e nominal (the north star's denominator)


def algorithmic_bytes(rp, ci, dtype, n_cols=None):
    """(s_v+4) nnz + 4(n+1) row_ptr + 4n bin_rows + s_v n_c x + s_v n y."""
    n = rp.numel() - 1
    nnz = ci.numel()
    sv = 8 if dtype == torch.float64 else 4
    n_c = int((torch.bincount(ci.long(), minlength=n if n_cols is None else n_cols) > 0).sum())
    return (sv + 4) * nnz + 4 * (n + 1) + 4 * n + sv * n_c + sv * n, n_c


def acsr_num_sms_host():
    return torch.cuda.get_device_properties(torch.cuda.current_device()).multi_processor_count


def workload_config(label, n, nnz, world, replicas=False):
    """The `config` of the default line: identical keys and values at every N (and in the
    reference arm), so the driver can match the lines."""
    return {"workload": label, "n_rows": n, "nnz": nnz,
            "l2": L2Flush.describe(),
            "parallelism": (f"independent matrix per rank x{world} (weak)" if replicas
                            else f"row-split x{world} (P:345)" if world > 1 else "1 GPU")}


def ncu_traffic(label):
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(p):
        d = json.load(open(p))
        v = d.get(label)
        if v:
            return v
    return None


# ------------------------------------------------------------------------------ acsr arm
def row_split(rp, ci, val, rank, world, b_nnz, b_row):
    """This rank's rows [splits[rank], splits[rank+1]) of one CSR (acsr_partition, O8),
    col/val copied with their global 16-byte phase (dist.aligned_slice) so every row is
    summed as on one GPU.  Returns (row_ptr_local, col_local, val_local, splits)."""
    import paper_conf_sc_ashariseps14_b200 as acsr
    from paper_conf_sc_ashariseps14_b200 import dist as pdist
    splits = acsr.acsr_partition(rp, world, b_nnz, b_row, align=32).cpu().numpy()
    lo, hi = int(splits[rank]), int(splits[rank + 1])
    k0, k1 = int(rp[lo]), int(rp[hi])
    rpl = (rp[lo:hi + 1].to(torch.int64) - k0).to(torch.int32)
    cil = pdist.aligned_slice(ci, k0, k1, 4)
    vl = None if val is None else pdist.aligned_slice(val, k0, k1, 16 // val.element_size())
    return rpl, cil, vl, splits


def run_acsr(args, dev, rank, world):
    import paper_conf_sc_ashariseps14_b200 as acsr

    replicas = args.replicas and world > 1
    label, dtype, rp, ci, val, x = make_workload(args.workload, dev, rank if replicas else 0)
    n_glob, nnz_glob = rp.numel() - 1, ci.numel()
    splits = None
    if world > 1 and not replicas:  # one matrix, row-split: this rank's rows
        rp, ci, val, splits = row_split(rp, ci, val, rank, world, 4 + val.element_size(), 16)
        torch.cuda.empty_cache()
    n, nnz = rp.numel() - 1, ci.numel()
    alg_bytes, n_c = algorithmic_bytes(rp, ci, dtype, n_cols=x.numel())
    stream = torch.cuda.current_stream()
    br = torch.empty(n, dtype=torch.int32, device=dev)
    bo = torch.empty(33, dtype=torch.int32, device=dev)
    ws = torch.empty(acsr.acsr_bin_workspace_bytes(n, x.numel(), nnz), dtype=torch.uint8, device=dev)
    y = torch.empty(n, dtype=dtype, device=dev)
    flush = L2Flush(dev)

    def step():
        acsr.acsr_bin(rp, None, nnz, br, bo, ws, col_idx=ci, n_cols=x.numel())
        acsr.acsr_spmv(rp, ci, val, x, br, bo, ws, None, y)

    for _ in range(args.warmup):
        flush.zero_()
        step()
    torch.cuda.synchronize()
    K = args.steps
    # the timed steps: acsr_bin + acsr_spmv back to back through the public calls, the K
    # steps (each after its L2 flush) issued from ONE CUDA graph captured from those calls, so
    # the device never waits for the Python host loop (issuing one call at a time from Python
    # is ~180 us per step, slower than the GPU: the eager loop below is reported beside).
    # Events only at the step's ends (graph event-record nodes): an event between the two
    # calls would break the programmatic-dependent-launch overlap of the binning's last
    # kernel with the SpMV's launch, measured +5.3 us per step (profiles/r2_step_events.json).
    def graphed(n_ev, body):
        evs = [[torch.cuda.Event(enable_timing=True, external=True) for _ in range(n_ev)] for _ in range(K)]
        g = torch.cuda.CUDAGraph()
        cap = torch.cuda.Stream()
        cap.wait_stream(stream)
        with torch.cuda.graph(g, stream=cap):
            for k in range(K):
                flush.zero_()
                body(evs[k])
        torch.cuda.synchronize()
        return g, evs

    def body_step(e):
        e[0].record()
        acsr.acsr_bin(rp, None, nnz, br, bo, ws, col_idx=ci, n_cols=x.numel())
        acsr.acsr_spmv(rp, ci, val, x, br, bo, ws, None, y)
        e[1].record()

    def body_split(e):
        e[0].record()
        acsr.acsr_bin(rp, None, nnz, br, bo, ws, col_idx=ci, n_cols=x.numel())
        e[1].record()
        acsr.acsr_spmv(rp, ci, val, x, br, bo, ws, None, y)
        e[2].record()

    g_step, ev = graphed(2, body_step)
    g_split, evb = graphed(3, body_split)
    g_split.replay()  # warm replays (first replay uploads the graph)
    g_step.replay()
    torch.cuda.synchronize()
    if world > 1:
        torch.distributed.barrier()
    torch.cuda.synchronize()
    with Clocks(torch.cuda.current_device()) as clk:
        t0 = time.perf_counter()
        g_step.replay()
        torch.cuda.synchronize()
        wall = time.perf_counter() - t0
    if world > 1:
        torch.distributed.barrier()
    t_step = np.array([ev[k][0].elapsed_time(ev[k][1]) for k in range(K)])
    # the breakdown (and the SpMV kernel's duration for the roofline): the same graphed steps
    # with an event between the calls, same flush protocol
    g_split.replay()
    torch.cuda.synchronize()
    t_bin = np.array([evb[k][0].elapsed_time(evb[k][1]) for k in range(K)])
    t_spmv = np.array([evb[k][1].elapsed_time(evb[k][2]) for k in range(K)])
    # the same steps issued eagerly, one Python call at a time (host-bound: reported only)
    eve = [[torch.cuda.Event(enable_timing=True) for _ in range(2)] for _ in range(K)]
    t1 = time.perf_counter()
    for k in range(K):
        flush.zero_()
        eve[k][0].record(stream)
        acsr.acsr_bin(rp, None, nnz, br, bo, ws, col_idx=ci, n_cols=x.numel())
        acsr.acsr_spmv(rp, ci, val, x, br, bo, ws, None, y)
        eve[k][1].record(stream)
    torch.cuda.synchronize()
    wall_eager = time.perf_counter() - t1
    t_step_eager = float(np.mean([eve[k][0].elapsed_time(eve[k][1]) for k in range(K)]))
    # warm variant (SURVEY §8(d) timing protocol): K back-to-back SpMVs, no flush -- the
    # iterative-use number; reported beside the flushed (cold-L2) step, not as `value`
    torch.cuda.synchronize()
    w0, w1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    w0.record(stream)
    for _ in range(K):
        acsr.acsr_spmv(rp, ci, val, x, br, bo, ws, None, y)
    w1.record(stream)
    torch.cuda.synchronize()
    t_spmv_warm = w0.elapsed_time(w1) / K
    tot = float(t_step.sum())
    if world > 1:
        tt = torch.tensor([tot], dtype=torch.float64, device=dev)
        torch.distributed.all_reduce(tt, op=torch.distributed.ReduceOp.MAX)
        tot = float(tt.item())
    # end-to-end through the public API with host buffers (pinned), copies inside
    rp_h, ci_h, val_h, x_h = (t.cpu().pin_memory() for t in (rp, ci, val, x))
    y_h = torch.empty(n, dtype=dtype).pin_memory()
    y_h2 = [torch.empty(n, dtype=dtype).pin_memory() for _ in range(2)]
    for _ in range(2):
        acsr.spmv_from_host(rp_h, ci_h, val_h, x_h, y_h, device=dev)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ke = max(3, min(K, 10))
    # one call after another on one stream (every step: all inputs in, y out, serialised)
    e0.record(stream)
    for _ in range(ke):
        acsr.spmv_from_host(rp_h, ci_h, val_h, x_h, y_h, device=dev)
    e1.record(stream)
    torch.cuda.synchronize()
    t_e2e_seq = e0.elapsed_time(e1) / ke
    # the same calls alternating between two streams (double-buffered streaming): step k+1's
    # host->device copies overlap step k's kernels and device->host copy (PCIe is full
    # duplex); every step still copies all of its inputs in and its y out
    sts = [torch.cuda.Stream(device=dev) for _ in range(2)]
    for k in range(2):
        acsr.spmv_from_host(rp_h, ci_h, val_h, x_h, y_h2[k], device=dev, stream=sts[k])
    torch.cuda.synchronize()
    p0, p1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    p0.record(stream)
    for st in sts:
        st.wait_event(p0)
    for k in range(ke):
        acsr.spmv_from_host(rp_h, ci_h, val_h, x_h, y_h2[k % 2], device=dev, stream=sts[k % 2])
    for st in sts:
        stream.wait_stream(st)
    p1.record(stream)
    torch.cuda.synchronize()
    t_e2e = p0.elapsed_time(p1) / ke
    if world > 1:
        te = torch.tensor([t_e2e_seq], dtype=torch.float64, device=dev)
        torch.distributed.all_reduce(te, op=torch.distributed.ReduceOp.MAX)
        t_e2e_seq = float(te.item())
    if world > 1:  # whole job: every rank ran its own e2e loop concurrently; max over ranks
        te = torch.tensor([t_e2e], dtype=torch.float64, device=dev)
        torch.distributed.all_reduce(te, op=torch.distributed.ReduceOp.MAX)
        t_e2e = float(te.item())
    # resident-matrix variant (the iterative / dynamic-graph use: the CSR stays in HBM):
    # per step H2D of x, acsr_bin + acsr_spmv through the public API, D2H of y
    x_d = torch.empty_like(x)
    for _ in range(2):
        x_d.copy_(x_h, non_blocking=True)
        acsr.acsr_bin(rp, None, nnz, br, bo, ws, col_idx=ci, n_cols=x.numel())
        acsr.acsr_spmv(rp, ci, val, x_d, br, bo, ws, None, y)
        y_h.copy_(y, non_blocking=True)
    torch.cuda.synchronize()
    r0, r1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    r0.record(stream)
    for _ in range(ke):
        x_d.copy_(x_h, non_blocking=True)
        acsr.acsr_bin(rp, None, nnz, br, bo, ws, col_idx=ci, n_cols=x.numel())
        acsr.acsr_spmv(rp, ci, val, x_d, br, bo, ws, None, y)
        y_h.copy_(y, non_blocking=True)
    r1.record(stream)
    torch.cuda.synchronize()
    t_res = r0.elapsed_time(r1) / ke
    # the same steps alternating between two streams, each with its own x / y / plan
    # buffers (a plan workspace must not be shared by concurrent calls): x in of step k+1
    # overlaps step k's kernels and y out
    rbuf = [(torch.empty_like(x), torch.empty_like(y), torch.empty_like(br), torch.empty_like(bo),
             torch.empty_like(ws), torch.empty(n, dtype=dtype).pin_memory()) for _ in range(2)]

    def res_step(k):
        xd, yd, brk, bok, wsk, yhk = rbuf[k % 2]
        with torch.cuda.stream(sts[k % 2]):
            s_ = sts[k % 2]
            xd.copy_(x_h, non_blocking=True)
            acsr.acsr_bin(rp, None, nnz, brk, bok, wsk, col_idx=ci, n_cols=x.numel(), stream=s_)
            acsr.acsr_spmv(rp, ci, val, xd, brk, bok, wsk, None, yd, stream=s_)
            yhk.copy_(yd, non_blocking=True)

    for k in range(2):
        res_step(k)
    torch.cuda.synchronize()
    r2, r3 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    r2.record(stream)
    for st in sts:
        st.wait_event(r2)
    for k in range(ke):
        res_step(k)
    for st in sts:
        stream.wait_stream(st)
    r3.record(stream)
    torch.cuda.synchronize()
    t_res2 = r2.elapsed_time(r3) / ke
    if world > 1:
        te = torch.tensor([t_res, t_res2], dtype=torch.float64, device=dev)
        torch.distributed.all_reduce(te, op=torch.distributed.ReduceOp.MAX)
        t_res, t_res2 = float(te[0].item()), float(te[1].item())
    h2d = sum(t.numel() * t.element_size() for t in (rp_h, ci_h, val_h, x_h))
    d2h = y_h.numel() * y_h.element_size()
    ctx = cusparse_context(rp, ci, val, x, n)
    rs = read_stream_gbs(dev)
    bstats = bin_stats(rp, bo)
    # gather-only pass over the same column array, same L2 flush: x[col] with torch's
    # index kernel (strictly less work than the SpMV: no values, no row sums) -- the
    # in-job measure of the random-gather bound the SpMV sits against
    g_out = torch.empty(nnz, dtype=dtype, device=dev)
    tg = []
    for k in range(max(5, min(K, 20))):
        flush.zero_()
        g0, g1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        g0.record(stream)
        torch.index_select(x, 0, ci, out=g_out)  # int32 indices, as the SpMV reads them
        g1.record(stream)
        torch.cuda.synchronize()
        if k >= 2:
            tg.append(g0.elapsed_time(g1))
    t_gather = float(np.median(tg))
    del g_out
    c4 = None if args.no_c4 else pagerank_dist_record(args, dev, rank, world)
    if rank != 0:
        return None
    peak, peak_kind = peaks()
    units = nnz * world if replicas else nnz_glob  # nnz multiplied per step by the whole job
    gflops = 2.0 * units * K / (tot * 1e-3) / 1e9
    spmv_ms = float(t_spmv.mean())
    achieved = alg_bytes / (spmv_ms * 1e-3) / 1e9
    line = {
        "metric": "SpMV GFLOP/s (bin+SpMV per step) & HBM GB/s vs peak",
        "value": round(gflops, 3), "unit": "GFLOP/s", "n_gpus": world, "steps": K, "warmup": args.warmup,
        "ms_per_step": round(tot / K, 5), "higher_is_better": True, "scaling": "weak" if replicas else "strong",
        "vs_baseline": None, "dtype": "f64" if dtype == torch.float64 else "f32", "data": "synthetic",
        "config": workload_config(label, n_glob, nnz_glob, world, replicas),
        "breakdown": {"rank0_rows": n, "rank0_nnz": nnz, "rank0_referenced_cols": n_c,
                      "splits": None if splits is None else [int(v) for v in splits],
                      "timing": "value: the K flushed steps issued from one CUDA graph captured from the public "
                                "calls, events (graph event-record nodes) at the step's ends only (bin + SpMV back "
                                "to back, PDL overlap); t_bin / t_spmv: a second graph with an event between the "
                                "calls; t_step_eager: the same steps issued one Python call at a time (host-bound)",
                      "t_step_eager_ms": round(t_step_eager, 5),
                      "wall_s_eager_loop": round(wall_eager, 4),
                      "t_bin_plus_spmv_split_ms": round(float((t_bin + t_spmv).mean()), 5),
                      "t_bin_ms": round(float(t_bin.mean()), 5), "t_spmv_ms": round(spmv_ms, 5),
                      "pt_st": round(float(t_bin.mean()) / spmv_ms, 3),
                      "spmv_gflops": round(2.0 * nnz / (spmv_ms * 1e-3) / 1e9, 2),
                      "t_spmv_min_ms": round(float(t_spmv.min()), 5),
                      "t_spmv_median_ms": round(float(np.median(t_spmv)), 5),
                      "t_spmv_warm_back_to_back_ms": round(t_spmv_warm, 5),
                      "wall_s_timed_loop": round(wall, 4),
                      "gather_pass_ms": round(t_gather, 5),
                      "gather_pass_note": "torch.index_select(x, 0, col) over the same matrix, L2 flushed: "
                                          "nnz random gathers + col read + nnz-value write, no row sums",
                      "spmv_over_gather_pass": round(spmv_ms / t_gather, 3),
                      "gather_roofline_ms": round(nnz / 197e9 * 1e3, 5),
                      "gather_roofline_note": "pure random 8-byte gathers from an L2-resident x run at ~198 G/s "
                                              "on this B200, limited by the L1TEX->XBAR request interface "
                                              "(profiles/r2_gather_limiter.json); one gather per nnz"},
        "context": ctx,
        "bins": bstats,
        "roofline": {"bound": "hbm", "achieved": round(achieved, 1), "peak": peak, "unit": "GB/s",
                     "frac": round(achieved / peak, 4), "traffic": ncu_traffic(label),
                     "kernel": "acsr::spmv_kernel", "peak_kind": peak_kind,
                     "algorithmic_bytes_per_launch": int(alg_bytes),
                     "vs_other_peaks": {"read_stream_measured_gbs": round(rs, 1),
                                        "frac_vs_read_stream": round(achieved / rs, 4),
                                        "spec_gbs": HBM_SPEC_GBS,
                                        "frac_vs_spec": round(achieved / HBM_SPEC_GBS, 4)}},
        "e2e": {"value": round(2.0 * units / (t_e2e * 1e-3) / 1e9, 3), "unit": "GFLOP/s",
                "h2d_bytes_per_step": int(h2d) * world, "d2h_bytes_per_step": int(d2h) * world,
                "ms_per_step": round(t_e2e, 4),
                "note": "whole CSR + x uploaded every step (PCIe-bound), spmv_from_host calls alternating "
                        "between two streams (step k+1's uploads overlap step k's kernels and y download); "
                        "sequential: the same calls on one stream; resident_matrix: CSR kept in HBM, "
                        "x in / y out per step",
                "sequential": {"value": round(2.0 * units / (t_e2e_seq * 1e-3) / 1e9, 3), "unit": "GFLOP/s",
                               "ms_per_step": round(t_e2e_seq, 4)},
                "resident_matrix": {"value": round(2.0 * units / (t_res2 * 1e-3) / 1e9, 3),
                                    "unit": "GFLOP/s", "ms_per_step": round(t_res2, 4),
                                    "h2d_bytes_per_step": int(x_h.numel() * x_h.element_size()) * world,
                                    "d2h_bytes_per_step": int(d2h) * world,
                                    "note": "two streams, own x / y / plan per stream; one stream: sequential_ms",
                                    "sequential_ms": round(t_res, 4)}},
        "gpu_launches": 4 * K * world,  # per step and rank: bin_count, bin_scan, bin_scatter, spmv_kernel
        "clocks": clk.summary(),
    }
    # the gather bound (profiles/r2_gather_limiter.json): one L1TEX->XBAR request per
    # SM-cycle; requests = one per nnz gather + the CSR streams in 128-byte lines + y store beats
    sv = 8 if dtype == torch.float64 else 4
    reqs = nnz + (4 + sv) * nnz / 128.0 + 8.0 * (n + 1) / 128.0 + sv * n / 32.0
    f_sm = (line["clocks"].get("sm_mhz") or 1965.0) * 1e6
    gb_ms = reqs / (acsr_num_sms_host() * f_sm) * 1e3
    line["roofline"]["vs_gather_bound"] = {
        "requests_per_launch": int(reqs), "bound_ms_at_1_req_per_sm_cycle": round(gb_ms, 5),
        "frac": round(gb_ms / spmv_ms, 4), "sustained_bound_ms_at_85pct": round(gb_ms / 0.85, 5),
        "frac_of_sustained": round(gb_ms / 0.85 / spmv_ms, 4),
        "note": "L2-resident x: the SM's L1TEX->XBAR request interface is the busiest unit of a pure random "
                "gather (ncu, 85 % of elapsed); no L1 hits assumed"}
    if c4 is not None:
        line["pagerank_dist"] = c4
    if not args.no_cpu_baseline and world == 1:  # the oracle baseline: rank 0 at N = 1 only
        line["cpu_baseline"] = cpu_baseline(rp, ci, val, x, dtype)
    return line


def cusparse_context(rp, ci, val, x, n):
    """Context only (not our path): cuSPARSE CSR SpMV through torch.sparse_csr on the same
    matrix, same L2 flush protocol.  Returns ms and GFLOP/s, or the error text."""
    try:
        A = torch.sparse_csr_tensor(rp.to(torch.int64), ci.to(torch.int64), val, size=(n, x.numel()))
        flush = torch.empty(256 << 20, dtype=torch.uint8, device=x.device)
        xs = x.view(-1, 1)
        for _ in range(3):
            (A @ xs)
        ts = []
        for _ in range(10):
            flush.zero_()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            (A @ xs)
            e1.record()
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1))
        ms = float(np.median(ts))
        return {"cusparse_csr_spmv_ms": round(ms, 5), "cusparse_gflops": round(2.0 * ci.numel() / (ms * 1e-3) / 1e9, 2),
                "note": "torch.sparse_csr @ dense (cuSPARSE), context only; no binning cost"}
    except Exception as e:  # pragma: no cover - context only
        return {"cusparse_error": str(e)[:200]}


def cpu_baseline(rp, ci, val, x, dtype, budget_s=12.0):
    """The oracle's plain sequential SpMV (O4') on 1 host core, repeated over the whole
    matrix for ~budget_s seconds; GFLOP/s with the same 2*nnz."""
    import oracle

    rph, cih = rp.cpu().numpy(), ci.cpu().numpy()
    vh, xh = val.cpu().numpy(), x.cpu().numpy()
    y = np.empty(rph.size - 1, vh.dtype)
    oracle.spmv_plain(rph, cih, vh, xh, out=y)
    reps, t0 = 0, time.perf_counter()
    while time.perf_counter() - t0 < budget_s or reps < 2:
        oracle.spmv_plain(rph, cih, vh, xh, out=y, threads=1)
        reps += 1
    dt = (time.perf_counter() - t0) / reps
    # the same loop split statically over all host cores (OpenMP), a few reps -- context
    nc = os.cpu_count() or 1
    oracle.spmv_plain(rph, cih, vh, xh, out=y, threads=nc)
    r2, t1 = 0, time.perf_counter()
    while time.perf_counter() - t1 < min(3.0, budget_s / 4) or r2 < 2:
        oracle.spmv_plain(rph, cih, vh, xh, out=y, threads=nc)
        r2 += 1
    dt_all = (time.perf_counter() - t1) / r2
    return {"value": round(2.0 * cih.size / dt / 1e9, 4), "unit": "GFLOP/s", "cores": 1, "kind": "oracle",
            "sample": f"whole matrix, plain sequential CSR SpMV (oracle O4'), {reps} reps, "
                      f"{dt * 1e3:.1f} ms each; host has {nc} cores",
            "all_cores": {"value": round(2.0 * cih.size / dt_all / 1e9, 4), "cores": nc,
                          "sample": f"same loop, OpenMP static over {nc} threads, {r2} reps"}}


# ------------------------------------------------------------------------------ PageRank (C4)
def run_pagerank(args, dev, rank, world):
    """C4 on one GPU per rank (independent replicas when N > 1): in-link pattern CSR of
    R-MAT scale S (default 24 on one GPU; 26 with --scale 26), one fused
    acsr_pagerank_step per iteration (SpMV + epilogue + Delta^2).  value = GTEPS
    (nnz per iteration / iteration time); also the cold-start iteration count."""
    import paper_conf_sc_ashariseps14_b200 as acsr

    S = args.scale or 24
    rp, ci = synth.rmat_csr(S, seed=S + 1000 * rank, device=dev, transpose=True)
    n, nnz = rp.numel() - 1, ci.numel()
    outdeg = torch.bincount(ci.long(), minlength=n).to(torch.int32)
    t_relabel = None
    if args.relabel:  # acsr_degree_relabel on the device (sort + scan + copy), timed with events
        srt = args.relabel_sort
        for _ in range(2):
            acsr.acsr_degree_relabel(rp, ci, outdeg, sort_rows=srt)
        torch.cuda.synchronize()
        r0, r1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        r0.record()
        rp2, ci2, od2, _ = acsr.acsr_degree_relabel(rp, ci, outdeg, sort_rows=srt)
        r1.record()
        torch.cuda.synchronize()
        t_relabel = r0.elapsed_time(r1) * 1e-3
        rp, ci, outdeg = rp2, ci2, od2
        del rp2, ci2, od2
        torch.cuda.empty_cache()
    n_nd = int((outdeg > 0).sum())
    m = acsr.ACSRMatrix(rp, ci)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    m.rebin()
    e1.record()
    torch.cuda.synchronize()
    t_bin = e0.elapsed_time(e1)
    x = torch.full((n,), 1.0 / n, dtype=torch.float64, device=dev)
    xs = acsr.acsr_pagerank_scale(x, outdeg)
    xn, xsn = torch.empty_like(x), torch.empty_like(x)
    d2 = torch.zeros(1, dtype=torch.float64, device=dev)
    tel = 0.15 / n

    def step():
        acsr.acsr_pagerank_step(m.row_begin, m.col_idx, m.bin_rows, m.bin_offsets, m.plan_ws, xs, x,
                                outdeg, xn, xsn, d2, 0.85, tel, n)

    for _ in range(args.warmup):
        step()
    K = args.steps
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(K + 1)]
    if world > 1:
        torch.distributed.barrier()
    torch.cuda.synchronize()
    with Clocks(torch.cuda.current_device()) as clk:
        ev[0].record()
        for k in range(K):
            step()
            ev[k + 1].record()
        torch.cuda.synchronize()
    ts = np.array([ev[k].elapsed_time(ev[k + 1]) for k in range(K)])
    tot = float(ts.sum())
    if world > 1:
        tt = torch.tensor([tot], dtype=torch.float64, device=dev)
        torch.distributed.all_reduce(tt, op=torch.distributed.ReduceOp.MAX)
        tot = float(tt.item())
    acsr.pagerank(m, outdeg, eps=1e-6)  # warm the loop (allocations)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    x2, it, dd = acsr.pagerank(m, outdeg, eps=1e-6)
    torch.cuda.synchronize()
    t_conv = time.perf_counter() - t0
    if rank != 0:
        return None
    peak, kind = peaks()
    alg = 4 * nnz + 36 * n + 8 * n_nd
    ms = tot / K
    traffic = ncu_traffic(f"pagerank_rmat{S}_inlink" + ("_degree_relabelled" if args.relabel else ""))
    return {"metric": "PageRank iteration GTEPS (in-link pattern SpMV + fused epilogue)",
            "value": round(nnz * world / (ms * 1e-3) / 1e9, 3), "unit": "GTEPS", "n_gpus": world, "steps": K,
            "warmup": args.warmup, "ms_per_step": round(ms, 5), "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": f"pagerank_rmat{S}_inlink" + ("_degree_relabelled" if args.relabel else ""),
                       "n_rows": n, "nnz": nnz, "non_dangling": n_nd,
                       "relabel": ("acsr_degree_relabel (device%s)" % (", rows sorted" if args.relabel_sort else ""))
                       if args.relabel else None,
                       "l2": "not flushed (iterative use); x = %d MB" % (8 * n >> 20),
                       "parallelism": "independent replica per rank" if world > 1 else "1 GPU"},
            "breakdown": {"t_bin_ms": round(t_bin, 4), "cold_iterations": it, "final_delta": dd ** 0.5,
                          "cold_run_ms": round(t_conv * 1e3, 3),
                          "relabel_ms": None if t_relabel is None else round(t_relabel * 1e3, 3),
                          "cold_solve_incl_relabel_and_bin_ms": None if t_relabel is None else
                          round((t_relabel + t_conv) * 1e3 + t_bin, 3),
                          "gflops_equiv": round(nnz / (ms * 1e-3) / 1e9, 2)},
            "roofline": {"bound": "hbm", "achieved": round(alg / (ms * 1e-3) / 1e9, 1), "peak": peak, "unit": "GB/s",
                         "frac": round(alg / (ms * 1e-3) / 1e9 / peak, 4),
                         "traffic": traffic,
                         "traffic_gbs_at_this_ms": None if not traffic else round(traffic / (ms * 1e-3) / 1e9, 1),
                         "traffic_frac_of_peak": None if not traffic else round(traffic / (ms * 1e-3) / 1e9 / peak, 4),
                         "traffic_note": "ncu DRAM bytes of one step (profiles/r2_ncu_c4_traffic.json): random xs misses "
                                         "fetch a full DRAM burst per 8 used bytes",
                         "vs_other_peaks": {"spec_gbs": HBM_SPEC_GBS,
                                            "frac_vs_spec": round(alg / (ms * 1e-3) / 1e9 / HBM_SPEC_GBS, 4)},
                         "kernel": "acsr::spmv_kernel<PR>", "peak_kind": kind,
                         "algorithmic_bytes_per_launch": int(alg)},
            "gpu_launches": K, "clocks": clk.summary()}


def run_spmv_split(args, dev, rank, world):
    """N4: ONE C2 matrix (R-MAT s20 fp64, the same seed on every rank) row-split across
    the ranks (nnz-balanced contiguous ranges, cost 12 len + 16), every rank bins
    its rows and runs acsr_spmv on them each step; y stays distributed (no exchange in the
    step).  Strong scaling: value = 2 nnz per step / max-over-ranks step time."""
    from paper_conf_sc_ashariseps14_b200 import dist as pdist

    rp, ci = synth.rmat_csr(20, seed=20, device=dev)
    n, nnz = rp.numel() - 1, ci.numel()
    val = synth.values(nnz, 1014, torch.float64, dev)
    x = synth.vector(n, 2014, torch.float64, dev)
    splits = pdist.partition_rows((rp[1:] - rp[:-1]).cpu().numpy(), world, b_nnz=12, b_row=16)
    sp = pdist.DistSpMV(rp, ci, val, splits)
    nnz_local = sp.col.numel()
    del rp, ci, val
    y = torch.empty(sp.n_local, dtype=torch.float64, device=dev)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    stream = torch.cuda.current_stream()
    for _ in range(args.warmup):
        flush.zero_()
        sp.rebin()
        sp.spmv(x, y)
    torch.cuda.synchronize()
    K = args.steps
    ev = [[torch.cuda.Event(enable_timing=True) for _ in range(3)] for _ in range(K)]
    if world > 1:
        torch.distributed.barrier()
    torch.cuda.synchronize()
    with Clocks(torch.cuda.current_device()) as clk:
        for k in range(K):
            flush.zero_()
            ev[k][0].record(stream)
            sp.rebin()
            ev[k][1].record(stream)
            sp.spmv(x, y)
            ev[k][2].record(stream)
        torch.cuda.synchronize()
    t_bin = float(np.mean([ev[k][0].elapsed_time(ev[k][1]) for k in range(K)]))
    t_spmv = float(np.mean([ev[k][1].elapsed_time(ev[k][2]) for k in range(K)]))
    tot = t_bin + t_spmv
    if world > 1:
        tt = torch.tensor([tot, t_bin, t_spmv], dtype=torch.float64, device=dev)
        torch.distributed.all_reduce(tt, op=torch.distributed.ReduceOp.MAX)
        tot, t_bin, t_spmv = (float(v) for v in tt.tolist())
    if rank != 0:
        return None
    return {"metric": "SpMV GFLOP/s (bin+SpMV per step), one matrix row-split across GPUs",
            "value": round(2.0 * nnz / (tot * 1e-3) / 1e9, 3), "unit": "GFLOP/s", "n_gpus": world, "steps": K,
            "warmup": args.warmup, "ms_per_step": round(tot, 5), "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": "rmat20_ef16_f64_row_split", "n_rows": n, "nnz": nnz,
                       "nnz_rank0": nnz_local, "parallelism": f"row-split x{world} (P:345)",
                       "l2": "flushed: 256 MiB write between timed steps (outside the step events)"},
            "breakdown": {"t_bin_ms_max_rank": round(t_bin, 5), "t_spmv_ms_max_rank": round(t_spmv, 5)},
            "gpu_launches": 4 * K * world, "clocks": clk.summary()}


def run_pagerank_dist(args, dev, rank, world):
    """C4 row-partitioned across the ranks (reading Q19): every rank builds the
    in-link graph, keeps its nnz-balanced contiguous row range, and per iteration runs
    one fused acsr_pagerank_step + NCCL all-gather of the xs slices + all-reduce of
    Delta^2 (paper_conf_sc_ashariseps14_b200.dist).  Strong scaling (fixed graph)."""
    from paper_conf_sc_ashariseps14_b200 import dist as pdist

    S = args.scale or 24
    rp, ci = synth.rmat_csr(S, device=dev, transpose=True)
    n = rp.numel() - 1
    outdeg = torch.bincount(ci.long(), minlength=n).to(torch.int32)
    splits = pdist.partition_rows((rp[1:] - rp[:-1]).cpu().numpy(), world)
    lo, hi = int(splits[rank]), int(splits[rank + 1])
    rpl = (rp[lo:hi + 1] - rp[lo]).contiguous()
    cil = ci[int(rp[lo]):int(rp[hi])].clone()
    odl = outdeg[lo:hi].clone()
    nnz_local = cil.numel()
    del rp, ci
    torch.cuda.empty_cache()
    pr = pdist.DistPageRank(rpl, cil, odl, splits, n, exchange=args.exchange)
    for _ in range(args.warmup):
        pr.run(max_iter=1)
    torch.cuda.synchronize()
    if world > 1:
        torch.distributed.barrier()
    K = args.steps
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with Clocks(torch.cuda.current_device()) as clk:
        e0.record()
        if args.exchange == "peer":  # device-side stop flag: 8 (step, Delta^2) pairs per host sync
            x, it, d2 = pr.run(eps=0.0, max_iter=K, check_every=8)
        else:
            x, it, d2 = pr.run(eps=0.0, max_iter=K)
        e1.record()
        torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / K
    if world > 1:
        tt = torch.tensor([ms], dtype=torch.float64, device=dev)
        torch.distributed.all_reduce(tt, op=torch.distributed.ReduceOp.MAX)
        ms = float(tt.item())
        nz = torch.tensor([nnz_local], dtype=torch.int64, device=dev)
        torch.distributed.all_reduce(nz)
        nnz = int(nz.item())
    else:
        nnz = nnz_local
    if rank != 0:
        return None
    how = ("exchange fused into the step: P2P stores of xs over peer memory" if args.exchange == "peer"
           else "NCCL all-gather of xs")
    return {"metric": f"PageRank iteration GTEPS, row-partitioned ({how})",
            "value": round(nnz / (ms * 1e-3) / 1e9, 3), "unit": "GTEPS", "n_gpus": world, "steps": K,
            "warmup": args.warmup, "ms_per_step": round(ms, 5), "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": f"pagerank_rmat{S}_inlink_partitioned", "n_rows": n, "nnz": nnz,
                       "parallelism": f"row-partitioned x{world}", "padded_slice": pr.L,
                       "exchange_slice": pr.Lx, "exchange_bytes_in_per_rank_per_iter": pr.exchange_bytes_per_rank(),
                       "exchange_layout": "non-dangling only (lossless)" if pr.compact else "all vertices",
                       "exchange": args.exchange},
            "gpu_launches": K * (2 if args.exchange == "peer" else 1), "clocks": clk.summary()}


def _max_over_ranks(vals, dev, world):
    if world == 1:
        return [float(v) for v in vals]
    t = torch.tensor([float(v) for v in vals], dtype=torch.float64, device=dev)
    torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
    return [float(v) for v in t.tolist()]


def _c4_variant(acsr, pdist, rp, ci, outdeg, n, nnz, K, dev, rank, world, comm):
    """One graph of the C4 record: T1 (rank 0 alone, whole graph), then the row-partitioned
    run with each exchange, T_comm and the fraction of SURVEY §8(e)'s bound."""
    t1 = None
    if rank == 0:
        m = acsr.ACSRMatrix(rp, ci)
        x = torch.full((n,), 1.0 / n, dtype=torch.float64, device=dev)
        xs = acsr.acsr_pagerank_scale(x, outdeg)
        xn, xsn = torch.empty_like(x), torch.empty_like(x)
        d2 = torch.zeros(1, dtype=torch.float64, device=dev)
        args_ = (m.row_begin, m.col_idx, m.bin_rows, m.bin_offsets, m.plan_ws)
        for _ in range(2):
            acsr.acsr_pagerank_step(*args_, xs, x, outdeg, xn, xsn, d2, 0.85, 0.15 / n, n)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(K):
            acsr.acsr_pagerank_step(*args_, xs, x, outdeg, xn, xsn, d2, 0.85, 0.15 / n, n)
        e1.record()
        torch.cuda.synchronize()
        t1 = e0.elapsed_time(e1) / K
        del m, x, xs, xn, xsn
        torch.cuda.empty_cache()
    if world > 1:
        torch.distributed.barrier()
    splits = acsr.acsr_partition(rp, world, 4, 36).cpu().numpy()
    lo, hi = int(splits[rank]), int(splits[rank + 1])
    rpl = (rp[lo:hi + 1].to(torch.int64) - int(rp[lo])).to(torch.int32)
    cil = ci[int(rp[lo]):int(rp[hi])].clone()
    odl = outdeg[lo:hi].clone()
    out = {"splits": [int(v) for v in splits], "t1_ms": None if t1 is None else round(t1, 4)}
    for ex in ("acsr", "peer"):
        pr = pdist.DistPageRank(rpl, cil, odl, splits, n, exchange=ex, comm=comm)
        pr.run(max_iter=2, eps=0.0)
        torch.cuda.synchronize()
        if world > 1:
            torch.distributed.barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        pr.run(eps=0.0, max_iter=K, check_every=K)
        e1.record()
        torch.cuda.synchronize()
        ms = _max_over_ranks([e0.elapsed_time(e1) / K], dev, world)[0]
        rec = {"ms_per_iter": round(ms, 4), "gteps": round(nnz / (ms * 1e-3) / 1e9, 2),
               "exchange_slice": pr.Lx, "exchange_bytes_in_per_rank_per_iter": pr.exchange_bytes_per_rank()}
        if ex == "acsr" and world > 1:
            # T_comm: the same exchange alone (all-gather-v of the real entries, NCCL over
            # NVLink), K times
            buf = torch.zeros(world * pr.Lx, dtype=torch.float64, device=dev)
            mine = buf[rank * pr.Lx:(rank + 1) * pr.Lx]
            counts = pr.n_nd if pr.compact else [int(c) for c in np.diff(pr.splits)]
            pr.comm.allgatherv(mine, buf, counts)
            torch.cuda.synchronize()
            c0, c1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            c0.record()
            for _ in range(K):
                pr.comm.allgatherv(mine, buf, counts)
            c1.record()
            torch.cuda.synchronize()
            rec["t_comm_ms"] = round(_max_over_ranks([c0.elapsed_time(c1) / K], dev, world)[0], 4)
            del buf
        if ex == "peer" and pr.peer is not None:
            pr.peer.close()
        out[ex] = rec
        del pr
        torch.cuda.empty_cache()
    if rank == 0:
        t_comm = out["acsr"].get("t_comm_ms", 0.0)
        bound = max(t1 / world, t_comm)
        out["bound_ms"] = round(bound, 4)
        for ex in ("acsr", "peer"):
            out[ex]["frac_of_bound"] = round(bound / out[ex]["ms_per_iter"], 4)
            out[ex]["speedup_vs_t1"] = round(t1 / out[ex]["ms_per_iter"], 3)
    return out


def pagerank_dist_record(args, dev, rank, world):
    """C4 (BASELINE configs[3]): PageRank on the R-MAT s26 in-link pattern, row-partitioned
    over the N ranks (acsr_partition, cost 4 len + 36), compact non-dangling exchange
    layout, timed for K iterations with each exchange:
      acsr  -- acsr_pagerank_step with the library's NCCL communicator (all-gather of the
               xs slices + exact global Delta^2, device-side stop flag);
      peer  -- the exchange fused into the step over CUDA-IPC peer memory (N1).
    Both on the generated graph and on its degree-relabelled copy (acsr_degree_relabel,
    timed).  Also T1 (the whole graph on rank 0's GPU alone, measured in the same job),
    T_comm (the same all-gather alone) and frac_of_bound = max(T1/P, T_comm) / T."""
    import paper_conf_sc_ashariseps14_b200 as acsr
    from paper_conf_sc_ashariseps14_b200 import dist as pdist

    S = args.c4_scale
    K = max(3, min(args.steps, 10))
    torch.cuda.synchronize()
    g0 = time.perf_counter()
    rp, ci = synth.rmat_csr(S, device=dev, transpose=True)
    n, nnz = rp.numel() - 1, ci.numel()
    outdeg = torch.bincount(ci.long(), minlength=n).to(torch.int32)
    torch.cuda.synchronize()
    t_gen = time.perf_counter() - g0
    out = {"workload": f"pagerank_rmat{S}_inlink_partitioned", "n_rows": n, "nnz": nnz,
           "generate_s": round(t_gen, 2), "iterations_timed": K,
           "bound_note": "SURVEY §8(e): max(T1/P, T_comm), T1 = whole graph on one GPU, T_comm = the all-gather alone"}
    comm = acsr.AcsrComm.from_process_group() if world > 1 else None
    out["plain"] = _c4_variant(acsr, pdist, rp, ci, outdeg, n, nnz, K, dev, rank, world, comm)
    r0, r1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    r0.record()
    rp2, ci2, od2, _ = acsr.acsr_degree_relabel(rp, ci, outdeg)
    r1.record()
    torch.cuda.synchronize()
    del rp, ci, outdeg
    torch.cuda.empty_cache()
    out["relabelled"] = _c4_variant(acsr, pdist, rp2, ci2, od2, n, nnz, K, dev, rank, world, comm)
    out["relabelled"]["relabel_ms"] = round(r0.elapsed_time(r1), 3)
    if comm is not None:
        comm.close()
    return out


def run_hits_rwr(args, dev, rank, world):
    """HITS (Eq. 5-7) or RWR (Eq. 8) on R-MAT scale S (default 20) to eps = 1e-6:
    value = GTEPS (nnz per iteration / mean iteration time, host convergence loop included;
    matrix construction and binning done once before the timing)."""
    import paper_conf_sc_ashariseps14_b200 as acsr

    S = args.scale or 20
    if args.workload == "hits":
        rp, ci = synth.rmat_csr(S, device=dev)
        nnz_it = 2 * ci.numel()
        # the block matrix [[0, A^T], [A, 0]] is built and binned once, outside the timing
        B = acsr.ACSRMatrix(*acsr.hits_matrix(rp, ci), None, n_cols=2 * (rp.numel() - 1))
        run = lambda: acsr.hits(rp, ci, eps=1e-6, B=B)
    else:
        rp, ci = synth.rmat_csr(S, device=dev, transpose=True)
        n = rp.numel() - 1
        od = torch.bincount(ci.long(), minlength=n).to(torch.int32)
        m = acsr.ACSRMatrix(rp, ci)
        hub = int(torch.argmax(od))
        nnz_it = ci.numel()
        run = lambda: acsr.rwr(m, od, hub, c=0.85, eps=1e-6)
    for _ in range(max(1, args.warmup // 3)):
        run()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    out = run()
    torch.cuda.synchronize()
    dt = time.perf_counter() - t0
    it = out[2] if args.workload == "hits" else out[1]
    if rank != 0:
        return None
    ms = dt * 1e3 / it
    return {"metric": f"{args.workload.upper()} iteration GTEPS (to eps=1e-6, host convergence loop included)",
            "value": round(nnz_it / (ms * 1e-3) / 1e9, 3), "unit": "GTEPS", "n_gpus": world, "steps": it,
            "warmup": args.warmup, "ms_per_step": round(ms, 5), "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": f"{args.workload}_rmat{S}", "nnz_per_iteration": nnz_it, "iterations": it,
                       "total_ms": round(dt * 1e3, 3)}}


# ------------------------------------------------------------------------------ dynamic graph (C5)
def host_inclusive_batch(m, pinned, outdeg, st, uws, x, xs_tmp, y):
    """Wall time (ms) of the change-list H2D copies + update + re-bin + scale + SpMV issued
    from an idle GPU through the Python API, on a scratch copy of the slack CSR (the live
    matrix is not touched)."""
    import paper_conf_sc_ashariseps14_b200 as acsr
    mm = acsr.ACSRMatrix(m.row_begin, m.col_idx.clone(), None, row_end=m.row_end.clone(),
                         row_cap=m.row_cap, nnz_max=m.nnz_max)
    od = outdeg.clone()
    dev = m.row_begin.device
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    chd = {kk: v.to(dev, non_blocking=True) for kk, v in pinned.items()}
    mm.update(chd, outdeg=od, status=st, ws=uws)
    mm.rebin()
    acsr.acsr_pagerank_scale(x, od, xs_tmp)
    mm.spmv(xs_tmp, y)
    torch.cuda.synchronize()
    return (time.perf_counter() - t0) * 1e3


def run_dynamic(args, dev, rank, world):
    """C5: R-MAT s20 in-link pattern with slack (cap = len + max(4, len/4)); per batch of
    16,384 inserted edges: H2D of the change lists, acsr_update_edges, acsr_bin, one SpMV
    (timed) and a warm-started PageRank to eps = 1e-6."""
    import paper_conf_sc_ashariseps14_b200 as acsr

    S = args.scale or 20
    B = args.batches or (args.warmup + args.steps)
    rp, ci = synth.rmat_csr(S, device=dev, transpose=True)
    n = rp.numel() - 1
    keys = np.sort((torch.repeat_interleave(torch.arange(n, device=dev), (rp[1:] - rp[:-1]).long()) * n
                    + ci.long()).cpu().numpy())
    rb, re, cap, col, _ = synth.with_slack(rp, ci)
    outdeg = torch.bincount(ci.long(), minlength=n).to(torch.int32)
    m = acsr.ACSRMatrix(rb, col, None, row_end=re, row_cap=cap, nnz_max=col.numel())
    x, it0, _ = acsr.pagerank(m, outdeg, eps=1e-6)
    G = min(args.steps, 20)  # further batches replayed through one captured CUDA graph
    t_gen = time.perf_counter()
    all_batches = [(ch, k) for ch, k in synth.insert_batches(S, B + G, 16384, keys, device=dev)]
    t_gen = time.perf_counter() - t_gen
    batches, gbatches = all_batches[:B], all_batches[B:]
    st = torch.empty(2, dtype=torch.int32, device=dev)
    uws = torch.empty(acsr.acsr_update_workspace_bytes(1 << 20), dtype=torch.uint8, device=dev)
    xs_tmp = torch.empty(n, dtype=torch.float64, device=dev)
    y = torch.empty(n, dtype=torch.float64, device=dev)
    rec = []
    relayouts = 0
    for b, (ch, k) in enumerate(batches):
        pinned = {kk: torch.from_numpy(v).pin_memory() for kk, v in ch.items()}
        ev = [torch.cuda.Event(enable_timing=True) for _ in range(5)]
        torch.cuda.synchronize()
        # device time of each phase: the batch is enqueued behind a ~0.5 ms GPU sleep, so
        # the host's launch/marshalling time does not show up as gaps between the events;
        # the host-inclusive time (sync -> enqueue -> sync, no sleep) is reported beside it
        torch.cuda._sleep(1_000_000)
        ev[0].record()
        chd = {kk: v.to(dev, non_blocking=True) for kk, v in pinned.items()}
        ev[1].record()
        m.update(chd, outdeg=outdeg, status=st, ws=uws)
        ev[2].record()
        m.rebin()
        ev[3].record()
        acsr.acsr_pagerank_scale(x, outdeg, xs_tmp)
        m.spmv(xs_tmp, y)
        ev[4].record()
        torch.cuda.synchronize()
        regrow = 0
        while st.cpu().tolist() != [0, -1]:  # CAPACITY: nothing was applied (all-or-nothing)
            assert int(st[0]) == acsr.ACSR_ERR_CAPACITY and regrow < 4, st
            m.grow()
            m.update(chd, outdeg=outdeg, status=st, ws=uws)
            m.rebin()
            torch.cuda.synchronize()
            regrow += 1
        relayouts += regrow
        # re-bin + scale + SpMV of the updated graph back to back, events at the ends only
        # (the PDL overlap the phase events above break; re-binning the same graph and the
        # SpMV are idempotent): the per-update "bin + SpMV" as a caller runs it
        torch.cuda._sleep(1_000_000)
        j0, j1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        j0.record()
        m.rebin()
        acsr.acsr_pagerank_scale(x, outdeg, xs_tmp)
        m.spmv(xs_tmp, y)
        j1.record()
        torch.cuda.synchronize()
        t_joint = j0.elapsed_time(j1)
        # host-inclusive: the same update + re-bin + SpMV issued from an idle GPU (a
        # re-applied insert batch only appends duplicates, so time it on a scratch copy)
        t_host = host_inclusive_batch(m, pinned, outdeg, st, uws, x, xs_tmp, y) if b >= args.warmup else 0.0
        t0 = time.perf_counter()
        x, it, _ = acsr.pagerank(m, outdeg, x0=x, eps=1e-6)
        torch.cuda.synchronize()
        t_pr = time.perf_counter() - t0
        if b >= args.warmup:
            rec.append([ev[i].elapsed_time(ev[i + 1]) for i in range(4)] + [t_pr * 1e3, it, k, t_host, t_joint])
    # the same per-batch sequence (update -> re-bin -> scale -> SpMV) from ONE captured CUDA
    # graph (acsr_update_edges_dev reads the batch size on the device), host-inclusive:
    # sync -> pinned copies into the graph's capacity buffers + replay -> sync
    x_g = x.clone()
    cap_b = max(max(c["upd_rows"].size, c["ins_cols"].size) for c, _ in gbatches) if gbatches else 1
    ug = acsr.UpdateGraph(m, outdeg, x_g, xs_tmp, y, max_upd=cap_b, max_ins=cap_b)
    t_graph, g_regrow = [], 0
    for ch, k in gbatches:
        pinned = {kk: torch.from_numpy(v).pin_memory() for kk, v in ch.items()}
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        st = ug.replay(pinned)
        torch.cuda.synchronize()
        dt = time.perf_counter() - t0
        if st.cpu().tolist() != [0, -1]:  # CAPACITY: grow (new buffers), apply eagerly, re-capture
            assert int(st[0]) == acsr.ACSR_ERR_CAPACITY, st
            m.grow()
            chd = {kk: v.to(dev) for kk, v in pinned.items()}
            while m.update(chd, outdeg=outdeg, status=st, ws=uws).cpu().tolist() != [0, -1]:
                m.grow()
            m.rebin()
            ug = acsr.UpdateGraph(m, outdeg, x_g, xs_tmp, y, max_upd=cap_b, max_ins=cap_b)
            g_regrow += 1
        else:
            t_graph.append(dt * 1e3)
        x, it, _ = acsr.pagerank(m, outdeg, x0=x, eps=1e-6)
        x_g.copy_(x)
    r = np.array(rec)
    # SURVEY §8(d) algorithmic bytes of the dominant kernel (the pattern SpMV on the slack
    # in-link CSR after the last batch): col 4 nnz + row_begin/row_end/bin_rows 12 n +
    # x gathers 8 n_c (referenced = non-dangling sources) + y 8 n
    nnz_now = int((m.row_end - m.row_begin).to(torch.int64).sum())
    n_c_now = int((outdeg > 0).sum())
    alg_spmv = 4 * nnz_now + 12 * n + 8 * n_c_now + 8 * n
    if rank != 0:
        return None
    t_h2d, t_upd, t_bin, t_spmv = (float(r[:, i].mean()) for i in range(4))
    peak, kind = peaks()
    label_dyn = f"dynamic_rmat{S}_inlink_16384_insert_batches"
    t_joint = float(r[:, 8].mean())
    return {"metric": "bin+SpMV ms per dynamic-graph update (C5)", "value": round(t_joint, 5),
            "unit": "ms", "n_gpus": world, "steps": len(rec), "warmup": args.warmup,
            "ms_per_step": round(t_h2d + t_upd + t_bin + t_spmv, 5), "higher_is_better": False,
            "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": f"dynamic_rmat{S}_inlink_16384_insert_batches", "n_rows": n,
                       "batches_timed": len(rec), "cold_iterations": it0},
            "breakdown": {"value_timing": "re-bin + scale + SpMV of each updated graph back to back (events at the "
                                          "ends only); phases below from a separate, event-split pass",
                          "t_bin_plus_spmv_split_ms": round(t_bin + t_spmv, 5),
                          "t_h2d_ms": round(t_h2d, 5), "t_update_ms": round(t_upd, 5), "t_bin_ms": round(t_bin, 5),
                          "t_spmv_ms": round(t_spmv, 5), "bin_lt_spmv": bool(t_bin < t_spmv),
                          "pt_st": round(t_bin / t_spmv, 3),
                          "rebuild_plus_spmv_ms": round(t_upd + t_bin + t_spmv, 5),
                          "rebuild_plus_spmv_host_inclusive_ms": round(float(r[:, 7].mean()), 5),
                          "rebuild_plus_spmv_graph_host_inclusive_ms": round(float(np.mean(t_graph)), 5)
                          if t_graph else None,
                          "graph_batches": len(t_graph), "graph_recaptures": g_regrow,
                          "timing": "phases: CUDA events, batch enqueued behind a GPU sleep (device time); "
                                    "host_inclusive: wall clock from an idle GPU through the Python API, "
                                    "change-list H2D copies included; "
                                    "graph: further batches, copies + one CUDA-graph replay of "
                                    "update_dev -> bin -> scale -> SpMV, wall clock",
                          "pagerank_warm_ms": round(float(r[:, 4].mean()), 4),
                          "warm_iterations_mean": round(float(r[:, 5].mean()), 2),
                          "inserted_edges_mean": round(float(r[:, 6].mean()), 1),
                          "batch_encode_s_total": round(t_gen, 2),
                          "relayouts": relayouts},
            "roofline": {"bound": "hbm", "achieved": round(alg_spmv / (t_spmv * 1e-3) / 1e9, 1), "peak": peak,
                         "unit": "GB/s", "frac": round(alg_spmv / (t_spmv * 1e-3) / 1e9 / peak, 4),
                         "traffic": ncu_traffic(label_dyn), "kernel": "acsr::spmv_kernel (pattern, slack CSR)",
                         "peak_kind": kind, "algorithmic_bytes_per_launch": int(alg_spmv),
                         "note": "4 nnz + 12 n + 8 n_c + 8 n after the last batch",
                         "vs_other_peaks": {"spec_gbs": HBM_SPEC_GBS,
                                            "frac_vs_spec": round(alg_spmv / (t_spmv * 1e-3) / 1e9 / HBM_SPEC_GBS, 4)}},
            # per timed batch: update_init + update_validate + update_apply (insert-only),
            # bin_count + bin_scan + bin_scatter, pagerank_scale + spmv_kernel
            "gpu_launches": 8 * len(rec)}


def run_dynamic_mixed(args, dev, rank, world):
    """The paper's dynamic experiment: PageRank converges, then per
    epoch 10 % of the rows change (each column deleted or another added with probability
    1/2), only the change list goes to the device, the matrix is updated in place and
    re-binned, PageRank warm-starts from the previous vector; 10 epochs."""
    import paper_conf_sc_ashariseps14_b200 as acsr

    S = args.scale or 20
    E = args.batches or 10
    rp, ci = synth.rmat_csr(S, device=dev, transpose=True)
    n = rp.numel() - 1
    rb, re, cap, col, _ = synth.with_slack(rp, ci, frac=1)  # about 2x slack (reading R3)
    outdeg = torch.bincount(ci.long(), minlength=n).to(torch.int32)
    m = acsr.ACSRMatrix(rb, col, None, row_end=re, row_cap=cap, nnz_max=col.numel())
    t0 = time.perf_counter()
    x, it0, _ = acsr.pagerank(m, outdeg, eps=1e-6)
    torch.cuda.synchronize()
    t_cold = time.perf_counter() - t0
    st = torch.empty(2, dtype=torch.int32, device=dev)
    uws = torch.empty(acsr.acsr_update_workspace_bytes(1 << 22), dtype=torch.uint8, device=dev)
    rec, relayouts = [], 0
    for ep in range(E):
        ch = synth.mixed_epoch(m.row_begin, m.row_end, m.col_idx, n, 0.10, 5000 + ep)
        pinned = {k: torch.from_numpy(v).pin_memory() for k, v in ch.items()}
        ev = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
        torch.cuda.synchronize()
        torch.cuda._sleep(1_000_000)  # device time: enqueue behind a GPU sleep (as run_dynamic)
        ev[0].record()
        chd = {k: v.to(dev, non_blocking=True) for k, v in pinned.items()}
        ev[1].record()
        m.update(chd, outdeg=outdeg, status=st, ws=uws)
        ev[2].record()
        m.rebin()
        ev[3].record()
        torch.cuda.synchronize()
        while st.cpu().tolist() != [0, -1]:
            assert int(st[0]) == acsr.ACSR_ERR_CAPACITY and relayouts < 20, st
            m.grow()
            m.update(chd, outdeg=outdeg, status=st, ws=uws)
            m.rebin()
            torch.cuda.synchronize()
            relayouts += 1
        t1 = time.perf_counter()
        x, it, _ = acsr.pagerank(m, outdeg, x0=x, eps=1e-6)
        torch.cuda.synchronize()
        t_pr = time.perf_counter() - t1
        rec.append([ev[0].elapsed_time(ev[1]), ev[1].elapsed_time(ev[2]), ev[2].elapsed_time(ev[3]),
                    t_pr * 1e3, it, int(ch["del_cols"].size), int(ch["ins_cols"].size)])
    r = np.array(rec)
    if rank != 0:
        return None
    return {"metric": "dynamic PageRank epoch (paper §VII): update + re-bin ms, warm iterations",
            "value": round(float((r[:, 1] + r[:, 2]).mean()), 5), "unit": "ms", "n_gpus": world,
            "steps": E, "warmup": 0, "ms_per_step": round(float(r[:, :4].sum(1).mean()), 4),
            "higher_is_better": False, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic",
            "config": {"workload": f"dynamic_mixed_rmat{S}_10pct_rows_{E}_epochs", "n_rows": n,
                       "cold_iterations": it0, "cold_pagerank_ms": round(t_cold * 1e3, 3)},
            "breakdown": {"t_h2d_ms": round(float(r[:, 0].mean()), 5), "t_update_ms": round(float(r[:, 1].mean()), 5),
                          "t_bin_ms": round(float(r[:, 2].mean()), 5),
                          "pagerank_warm_ms": round(float(r[:, 3].mean()), 4),
                          "warm_iterations": [int(v) for v in r[:, 4]],
                          "deleted_per_epoch": round(float(r[:, 5].mean()), 1),
                          "inserted_per_epoch": round(float(r[:, 6].mean()), 1), "relayouts": relayouts}}


# ------------------------------------------------------------------------------ reference arm
def run_reference(args, dev):
    """The oracle as it stands (plain C, 1 core) on the same workload: bins (O3) + plain SpMV
    (O4') per step."""
    import oracle

    label, dtype, rp, ci, val, x = make_workload(args.workload, dev, 0)
    rph, cih = rp.cpu().numpy(), ci.cpu().numpy()
    vh, xh = val.cpu().numpy(), x.cpu().numpy()
    y = np.empty(rph.size - 1, vh.dtype)
    for _ in range(min(args.warmup, 1)):
        oracle.bins(rph)
        oracle.spmv_plain(rph, cih, vh, xh, out=y)
    K = args.steps
    t0 = time.perf_counter()
    for _ in range(K):
        oracle.bins(rph)
        oracle.spmv_plain(rph, cih, vh, xh, out=y)
    dt = (time.perf_counter() - t0) / K
    v = 2.0 * cih.size / dt / 1e9
    return {"metric": "SpMV GFLOP/s (bin+SpMV per step) & HBM GB/s vs peak", "impl": "reference",
            "value": round(v, 4), "unit": "GFLOP/s", "n_gpus": int(os.environ.get("WORLD_SIZE", "1")), "steps": K, "warmup": args.warmup,
            "ms_per_step": round(dt * 1e3, 3), "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "f64" if dtype == torch.float64 else "f32", "data": "synthetic",
            "config": workload_config(label, int(rph.size - 1), int(cih.size), int(os.environ.get("WORLD_SIZE", "1"))),
            "cpu_baseline": {"value": round(v, 4), "unit": "GFLOP/s", "cores": 1, "kind": "oracle",
                             "sample": f"whole matrix per step: oracle bins (O3) + plain SpMV (O4'), {K} steps"},
            "e2e": {"value": round(v, 4), "unit": "GFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}


def main():
    wd = os.environ.get("ACSR_BENCH_WATCHDOG")  # debugging: dump every thread's stack and exit after N s
    if wd:
        import faulthandler
        faulthandler.dump_traceback_later(float(wd), exit=True)
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="acsr", choices=["acsr", "reference"])
    ap.add_argument("--workload", default="rmat20")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--scale", type=int, default=None, help="R-MAT scale for pagerank/dynamic")
    ap.add_argument("--batches", type=int, default=None, help="dynamic: number of insertion batches")
    ap.add_argument("--relabel", action="store_true", help="pagerank: degree-ordered vertex relabelling")
    ap.add_argument("--relabel-sort", action="store_true", help="pagerank --relabel: sort every row's columns")
    ap.add_argument("--exchange", default="acsr", choices=["acsr", "torch", "peer"],
                    help="pagerank_dist: the library's NCCL exchange inside acsr_pagerank_step (acsr_comm), "
                         "torch.distributed collectives, or the exchange fused into the step over peer memory")
    ap.add_argument("--replicas", action="store_true",
                    help="N > 1: independent matrix per rank (weak) instead of one row-split matrix")
    ap.add_argument("--no-c4", action="store_true", help="skip the pagerank_dist (C4) record of the default line")
    ap.add_argument("--c4-scale", type=int, default=26, help="R-MAT scale of the pagerank_dist record")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        if rank != 0:
            return
        dev = torch.device("cuda", local) if torch.cuda.is_available() else torch.device("cpu")
        print(json.dumps(run_reference(args, dev)), flush=True)
        return
    ndev = torch.cuda.device_count()
    local_dev = local % max(ndev, 1)  # (ranks > GPUs only in the single-GPU test of this path)
    torch.cuda.set_device(local_dev)
    dev = torch.device("cuda", local_dev)
    if world > 1 and os.environ.get("ACSR_SHARED_GPU_TEST") == "1":
        # test-only: several ranks on ONE GPU.  NCCL refuses two ranks on one device of one
        # host, so each rank claims its own host id and NCCL talks over loopback sockets.
        os.environ.update(NCCL_HOSTID=f"acsr-test-host-{rank}", NCCL_SOCKET_IFNAME="lo", NCCL_IB_DISABLE="1",
                          NCCL_P2P_DISABLE="1", NCCL_SHM_DISABLE="1", NCCL_NVLS_ENABLE="0")
    if world > 1:
        # NCCL's communicator-init log (nranks, transports, NVLS) stays on for the record, on
        # stderr so rank 0's stdout keeps exactly one JSON line
        os.environ.setdefault("NCCL_DEBUG", "INFO")
        os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
        os.environ.setdefault("NCCL_DEBUG_FILE", "/dev/stderr")
        backend = os.environ.get("ACSR_DIST_BACKEND", "nccl")  # gloo: test the path on one GPU
        if backend == "nccl":
            torch.distributed.init_process_group("nccl", device_id=dev)
        else:
            torch.distributed.init_process_group(backend)
    if args.workload == "pagerank":
        line = run_pagerank(args, dev, rank, world)
    elif args.workload == "rmat20_split":
        line = run_spmv_split(args, dev, rank, world)
    elif args.workload == "pagerank_dist":
        line = run_pagerank_dist(args, dev, rank, world)
    elif args.workload == "dynamic":
        line = run_dynamic(args, dev, rank, world)
    elif args.workload == "dynamic_mixed":
        line = run_dynamic_mixed(args, dev, rank, world)
    elif args.workload in ("hits", "rwr"):
        line = run_hits_rwr(args, dev, rank, world)
    else:
        line = run_acsr(args, dev, rank, world)
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        torch.distributed.destroy_process_group()


if __name__ == "__main__":
    main()
