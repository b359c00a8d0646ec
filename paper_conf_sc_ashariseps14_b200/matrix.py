"""Convenience objects over the C ABI (argument marshalling only).

``ACSRMatrix`` owns a (possibly slack) CSR on the device together with its bins and
plan workspace; ``spmv_from_host`` is the end-to-end path a user with host arrays
takes (pinned H2D copies, bin, SpMV, D2H); ``pagerank`` is the single-GPU Alg. 5 loop
 with the convergence test of reading Q9.
"""
from __future__ import annotations

import torch

from . import (ACSR_CTRL_PLAN_ERROR, acsr_bin, acsr_bin_workspace_bytes, acsr_hits_normalize,
               acsr_hits_workspace_bytes, acsr_pagerank_scale, acsr_pagerank_step, acsr_plan_status, acsr_relayout,
               acsr_spmv, acsr_update_edges, acsr_update_workspace_bytes)


class ACSRMatrix:
    """Device CSR + ACSR bins.  row_end None => standard CSR (row_begin has n+1 entries)."""

    def __init__(self, row_begin, col_idx, values=None, n_cols=None, row_end=None, row_cap=None,
                 nnz_max=None, short_rows="window"):
        self.short_rows = short_rows  # SpMV mapping of bins 0..5: "window" or "alg2" (acsr_bin_ex)
        self.row_begin = row_begin
        self.row_end = row_end
        self.row_cap = row_cap
        self.col_idx = col_idx
        self.values = values
        self.n_rows = row_begin.numel() - 1 if row_end is None else row_begin.numel()
        self.n_cols = self.n_rows if n_cols is None else n_cols
        self.nnz_max = col_idx.numel() if nnz_max is None else nnz_max
        dev = row_begin.device
        self.bin_rows = torch.empty(self.n_rows, dtype=torch.int32, device=dev)
        self.bin_offsets = torch.empty(33, dtype=torch.int32, device=dev)
        self.plan_ws = torch.empty(acsr_bin_workspace_bytes(self.n_rows, self.n_cols, self.nnz_max),
                                   dtype=torch.uint8, device=dev)
        self.rebin()

    def rebin(self, stream=None):
        acsr_bin(self.row_begin, self.row_end, self.nnz_max, self.bin_rows, self.bin_offsets,
                 self.plan_ws, stream, col_idx=self.col_idx, n_cols=self.n_cols, short_rows=self.short_rows)

    def plan_status(self, stream=None):
        """Synchronising check that the plan is valid (raises ACSRError otherwise)."""
        acsr_plan_status(self.plan_ws, stream)

    def spmv(self, x, y=None, stream=None):
        return acsr_spmv(self.row_begin, self.col_idx, self.values, x, self.bin_rows,
                         self.bin_offsets, self.plan_ws, self.row_end, y, stream)

    def update(self, changes, outdeg=None, ins_vals=None, status=None, ws=None, stream=None, n_upd_dev=None):
        """changes: dict of CUDA int32 tensors upd_rows, ins_ptr, ins_cols[, del_ptr, del_cols].
        n_upd_dev: device batch size (the tensors are then capacity buffers; graph-capturable)."""
        assert self.row_end is not None and self.row_cap is not None, "update needs slack CSR"
        return acsr_update_edges(self.n_cols, self.row_begin, self.row_end, self.row_cap,
                                 self.col_idx, self.values, changes["upd_rows"], changes["ins_ptr"],
                                 changes["ins_cols"], ins_vals, changes.get("del_ptr"),
                                 changes.get("del_cols"), outdeg, status, ws, stream=stream, n_upd_dev=n_upd_dev)

    def grow(self, min_slack=8, frac=2, stream=None):
        """Re-lay the slack CSR out with more room (reading R4: after a CAPACITY rejection):
        cap_r <- max(cap_r + max(min_slack, ceil(cap_r / frac)), len_r + max(min_slack,
        ceil(len_r / frac))) -- every row grows, so repeated rejections always progress.
        Then re-bin."""
        assert self.row_end is not None
        from . import acsr_grow_layout
        new_begin, cap, total = acsr_grow_layout(self.row_begin, self.row_end, self.row_cap, min_slack, frac,
                                                 stream=stream)
        if total >= 2 ** 31:
            raise OverflowError("grown slack CSR exceeds int32 indices")
        dev = self.row_begin.device
        new_end = torch.empty_like(new_begin)
        new_col = torch.full((max(total, 1),), -1, dtype=torch.int32, device=dev)
        new_val = None if self.values is None else torch.zeros(max(total, 1), dtype=self.values.dtype,
                                                               device=dev)
        acsr_relayout(self.row_begin, self.row_end, self.col_idx, self.values, new_begin, new_end, new_col,
                      new_val, stream=stream)
        self.row_begin, self.row_end, self.row_cap = new_begin, new_end, cap
        self.col_idx, self.values = new_col, new_val
        if total > self.nnz_max:
            self.nnz_max = total
            self.plan_ws = torch.empty(acsr_bin_workspace_bytes(self.n_rows, self.n_cols, self.nnz_max),
                                       dtype=torch.uint8, device=dev)
        self.rebin(stream)


class UpdateGraph:
    """The C5 per-batch device sequence -- acsr_update_edges_dev -> acsr_bin ->
    acsr_pagerank_scale -> acsr_spmv -- captured ONCE into a CUDA graph and
    replayed for every insert-only batch: the change lists are copied into fixed capacity
    buffers and the batch size into a device int64 (the update reads it there), so one
    graph serves batches of any size up to the capacities.  Pointers are baked in: build a
    new UpdateGraph after m.grow().  After replay(), self.status holds the update status and
    y = A xs with xs = x / outdeg of the updated graph."""

    def __init__(self, m: ACSRMatrix, outdeg, x, xs, y, max_upd: int, max_ins: int):
        dev = m.row_begin.device
        self.max_upd, self.max_ins = int(max_upd), int(max_ins)
        self.n_dev = torch.zeros(1, dtype=torch.int64, device=dev)
        self.n_host = torch.zeros(1, dtype=torch.int64).pin_memory()
        self.bufs = {"upd_rows": torch.zeros(self.max_upd, dtype=torch.int32, device=dev),
                     "ins_ptr": torch.zeros(self.max_upd + 1, dtype=torch.int32, device=dev),
                     "ins_cols": torch.zeros(self.max_ins, dtype=torch.int32, device=dev)}
        self.status = torch.zeros(2, dtype=torch.int32, device=dev)
        self.ws = torch.empty(acsr_update_workspace_bytes(self.max_upd), dtype=torch.uint8, device=dev)
        self._h2d_done = None  # event after the last replay's H2D copies
        self._pending = None   # the last replay's host change lists (alive until copied)

        def seq():
            m.update(self.bufs, outdeg=outdeg, status=self.status, ws=self.ws, n_upd_dev=self.n_dev)
            m.rebin()
            acsr_pagerank_scale(x, outdeg, xs)
            m.spmv(xs, y)

        self.n_dev.zero_()
        seq()  # eager once with an empty batch: lazy kernel attributes are set outside the capture
        torch.cuda.synchronize()
        self.graph = torch.cuda.CUDAGraph()
        with torch.cuda.graph(self.graph):
            seq()

    def replay(self, changes_host):
        """changes_host: dict of pinned host int32 tensors upd_rows, ins_ptr, ins_cols.
        The H2D copies are asynchronous: the pinned batch size this object writes is only
        rewritten after the previous replay's copies have executed (an event), and the
        caller's change tensors are kept referenced until the next replay, so several
        replays may be enqueued without a synchronisation."""
        n = changes_host["upd_rows"].numel()
        k = changes_host["ins_cols"].numel()
        if n > self.max_upd or k > self.max_ins:
            raise ValueError("batch exceeds the UpdateGraph capacities")
        if self._h2d_done is not None:
            self._h2d_done.synchronize()  # the previous DMA has read n_host (and its lists)
        self.bufs["upd_rows"][:n].copy_(changes_host["upd_rows"], non_blocking=True)
        self.bufs["ins_ptr"][:n + 1].copy_(changes_host["ins_ptr"], non_blocking=True)
        self.bufs["ins_cols"][:k].copy_(changes_host["ins_cols"], non_blocking=True)
        self.n_host[0] = n
        self.n_dev.copy_(self.n_host, non_blocking=True)
        self._h2d_done = torch.cuda.Event()
        self._h2d_done.record()
        self._pending = changes_host
        self.graph.replay()
        return self.status


def spmv_from_host(row_ptr_h, col_h, val_h, x_h, y_h=None, device="cuda", stream=None):
    """End-to-end y = A x from (pinned) host arrays: H2D, acsr_bin, acsr_spmv, D2H, all
    enqueued on `stream` (default: the current stream).  Calls on different streams
    overlap: one call's host->device copies run while another's kernels and device->host
    copy run (PCIe is full duplex)."""
    if stream is not None and not isinstance(stream, torch.cuda.Stream):
        stream = torch.cuda.ExternalStream(int(stream))
    with torch.cuda.stream(stream if stream is not None else torch.cuda.current_stream()):
        s = torch.cuda.current_stream()
        rp = row_ptr_h.to(device, non_blocking=True)
        ci = col_h.to(device, non_blocking=True)
        va = None if val_h is None else val_h.to(device, non_blocking=True)
        x = x_h.to(device, non_blocking=True)
        br, bo, ws = acsr_bin(rp, None, ci.numel(), stream=s, col_idx=ci, n_cols=x.numel())
        y = acsr_spmv(rp, ci, va, x, br, bo, ws, stream=s)
        if y_h is None:
            return y.cpu()
        y_h.copy_(y, non_blocking=True)
        return y_h


def _power_loop(m: ACSRMatrix, outdeg, x, damping, teleport, eps, max_iter, check_every, stream,
                restart=-1, restart_weight=0.0, graph=False):
    """Alg. 5-style loop with device-side convergence: up to check_every fused steps are
    enqueued between host synchronisations; a step after convergence is a no-op (ctrl[0]),
    so results equal a host test after every step.  With graph=True (and the default
    stream) the block of check_every steps is captured once into a CUDA graph and
    replayed, so the host issues one launch per block instead of one per step (the
    buffers alternate with the step parity and check_every is even, so every block sees
    the same pointers).  Capturing costs milliseconds (torch.cuda.graph synchronises and
    collects), so it pays only for long solves on small matrices, where a step is shorter
    than its host launch; off by default.  Returns (x, iterations, delta2)."""
    n = m.n_rows
    dev = m.row_begin.device
    bufs = [x, torch.empty_like(x)]
    sbufs = [acsr_pagerank_scale(x, outdeg, stream=stream), torch.empty_like(x)]
    d2 = torch.zeros(1, dtype=torch.float64, device=dev)
    ctrl = torch.zeros(2, dtype=torch.int32, device=dev)
    eps2 = eps * eps if eps >= 0 else -1.0

    def step(k):
        acsr_pagerank_step(m.row_begin, m.col_idx, m.bin_rows, m.bin_offsets, m.plan_ws, sbufs[k % 2],
                           bufs[k % 2], outdeg, bufs[(k + 1) % 2], sbufs[(k + 1) % 2], d2, damping,
                           teleport, n, m.row_end, stream, restart=restart, restart_weight=restart_weight,
                           ctrl=ctrl, eps2=eps2)

    use_graph = graph and stream is None and check_every % 2 == 0 and check_every > 0
    g = None
    k = 0
    while k < max_iter:
        nblk = min(check_every, max_iter - k)
        if use_graph and k > 0 and nblk == check_every:
            if g is None:  # the first block ran eagerly (lazy kernel attributes are set)
                g = torch.cuda.CUDAGraph()
                with torch.cuda.graph(g):
                    for j in range(check_every):
                        step(j)
            g.replay()
            k += check_every
        else:
            for _ in range(nblk):
                step(k)
                k += 1
        c = ctrl.cpu()
        if int(c[0]) == ACSR_CTRL_PLAN_ERROR:
            acsr_plan_status(m.plan_ws, stream)  # raises: the plan is invalid (outputs are NaN)
        if int(c[0]):
            break
    it = int(c[1])
    return bufs[it % 2], it, float(d2.item())


def pagerank(m: ACSRMatrix, outdeg, x0=None, damping=0.85, eps=1e-6, max_iter=1000, stream=None,
             check_every=8, graph=False):
    """Alg. 5 on one GPU over the in-link pattern matrix m (stop when
    ||x' - x||_2 <= eps, reading Q9).  Returns (x, iterations, delta2)."""
    n = m.n_rows
    dev = m.row_begin.device
    x = torch.full((n,), 1.0 / n, dtype=torch.float64, device=dev) if x0 is None else x0.clone()
    return _power_loop(m, outdeg, x, damping, (1.0 - damping) / n, eps, max_iter, check_every, stream,
                       graph=graph)


def rwr(m: ACSRMatrix, outdeg, restart: int, c=0.85, eps=1e-6, max_iter=1000, r0=None, stream=None,
        check_every=8, graph=False):
    """Random Walk with Restart (Eq. 8; reading R5) on the in-link pattern m:
    r' = c (W r) + (1-c) e_restart, r^0 = e_restart.  One fused acsr_pagerank_step per
    iteration (teleport 0, restart weight 1-c).  Returns (r, iterations, delta2)."""
    n = m.n_rows
    dev = m.row_begin.device
    if r0 is None:
        r = torch.zeros(n, dtype=torch.float64, device=dev)
        r[restart] = 1.0
    else:
        r = r0.clone()
    return _power_loop(m, outdeg, r, c, 0.0, eps, max_iter, check_every, stream, restart=restart,
                       restart_weight=1.0 - c, graph=graph)


def hits_matrix(out_ptr, out_col, n=None):
    """The 2n x 2n pattern CSR [[0, A^T], [A, 0]] of Eq. 7 from the out-link CSR of A
    (input construction: torch sort/scan on the device)."""
    n = out_ptr.numel() - 1 if n is None else n
    dev = out_ptr.device
    ln = (out_ptr[1:] - out_ptr[:-1]).long()
    src = torch.repeat_interleave(torch.arange(n, device=dev), ln)
    dst = out_col.long()
    order = torch.sort(dst * n + src).indices  # A^T rows = targets, sorted by source
    in_ptr = torch.zeros(n + 1, dtype=torch.int64, device=dev)
    in_ptr[1:] = torch.cumsum(torch.bincount(dst, minlength=n), 0)
    in_col = src[order]
    nnz = out_col.numel()
    row_ptr = torch.cat([in_ptr, out_ptr[1:].long() + nnz]).to(torch.int32)
    col = torch.cat([in_col + n, out_col.long()]).to(torch.int32)
    return row_ptr, col


def hits(out_ptr, out_col, eps=1e-6, max_iter=1000, stream=None, B=None, check_every=8):
    """HITS (Eq. 5-7; reading R6): one acsr_spmv on [[0, A^T], [A, 0]] per
    iteration plus acsr_hits_normalize.  a^0 = h^0 = 1/|V|.  B: the binned block
    matrix (ACSRMatrix of hits_matrix(out_ptr, out_col)), built here when None.  The stop
    test (both distances <= eps) runs on the device: check_every iterations are
    enqueued per host synchronisation and iterations after convergence are no-ops -- the
    same result as a host test after every iteration.  Returns (a, h, iters)."""
    n = out_ptr.numel() - 1
    dev = out_ptr.device
    if B is None:
        rp, col = hits_matrix(out_ptr, out_col, n)
        B = ACSRMatrix(rp, col, None, n_cols=2 * n)
    bufs = [torch.full((2 * n,), 1.0 / n, dtype=torch.float64, device=dev),
            torch.empty(2 * n, dtype=torch.float64, device=dev)]
    y = torch.empty_like(bufs[0])
    d2 = torch.zeros(2, dtype=torch.float64, device=dev)
    ctrl = torch.zeros(2, dtype=torch.int32, device=dev)
    ws = torch.empty(acsr_hits_workspace_bytes(n), dtype=torch.uint8, device=dev)
    eps2 = eps * eps if eps >= 0 else -1.0
    k = 0
    while k < max_iter:
        for _ in range(min(max(1, check_every), max_iter - k)):
            B.spmv(bufs[k % 2], y, stream)
            acsr_hits_normalize(y, bufs[k % 2], bufs[(k + 1) % 2], d2, ws, stream, ctrl=ctrl, eps2=eps2)
            k += 1
        if int(ctrl[0].item()):
            break
    it = int(ctrl[1].item())
    v = bufs[it % 2]
    return v[:n], v[n:], it


def degree_relabel(in_ptr, in_col, outdeg, sort_rows=False):
    """Vertex relabelling for PageRank locality (an application-level preprocessing step,
    not part of ACSR), on the device: acsr_degree_relabel (include/acsr.h) -- vertices by
    decreasing out-degree (ties by id), rows and columns alike (P A P^T), so the kernels run
    unchanged and PR in the original order is x_new[perm].  Returns
    (row_ptr', col', outdeg', perm) with perm[v] = new id of vertex v (int64)."""
    from . import acsr_degree_relabel
    rp2, c2, od2, perm = acsr_degree_relabel(in_ptr, in_col, outdeg, sort_rows=sort_rows)
    return rp2, c2, od2, perm.to(torch.int64)
