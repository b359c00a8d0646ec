"""Row-partitioned multi-GPU PageRank (§VIII P:343-348 "a simple division ... each GPU is
thus responsible for computing half the results", generalised to P ranks; reading Q19).

One process per GPU (torchrun).  Per iteration each rank runs ONE fused
``acsr_pagerank_step`` on its contiguous row range (SpMV on the in-link pattern +
teleport/damping epilogue + xs slice + exact Delta^2 partial) and the exchange, A9 of
SURVEY §8(a).  Three exchanges, all bitwise-equivalent:

  * ``exchange="acsr"`` (default on GPUs): the library owns it (include/acsr.h,
    ``acsr_comm``): the same ``acsr_pagerank_step`` call, given the communicator, runs an
    in-place NCCL all-gather of the equal-length slices and an all-gather of the ranks'
    exact fixed-point Delta^2 partials on the caller's stream; the global Delta^2 and the
    device-side stop flag are identical on every rank, so steps are enqueued back to back
    with a host check every ``check_every`` steps, as on one GPU.  torch.distributed only
    carries the 128-byte NCCL id at setup.
  * ``exchange="torch"``: the same data movement through torch.distributed collectives
    (all_gather_into_tensor + all_reduce of Delta^2); used by the gloo tests on CPU
    (tests/test_dist_gloo.py, oracle step) and by ranks sharing one GPU over gloo.
  * ``exchange="peer"``: the all-gather disappears into the step kernel itself, which
    stores every finished xs' slice entry into all ranks' replicated xs over peer memory
    (``acsr_pagerank_step_peer``).

Host logic here (partition, column renumbering into the padded or compact layout, the
loop) is device-agnostic so it is unit-tested with the gloo backend on CPU by injecting a
CPU step function; on GPUs the step is the CUDA kernel.
"""
from __future__ import annotations

import numpy as np
import torch
import torch.distributed as dist


def partition_rows(row_lengths: np.ndarray, P: int, b_nnz: int = 4, b_row: int = 36, align: int = 1) -> np.ndarray:
    """Contiguous split balanced on cost(r) = b_nnz*len_r + b_row (integer bytes; PageRank
    pattern: 4 B per column index + 36 B per row).  splits[0] = 0, splits[P] = n and
    splits[k] = min{r : sum_{r'<r} cost >= ceil(k*total/P)}, rounded up to a multiple of
    align (reading R7).  Host version for the CPU tests; GPUs use acsr_partition."""
    ln = np.asarray(row_lengths, dtype=np.int64)
    n = ln.size
    pref = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(b_nnz * ln + b_row, out=pref[1:])
    total = int(pref[-1])
    s = np.empty(P + 1, dtype=np.int64)
    s[0], s[P] = 0, n
    for k in range(1, P):
        t = -(-k * total // P)
        s[k] = int(np.searchsorted(pref, t, side="left"))
        if align > 1:
            s[k] = min(n, -(-int(s[k]) // align) * align)
    return s


def padded_layout(splits: np.ndarray):
    """Equal-size slices for the in-place all-gather: vertex v of rank k lives at
    k*L + (v - splits[k]) with L = max slice length."""
    sizes = np.diff(splits)
    L = int(sizes.max()) if sizes.size else 0
    return L


def renumber_columns(col: torch.Tensor, splits: np.ndarray, L: int) -> torch.Tensor:
    """Global vertex ids -> padded positions (setup, once per graph)."""
    sp = torch.as_tensor(splits[1:-1], dtype=torch.int64, device=col.device)
    c = col.to(torch.int64)
    owner = torch.searchsorted(sp, c, right=True)
    start = torch.as_tensor(splits[:-1], dtype=torch.int64, device=col.device)[owner]
    return (owner * L + (c - start)).to(torch.int32)


def permute_rows(row_ptr: torch.Tensor, col: torch.Tensor, perm: torch.Tensor):
    """CSR with its rows reordered: new row i = old row perm[i] (columns untouched)."""
    rp = row_ptr.to(torch.int64)
    lens = (rp[1:] - rp[:-1])[perm]
    new_rp = torch.zeros_like(rp)
    torch.cumsum(lens, 0, out=new_rp[1:])
    nnz = int(new_rp[-1])
    row_of = torch.repeat_interleave(torch.arange(perm.numel(), device=rp.device), lens, output_size=nnz)
    old = rp[perm][row_of] + torch.arange(nnz, device=rp.device) - new_rp[:-1][row_of]
    return new_rp.to(torch.int32), col[old].contiguous()


class DistPageRank:
    """PageRank over P ranks.  Each rank passes its local in-link CSR rows
    [splits[rank], splits[rank+1]) with GLOBAL column ids; the object renumbers the
    columns once and owns the replicated padded xs buffers.

    Exchange layouts (world > 1):
      compact=False  every vertex has a slot: slice length L = max rows per rank.
      compact=True   (default) only vertices with outdeg > 0 have a slot.  xs_u = 0
                     exactly when outdeg_u = 0 (Alg. 5 with reading Q11) and such a
                     vertex is never a column of the in-link pattern, so the all-gather
                     carries only the non-dangling entries (R-MAT: about half of the
                     vertices are dangling) -- lossless.  Each rank
                     orders its local rows non-dangling first (a local relabelling, undone
                     on output), so its exchanged slice is a prefix of its local xs.
                     A column whose vertex is dangling (inconsistent outdeg input) reads a
                     trailing slot that is always 0, as Alg. 5 prescribes.

    step_fn(xs, x, x_new, xs_next_local, delta2) computes one local step on
    (self.row_ptr, self.col, self.outdeg); the default runs the CUDA kernel
    (acsr_pagerank_step)."""

    def __init__(self, row_ptr_local, col_local, outdeg_local, splits, n_global, damping=0.85,
                 group=None, step_fn=None, scale_fn=None, device=None, compact=True, exchange=None, comm=None):
        if exchange is None:
            exchange = "torch" if step_fn is not None else "acsr"
        if exchange not in ("acsr", "torch", "peer"):
            raise ValueError(f"exchange must be 'acsr' (library NCCL), 'torch' (torch.distributed) or 'peer', "
                             f"not {exchange!r}")
        if exchange in ("peer", "acsr") and (step_fn is not None or scale_fn is not None):
            raise ValueError(f"exchange={exchange!r} runs inside the library's CUDA step (no step_fn)")
        self.exchange_mode = exchange
        self.comm = None
        if exchange == "acsr":
            from . import AcsrComm
            self.comm = comm if comm is not None else AcsrComm.from_process_group(group)
        self.group = group
        self.rank = dist.get_rank(group) if dist.is_initialized() else 0
        self.world = dist.get_world_size(group) if dist.is_initialized() else 1
        self.splits = np.asarray(splits, dtype=np.int64)
        assert self.splits.size == self.world + 1
        self.n_global = int(n_global)
        self.n_local = int(self.splits[self.rank + 1] - self.splits[self.rank])
        self.L = padded_layout(self.splits)
        self.damping = float(damping)
        self.teleport = (1.0 - self.damping) / self.n_global  # computed once, same bits on all ranks
        self.device = row_ptr_local.device if device is None else device
        self.compact = bool(compact) and self.world > 1
        self.perm = None
        if self.compact:
            self._setup_compact(row_ptr_local, col_local, outdeg_local)
        else:
            self.row_ptr = row_ptr_local
            self.col = renumber_columns(col_local, self.splits, self.L) if self.world > 1 else col_local
            self.outdeg = outdeg_local
            self.Lx = self.L
        use_cuda = step_fn is None
        self.step_fn = step_fn or self._cuda_step
        self.scale_fn = scale_fn or self._cuda_scale
        dev = self.device
        # replicated gathered xs (+1 trailing always-zero slot in the compact layout)
        nx = self.world * self.Lx + (1 if self.compact else 0)
        self.nx = nx
        self.peer = None
        if exchange == "peer":
            self._setup_peer(nx)
            self.xs = self.xs_next = torch.zeros(0, dtype=torch.float64, device=dev)  # in the peer regions
        else:
            self.xs = torch.zeros(nx, dtype=torch.float64, device=dev)
            self.xs_next = torch.zeros_like(self.xs)
        # compact: the kernel writes the local xs here; its first Lx entries are exchanged
        self.xs_loc = (torch.zeros(max(self.n_local, self.Lx), dtype=torch.float64, device=dev)
                       if self.compact else None)
        self.delta2 = torch.zeros(1, dtype=torch.float64, device=dev)
        self._m = None
        if use_cuda:
            from .matrix import ACSRMatrix
            self._m = ACSRMatrix(self.row_ptr, self.col, None, n_cols=nx)

    def _setup_peer(self, nx):
        """acsr_peer regions: xs double buffer + flags per rank, handles all-gathered once."""
        from . import AcsrPeer
        if self.compact:
            off, ln = self.rank * self.Lx, self.n_nd[self.rank]
        else:
            off, ln = self.rank * self.L, self.n_local
        self.peer = AcsrPeer(self.world, self.rank, nx, off, ln)
        if self.world > 1:
            hs = [None] * self.world
            dist.all_gather_object(hs, self.peer.handle_bytes(), group=self.group)
        else:
            hs = [self.peer.handle_bytes()]
        self.peer.open(hs)

    def _setup_compact(self, row_ptr_local, col_local, outdeg_local):
        dev = row_ptr_local.device
        world, L = self.world, self.L
        nd_local = (outdeg_local > 0)
        # global non-dangling mask: all-gather the padded local masks (setup, once)
        pad = torch.zeros(L, dtype=torch.uint8, device=dev)
        pad[: self.n_local] = nd_local.to(torch.uint8)
        allm = torch.zeros(world * L, dtype=torch.uint8, device=dev)
        if self.comm is not None:
            self.comm.allgather(pad, allm)
        else:
            dist.all_gather_into_tensor(allm, pad.clone() if dev.type == "cpu" else pad, group=self.group)
        sizes = np.diff(self.splits)
        nd = torch.cat([allm[k * L: k * L + int(sizes[k])] for k in range(world)])
        if dev.type == "cuda":
            # the layout arithmetic in the library (acsr_exchange_layout, acsr_permute_graph)
            from . import acsr_exchange_layout, acsr_permute_graph
            sp = torch.as_tensor(self.splits, dtype=torch.int64, device=dev)
            pos, order, nnd, self.Lx = acsr_exchange_layout(nd.contiguous(), sp, rank=self.rank)
            self.n_nd = nnd
            self.perm = order.to(torch.int64)
            self.row_ptr, self.col = acsr_permute_graph(row_ptr_local.to(torch.int32).contiguous(),
                                                        col_local.contiguous(), order, col_map=pos)
            self.outdeg = outdeg_local[self.perm].contiguous()
            return
        nd = nd.to(torch.bool)
        nnd = [int(allm[k * L: k * L + int(sizes[k])].sum()) for k in range(world)]
        self.n_nd = nnd
        self.Lx = max(1, max(nnd))
        # compact position of every vertex: owner * Lx + rank among the owner's non-dangling
        sp = torch.as_tensor(self.splits, dtype=torch.int64, device=dev)
        csum = torch.cumsum(nd.to(torch.int64), 0)
        ex = csum - nd.to(torch.int64)  # exclusive prefix over all vertices
        owner = torch.searchsorted(sp[1:-1], torch.arange(self.n_global, device=dev), right=True)
        base = torch.cat([torch.zeros(1, dtype=torch.int64, device=dev), csum])[sp[:-1]][owner]
        pos = torch.where(nd, owner * self.Lx + (ex - base), torch.full_like(ex, world * self.Lx))
        col = pos[col_local.to(torch.int64)].to(torch.int32)
        # local rows: non-dangling first (stable), so the exchanged slice is a prefix
        perm = torch.cat([torch.nonzero(nd_local).flatten(), torch.nonzero(~nd_local).flatten()])
        self.perm = perm
        self.row_ptr, self.col = permute_rows(row_ptr_local, col, perm)
        self.outdeg = outdeg_local[perm].contiguous()

    def _local_out(self):
        """Where the local step writes its xs slice."""
        if self.compact:
            return self.xs_loc[: self.n_local]
        return self.xs_next[self.rank * self.L: self.rank * self.L + self.n_local]

    def _cuda_step(self, xs, x, x_new, xs_next_slice, delta2):
        from . import acsr_pagerank_step
        m = self._m
        acsr_pagerank_step(m.row_begin, m.col_idx, m.bin_rows, m.bin_offsets, m.plan_ws, xs, x,
                           self.outdeg, x_new, xs_next_slice, delta2, self.damping, self.teleport,
                           self.n_global)

    def _cuda_scale(self, x, outdeg, out):
        from . import acsr_pagerank_scale
        acsr_pagerank_scale(x, outdeg, out)

    def exchange(self, buf):
        """Gather every rank's slice into buf (the replicated xs of the next step)."""
        if self.compact:
            dist.all_gather_into_tensor(buf[: self.world * self.Lx], self.xs_loc[: self.Lx], group=self.group)
        elif self.world > 1:
            chunk = buf[self.rank * self.L:(self.rank + 1) * self.L]  # padded: tail stays 0
            dist.all_gather_into_tensor(buf, chunk.clone() if buf.device.type == "cpu" else chunk,
                                        group=self.group)

    def _run_peer(self, x, eps, max_iter, check_every):
        """Steps are enqueued back to back (no per-step collective or extra launch); each
        step tests the global Delta^2 of the previous one at entry (device-side stop
        flag), and the host reads the global Delta^2 every check_every steps."""
        from . import acsr_pagerank_step_peer
        m, peer = self._m, self.peer
        peer.push(x, self.outdeg)
        bufs = [x, torch.empty_like(x)]
        part = torch.zeros(1, dtype=torch.float64, device=self.device)
        ctrl = torch.zeros(2, dtype=torch.int32, device=self.device)
        eps2 = eps * eps if eps >= 0 else -1.0
        k = 0
        while k < max_iter:
            for _ in range(min(check_every, max_iter - k)):
                acsr_pagerank_step_peer(peer, m.row_begin, m.col_idx, m.bin_rows, m.bin_offsets, m.plan_ws,
                                        bufs[k % 2], self.outdeg, bufs[(k + 1) % 2], None, part,
                                        self.damping, self.teleport, self.n_global, ctrl=ctrl, eps2=eps2)
                k += 1
            peer.delta2(self.delta2)  # global Delta^2 of the last executed step
            c = ctrl.cpu()
            if int(c[0]) or float(self.delta2.item()) <= eps2:
                break
        it = int(ctrl[1].item())
        _, err, _ = peer.query()
        if err:
            raise RuntimeError("acsr_peer: a peer barrier timed out (a rank stopped issuing steps?)")
        return bufs[it % 2], it, float(self.delta2.item())

    def _run_acsr(self, x, eps, max_iter, check_every):
        """Library-owned exchange: every acsr_pagerank_step call carries the communicator,
        so the step, the xs all-gather and the exact global Delta^2 (+ device-side stop
        flag, identical on every rank) are enqueued back to back; the host looks at the
        flag every check_every steps.  Same results as a host test after every step."""
        from . import acsr_pagerank_init, acsr_pagerank_step
        m, comm = self._m, self.comm
        Ls = self.Lx if self.compact else self.L  # exchanged entries per rank

        def local_out(buf):
            if self.compact:
                return self.xs_loc  # the exchanged prefix is xs_loc[:Lx]
            return buf[self.rank * self.L:(self.rank + 1) * self.L]  # in place

        bufs = [x, torch.empty_like(x)]
        xsb = [self.xs, self.xs_next]
        # all-gather-v: only each rank's real entries move (non-dangling counts, or row counts)
        counts = self.n_nd if self.compact else [int(c) for c in np.diff(self.splits)]
        acsr_pagerank_init(x, self.outdeg, local_out(xsb[0]), comm=comm, xs_all=xsb[0], slice_len=Ls,
                           slice_counts=counts)
        ctrl = torch.zeros(2, dtype=torch.int32, device=self.device)
        eps2 = eps * eps if eps >= 0 else -1.0
        k = 0
        while k < max_iter:
            for _ in range(min(check_every, max_iter - k)):
                a, b = k % 2, (k + 1) % 2
                acsr_pagerank_step(m.row_begin, m.col_idx, m.bin_rows, m.bin_offsets, m.plan_ws, xsb[a], bufs[a],
                                   self.outdeg, bufs[b], local_out(xsb[b]), self.delta2, self.damping,
                                   self.teleport, self.n_global, ctrl=ctrl, eps2=eps2, comm=comm, xs_all=xsb[b],
                                   slice_len=Ls, slice_counts=counts)
                k += 1
            c = ctrl.cpu()
            if int(c[0]):
                break
        it = int(ctrl[1].item())
        if int(ctrl[0]) == 2:
            m.plan_status()  # raises: invalid plan
        return bufs[it % 2], it, float(self.delta2.item())

    def exchange_bytes_per_rank(self):
        """Bytes this rank receives per iteration: the other ranks' real entries with the
        library exchange (all-gather-v) or the peer pushes, the padded slices with torch."""
        if self.exchange_mode in ("acsr", "peer"):
            counts = self.n_nd if self.compact else [int(c) for c in np.diff(self.splits)]
            return 8 * (sum(counts) - counts[self.rank])
        return (self.world - 1) * self.Lx * 8

    def run(self, x0_local=None, eps=1e-6, max_iter=1000, check_every=None):
        """Alg. 5 loop; returns (x_local, iterations, delta2_global) with x_local in the
        caller's local row order.  check_every (acsr / peer exchanges): steps enqueued
        between host synchronisations (default 8 / 1); steps after convergence are no-ops on
        every rank (device-side stop flag) -- same results as checking every step."""
        dev = self.device
        if x0_local is None:
            x = torch.full((self.n_local,), 1.0 / self.n_global, dtype=torch.float64, device=dev)
        else:
            x = x0_local.clone() if self.perm is None else x0_local[self.perm].contiguous()
        if self.exchange_mode in ("peer", "acsr"):
            ce = check_every if check_every is not None else (8 if self.exchange_mode == "acsr" else 1)
            run = self._run_peer if self.exchange_mode == "peer" else self._run_acsr
            x, it, d2 = run(x, eps, max_iter, max(1, int(ce)))
            if self.perm is not None:
                out = torch.empty_like(x)
                out[self.perm] = x
                x = out
            return x, it, d2
        # xs^0 slice = x^0 / outdeg (IEEE division), then gather
        if self.compact:
            self.scale_fn(x, self.outdeg, self._local_out())
            self.exchange(self.xs)
        else:
            self.scale_fn(x, self.outdeg, self.xs[self.rank * self.L: self.rank * self.L + self.n_local])
            self.exchange(self.xs)
        x_new = torch.empty_like(x)
        it, d2 = 0, float("inf")
        while it < max_iter:
            self.step_fn(self.xs, x, x_new, self._local_out(), self.delta2)
            self.exchange(self.xs_next)
            if self.world > 1:
                dist.all_reduce(self.delta2, group=self.group)
            x, x_new = x_new, x
            self.xs, self.xs_next = self.xs_next, self.xs
            it += 1
            d2 = float(self.delta2.item())
            if d2 ** 0.5 <= eps:
                break
        if self.perm is not None:
            out = torch.empty_like(x)
            out[self.perm] = x
            x = out
        return x, it, d2


def aligned_slice(t: torch.Tensor, start: int, stop: int, elems_per_16b: int) -> torch.Tensor:
    """Copy t[start:stop] into a fresh buffer whose first element sits at the same
    16-byte phase as t[start] does in t (elements of width 16/elems_per_16b).  The SpMV
    groups 128-bit vector loads by that phase, so a row's summation order -- and its
    result bits -- are the same in the slice as in the whole array (SURVEY §8(c),
    "P-invariance")."""
    ph = start % elems_per_16b
    buf = torch.empty(stop - start + ph, dtype=t.dtype, device=t.device)
    out = buf[ph:]
    out.copy_(t[start:stop])
    return out


class DistSpMV:
    """One SpMV y = A x row-split across P ranks (§VIII: "map half of the rows in
    each bin to each device, each GPU is thus responsible for computing half the
    results", generalised to P ranks as contiguous nnz-balanced row ranges, reading Q19;
    SURVEY §8(f) N4).  Rank k holds rows [splits[k], splits[k+1]) with GLOBAL column ids
    and the whole x; it bins its rows once (acsr_bin) and every call runs acsr_spmv on
    them -- no exchange in the SpMV itself.  gather() all-gathers the y slices (padded,
    in place) when every rank needs the whole y.

    The local col/val keep their global 16-byte phase (aligned_slice) and, with split points
    on 32-row boundaries (partition align=32, reading R7), every short-row window holds the
    same rows, so every row is summed exactly as on one GPU: the P-rank y equals the 1-GPU
    y bit for bit.

    spmv_fn(row_ptr, col, val, x) -> y_local overrides the CUDA call (CPU tests)."""

    def __init__(self, row_ptr, col, val, splits, group=None, spmv_fn=None, b_nnz=None, b_row=16):
        self.group = group
        self.rank = dist.get_rank(group) if dist.is_initialized() else 0
        self.world = dist.get_world_size(group) if dist.is_initialized() else 1
        self.splits = np.asarray(splits, dtype=np.int64)
        assert self.splits.size == self.world + 1
        lo, hi = int(self.splits[self.rank]), int(self.splits[self.rank + 1])
        rp = row_ptr.to(torch.int64)
        k0, k1 = int(rp[lo]), int(rp[hi])
        self.row_ptr = (rp[lo:hi + 1] - k0).to(torch.int32)
        self.col = aligned_slice(col, k0, k1, 4)
        self.val = None if val is None else aligned_slice(val, k0, k1, 16 // val.element_size())
        self.n_local = hi - lo
        self.L = padded_layout(self.splits)
        self._m = None
        self.spmv_fn = spmv_fn
        self.n_cols = None

    def _matrix(self, n_cols):
        if self._m is None:
            from .matrix import ACSRMatrix
            self._m = ACSRMatrix(self.row_ptr, self.col, self.val, n_cols=n_cols)
        return self._m

    def spmv(self, x, y_local=None):
        """This rank's rows of A x."""
        if self.spmv_fn is not None:
            return self.spmv_fn(self.row_ptr, self.col, self.val, x)
        return self._matrix(x.numel()).spmv(x, y_local)

    def rebin(self):
        if self._m is not None:
            self._m.rebin()

    def gather(self, y_local, comm=None):
        """Whole y on every rank (padded equal-size all-gather of the slices): through the
        library's NCCL communicator (acsr_comm_allgather) when comm is given, else
        torch.distributed (the gloo CPU tests)."""
        if self.world == 1:
            return y_local
        pad = torch.zeros(self.L, dtype=y_local.dtype, device=y_local.device)
        pad[: self.n_local] = y_local
        allp = torch.empty(self.world * self.L, dtype=y_local.dtype, device=y_local.device)
        if comm is not None:
            comm.allgather(pad, allp)
        else:
            dist.all_gather_into_tensor(allp, pad, group=self.group)
        sizes = np.diff(self.splits)
        return torch.cat([allp[k * self.L: k * self.L + int(sizes[k])] for k in range(self.world)])
