/*
 * acsr.h -- C ABI of libacsr.so: adaptive CSR SpMV (ACSR, Ashari et al., SC'14)
 * for NVIDIA B200 (sm_100a).
 *
 * Citations "P:L" refer to line L of the paper text; "§8(x)" to
 * SURVEY.md; "Qn" to the readings listed in DESIGN.md.
 *
 * Conventions (all entry points)
 *  - Every pointer is a DEVICE pointer unless marked HOST.
 *  - Every call is asynchronous on the caller's `stream` (a cudaStream_t; NULL =
 *    legacy default stream).  Nothing is allocated inside the calls: scratch comes
 *    from a caller-owned workspace sized by the matching *_workspace_bytes query.
 *  - Argument errors detectable on the host (NULL where required, negative sizes,
 *    workspace too small, unknown dtype) return synchronously and enqueue nothing.
 *    Data-dependent errors (update batches) are reported in a DEVICE status word.
 *    A failed kernel launch returns ACSR_ERR_CUDA; acsr_last_error() holds the text.
 *  - Index arrays are int32, row lengths must fit int32, sum of lengths < 2^31.
 *  - CSR may carry reserved slack after each row (§VII): row r occupies
 *    [row_begin[r], row_end[r]).  Passing row_end == NULL means standard CSR
 *    (§II: row r occupies [RowOffset[r], RowOffset[r+1]), i.e.
 *    row_end = row_begin + 1 and row_begin has n_rows + 1 entries).
 *  - There is no CPU fallback: on a machine without an sm_100 device every call
 *    that would launch returns ACSR_ERR_CUDA.
 */
#ifndef ACSR_H
#define ACSR_H

#include <stddef.h>
#include <stdint.h>
#include <cuda_runtime_api.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    ACSR_OK = 0,
    ACSR_ERR_INVALID_VALUE = 1, /* bad argument, or (device status) malformed change list */
    ACSR_ERR_WORKSPACE = 2,     /* workspace pointer NULL or smaller than the query */
    ACSR_ERR_CAPACITY = 3,      /* (device status) an updated row exceeds its reserved slack */
    ACSR_ERR_CUDA = 4,          /* CUDA launch / runtime failure, see acsr_last_error() */
    ACSR_ERR_NCCL = 5,          /* NCCL failure in the multi-GPU exchange, see acsr_last_error() */
    ACSR_ERR_UNSUPPORTED = 6    /* e.g. no sm_100 device */
} acsr_status;

typedef enum { ACSR_F32 = 0, ACSR_F64 = 1 } acsr_dtype;

enum { ACSR_NBINS = 32 };

/* ------------------------------------------------------------------------ */
/* Binning (Alg. 1 "if (this is the first iteration) ... foreach row r do
 * b_r <- b_r U {r}"; §III-A).  Inputs are those of
 * Alg. 1: the CSR matrix (row offsets, col_idx).
 *
 * Row r with len_r = row_end[r] - row_begin[r] non-zeros goes to bin
 *     b = 0 if len_r == 0;  1 if len_r <= 2;  else ceil(log2(len_r))
 * i.e. bin i holds [2^{i-1}+1 .. 2^i] non-zeros (reading Q1), bin 0 the
 * empty rows (reading Q2).  Outputs:
 *   bin_rows[n_rows]        row ids grouped by bin, ascending row id inside a bin
 *                           (stable; reading Q3) -- the paper's BIN#N_Rows lists
 *   bin_offsets[33]         bin b = bin_rows[bin_offsets[b] .. bin_offsets[b+1]),
 *                           bin_offsets[32] = n_rows
 *   plan_ws                 the SpMV work map (replaces Alg. 1's G1/G2 split and
 *                           the dynamic-parallelism parent/child launches, P:61,
 *                           P:68-105): warp work units in row-space order, the
 *                           split plan for rows longer than 1024 non-zeros, and
 *                           (if col_idx != NULL) the hot-column table of the SpMV's
 *                           shared-memory x cache (the B200 stand-in for the paper's
 *                           texture-bound x): occurrence counts over a strided
 *                           sample of ~2^20 entries, per-slot most frequent column --
 *                           a performance hint only, never a result.
 * n_cols is the length of x (column ids outside [0, n_cols) are ignored by the
 * sampler).  nnz_max bounds the number of stored entries (sum of row lengths)
 * that any later acsr_bin on this workspace will see (slack CSR: the capacity).
 * The row-length array is read twice (count pass + stable scatter pass); no
 * host synchronisation happens.  bin_rows/bin_offsets are deterministic and
 * equal the oracle bit for bit.  plan_ws must not be shared by concurrent calls. */
size_t acsr_bin_workspace_bytes(int64_t n_rows, int64_t n_cols, int64_t nnz_max);

/* Plan health.  If nnz_max understates the stored entries seen by acsr_bin, the SpMV work
 * list no longer fits the workspace: the plan is marked invalid (nothing is written out of
 * bounds), and every later acsr_spmv / acsr_pagerank_step on it writes a quiet NaN to every
 * output row (PageRank: *delta2 = NaN, and ctrl[0] = ACSR_CTRL_PLAN_ERROR so a device-side
 * loop stops) instead of leaving stale data.  acsr_plan_status synchronises `stream` and
 * returns ACSR_ERR_CAPACITY for such a plan (detail in acsr_last_error()), ACSR_OK
 * otherwise; call it after acsr_bin whenever nnz_max is not known to be an upper bound. */
enum { ACSR_CTRL_PLAN_ERROR = 2 };
acsr_status acsr_plan_status(const void *plan_ws, size_t plan_ws_bytes, cudaStream_t stream);

acsr_status acsr_bin(int64_t n_rows, int64_t n_cols, int64_t nnz_max,
                     const int32_t *row_begin, const int32_t *row_end /* NULL => standard CSR */,
                     const int32_t *col_idx /* NULL => no x cache */,
                     int32_t *bin_rows /* [n_rows] out */,
                     int32_t *bin_offsets /* [ACSR_NBINS + 1] out */,
                     void *plan_ws, size_t plan_ws_bytes, cudaStream_t stream);

/* acsr_bin_ex: acsr_bin with plan flags (acsr_bin == acsr_bin_ex(..., 0, stream)).
 *   ACSR_BIN_SHORT_ALG2   rows of bins 0..5 (<= 32 non-zeros) get per-bin work units
 *                         and the SpMV maps them exactly as Alg. 2: a
 *                         sub-warp of 2^{b-1} lanes per row, width-2^{b-1} shuffle
 *                         reduction, lane 0 writes.  Without the flag (default) they
 *                         are processed in short-row windows: a warp takes 32
 *                         consecutive rows (one per lane), loads the concatenated
 *                         non-zeros of its short rows coalesced, and each lane sums
 *                         its own row's products in element order (DESIGN.md §6:
 *                         fewer L2 sectors per short row on B200).  Both are exact
 *                         y = A x mappings (reading Q4); bin_rows/bin_offsets are
 *                         identical either way.  Unknown flag bits ->
 *                         ACSR_ERR_INVALID_VALUE. */
enum { ACSR_BIN_SHORT_ALG2 = 1u };
acsr_status acsr_bin_ex(int64_t n_rows, int64_t n_cols, int64_t nnz_max,
                        const int32_t *row_begin, const int32_t *row_end,
                        const int32_t *col_idx, int32_t *bin_rows, int32_t *bin_offsets,
                        void *plan_ws, size_t plan_ws_bytes, unsigned flags, cudaStream_t stream);

/* ------------------------------------------------------------------------ */
/* SpMV y = A x, computed directly on CSR with bin-specific mappings
 * (Alg. 2): bins 0..5 in short-row windows (default plan) or, with an
 * ACSR_BIN_SHORT_ALG2 plan, a sub-warp of 2^{b-1} lanes per row with shuffle
 * reduction (exactly Alg. 2); bin 6 always Alg. 2 (32 lanes); bins 7..10 a warp per row; rows longer
 * than 1024 non-zeros are cut into fixed chunks processed by different warps and
 * combined in chunk order by the last-arriving warp (replaces the dynamic-
 * parallelism parent/child kernels of Alg. 3/4; reading Q4/Q7/Q8).
 *   dt          ACSR_F64: values/x/y are double; ACSR_F32: float (accumulated
 *               in double, rounded once per row).
 *   values      [nnz] or NULL => pattern matrix (all ones).
 *   x           [n_cols];  y [n_rows] is overwritten, never read (reading Q5);
 *               empty rows get +0.0 (reading Q2).
 *   bin_rows, bin_offsets, plan_ws: produced by acsr_bin on the same row
 *               lengths (re-bin after every acsr_update_edges).
 * Deterministic: the summation order of every row depends only on the row's
 * length and address alignment, never on scheduling. */
acsr_status acsr_spmv(acsr_dtype dt, int64_t n_rows, int64_t n_cols,
                      const int32_t *row_begin, const int32_t *row_end /* NULL => standard */,
                      const int32_t *col_idx, const void *values /* NULL => ones */,
                      const void *x, void *y,
                      const int32_t *bin_rows, const int32_t *bin_offsets,
                      void *plan_ws, size_t plan_ws_bytes, cudaStream_t stream);

/* ------------------------------------------------------------------------ */
/* Multi-GPU communicator (§VIII: "map half of the rows ... to each device.  Each
 * GPU is thus responsible for computing half the results", generalised to P ranks as
 * contiguous row ranges, reading Q19).  One rank per GPU (one process per GPU, a single
 * node: NCCL over NVLink / NVSwitch).  The library owns the NCCL communicator and a small
 * device buffer; nothing else.  Protocol: rank 0 calls acsr_comm_get_unique_id and ships
 * the ACSR_COMM_ID_BYTES HOST bytes to every rank (any host transport); every rank then
 * calls acsr_comm_init with the SAME CUDA device current that it will use for the steps.
 * acsr_comm_init blocks until all nranks ranks joined.  NCCL failures return
 * ACSR_ERR_NCCL with the NCCL text in acsr_last_error(). */
enum { ACSR_COMM_ID_BYTES = 128 };
typedef struct acsr_comm acsr_comm;
acsr_status acsr_comm_get_unique_id(void *id /* HOST out, ACSR_COMM_ID_BYTES */);
acsr_status acsr_comm_init(acsr_comm **out, int nranks, int rank, const void *id /* HOST */);
acsr_status acsr_comm_destroy(acsr_comm *comm);
acsr_status acsr_comm_query(const acsr_comm *comm, int *nranks /* HOST out, nullable */,
                            int *rank /* HOST out, nullable */);
/* recv[q * bytes_per_rank ...] = rank q's send (in place allowed: send == recv + rank *
 * bytes_per_rank).  For setup-time layout work (e.g. the non-dangling masks of the compact
 * exchange layout, handles) and for gathering a row-split SpMV's y slices. */
acsr_status acsr_comm_allgather(acsr_comm *comm, const void *send, void *recv, size_t bytes_per_rank,
                                cudaStream_t stream);
/* All-gather-v: recv[q * stride_bytes ...] receives counts_bytes[q] bytes (HOST array) of rank
 * q's send (one grouped ncclBroadcast per rank; bytes past a count are left untouched). */
acsr_status acsr_comm_allgatherv(acsr_comm *comm, const void *send, void *recv, size_t stride_bytes,
                                 const int64_t *counts_bytes, cudaStream_t stream);

/* O8 row partition, on the device: splits[0] = 0, splits[nranks] = n_rows and
 *   splits[k] = min{ r : sum_{r' < r} cost(r') >= ceil(k * total / nranks) },
 *   cost(r) = b_nnz * len_r + b_row   (integer bytes of the rank's traffic per row:
 *   PageRank pattern 4 * len + 36, weighted fp64 SpMV 12 * len + 16),
 * then each splits[k] rounded up to a multiple of `align` (<= 1: unchanged) and clamped to
 * n_rows (reading R7: with align = 32 every rank's rows start on a 32-row boundary, so
 * the SpMV's short-row windows hold the same rows on P ranks as on one GPU and a
 * row-split SpMV gives the one-GPU y bit for bit).
 * splits: DEVICE int64 [nranks + 1].  ws: acsr_partition_workspace_bytes(n_rows) bytes
 * (an int64 prefix of the costs + the scan's scratch). */
size_t acsr_partition_workspace_bytes(int64_t n_rows);
acsr_status acsr_partition(int64_t n_rows, const int32_t *row_begin, const int32_t *row_end /* NULL => standard */,
                           int64_t b_nnz, int64_t b_row, int nranks, int64_t align, int64_t *splits, void *ws,
                           size_t ws_bytes, cudaStream_t stream);

/* Compact exchange layout of the row-partitioned PageRank (SURVEY §8(e) lever 2): xs_u = 0
 * exactly when outdeg_u = 0 (Alg. 5 with reading Q11), and such a vertex is never a column
 * of the in-link pattern, so only non-dangling vertices get a slot.  Inputs: the global
 * non-dangling mask nd[n_global] (DEVICE u8; assembled from every rank's local mask, e.g. by
 * acsr_comm_allgather) and the partition splits (DEVICE int64 [nranks + 1]).  Outputs:
 *   counts[k] (DEVICE int64)  non-dangling vertices of rank k;  lx[0] = max(1, max counts)
 *   pos[v]  (DEVICE int32)    owner(v) * Lx + (rank of v among its owner's non-dangling
 *                             vertices) for non-dangling v, nranks * Lx (a trailing slot that
 *                             is always 0) otherwise -- the column renumbering;
 *   order   (DEVICE int32, nullable; [splits[rank+1] - splits[rank]])  this rank's local rows,
 *                             non-dangling first, each group in row order (new -> old), so the
 *                             exchanged slice is a prefix of the local xs (acsr_permute_graph).
 * ws: acsr_exchange_layout_workspace_bytes(n_global) bytes. */
size_t acsr_exchange_layout_workspace_bytes(int64_t n_global);
acsr_status acsr_exchange_layout(int64_t n_global, int nranks, const int64_t *splits, const uint8_t *nd, int rank,
                                 int32_t *pos, int32_t *order, int64_t *counts, int64_t *lx, void *ws, size_t ws_bytes,
                                 cudaStream_t stream);

/* Rows of a standard CSR reordered (new row i = old row order[i]) with every column mapped
 * through col_map (DEVICE int32 [n_cols], NULL: kept); entry order inside a row kept.  The
 * copy machinery of acsr_degree_relabel.  ws: acsr_permute_workspace_bytes(n) bytes. */
size_t acsr_permute_workspace_bytes(int64_t n);
acsr_status acsr_permute_graph(int64_t n, const int32_t *row_ptr, const int32_t *col_idx, const int32_t *order,
                               const int32_t *col_map, int32_t *row_ptr_out, int32_t *col_out, void *ws, size_t ws_bytes,
                               cudaStream_t stream);

/* ------------------------------------------------------------------------ */
/* PageRank step (Alg. 5; §VI-A) on one rank's rows.
 *   PR^{k+1} = (1-d) PR^(0) + d (A^T PR^k),  A row-normalised.
 * Storage (reading Q12): the IN-LINK pattern CSR (row v lists the sources u of
 * the edges u -> v) and the scaled vector xs_u = PR_u / outdeg_u (0 when
 * outdeg_u == 0, reading Q11).  One fused launch computes, for local row v,
 *   y_v = sum_{u -> v} xs[u]
 *   x_new[v]   = teleport + damping * y_v          (teleport = (1-d)/n, host)
 *   xs_next[v] = outdeg[v] > 0 ? x_new[v] / outdeg[v] : 0
 *   *delta2    = sum_v (x_new[v] - x[v])^2          (deterministic order)
 * Multi-GPU (§VIII, reading Q19): each rank calls this on its contiguous row range
 * (col ids index the replicated xs) with `comm` set.  The call then also runs the
 * exchange on `stream`, right after the step kernel (A9 of SURVEY §8(a)):
 *   xs_all[q * slice_len + i] = rank q's xs_next[i], i < slice_len   (ncclAllGather; in
 *       place when xs_next == xs_all + rank * slice_len; xs_next must hold >= slice_len
 *       entries -- entries i >= n_rows are padding the caller keeps at 0 -- and a rank
 *       may exchange fewer than n_rows entries, e.g. only its non-dangling prefix);
 *   *delta2 = the GLOBAL sum of (x_new - x)^2 over every rank's rows: the ranks' exact
 *       192-bit fixed-point partials are all-gathered and added in rank order, so every
 *       rank gets the same bits -- equal to the single-GPU Delta^2 of the same iterate;
 *   ctrl (if given): the stop decision is taken on the global Delta^2, identically on
 *       every rank, so device-side loops stay in lock step.
 * Every rank must issue the same sequence of calls.  xs_all is the xs of the NEXT step
 * (double-buffer xs / xs_all across steps). */
typedef struct {
    int64_t n_rows;               /* local rows */
    int64_t n_cols;               /* length of xs (global, possibly padded) */
    const int32_t *row_begin;     /* local in-link CSR */
    const int32_t *row_end;       /* NULL => standard CSR */
    const int32_t *col_idx;       /* source ids, index into xs */
    const int32_t *bin_rows;      /* from acsr_bin on the local rows */
    const int32_t *bin_offsets;
    void *plan_ws;
    size_t plan_ws_bytes;
    const double *xs;             /* [n_cols] PR^k / outdeg, replicated */
    const double *x;              /* [n_rows] PR^k of the local rows */
    const int32_t *outdeg;        /* [n_rows] out-degree of the local vertices */
    double *x_new;                /* [n_rows] PR^{k+1} */
    double *xs_next;              /* [n_rows] PR^{k+1} / outdeg (the local slice) */
    double damping;               /* d = 0.85; c for RWR */
    double teleport;              /* (1-d)/n_global, computed once on the host; 0 for RWR */
    double *delta2;               /* [1] local sum of squared differences */
    int64_t restart;              /* RWR restart row (local index) or -1 */
    double restart_weight;        /* added to x_new[restart]: (1-c) for RWR */
    int32_t *ctrl;                /* NULL, or [2] device: device-side convergence control.
                                   * If ctrl[0] != 0 the call is a no-op (nothing written);
                                   * otherwise the step runs, ctrl[1] += 1 and ctrl[0] = 1 when
                                   * *delta2 <= eps2.  Lets the host enqueue several steps
                                   * between synchronisations with results identical to a
                                   * test after every step (single GPU). */
    double eps2;                  /* convergence threshold on delta2 (eps^2) */
    acsr_comm *comm;              /* NULL => single GPU, no exchange; else see above */
    double *xs_all;               /* with comm: [n_cols] replicated xs' receiving every slice */
    int64_t slice_len;            /* with comm: entries per rank in xs_all (n_cols >= nranks * slice_len) */
    const int64_t *slice_counts;  /* with comm: HOST [nranks] or NULL.  If given, only the first
                                   * slice_counts[q] <= slice_len entries of rank q's slice are
                                   * exchanged (all-gather-v: one grouped ncclBroadcast per rank),
                                   * so unequal slices -- e.g. the non-dangling counts of a
                                   * degree-relabelled partition -- cost their sum, not
                                   * nranks * max.  Entries past the counts are left untouched.
                                   * Must hold the same values on every rank. */
} acsr_pr_args;

acsr_status acsr_pagerank_step(const acsr_pr_args *args, cudaStream_t stream);

/* First iterate of Alg. 5 (PR^(0) = 1/n; or a warm start): xs_next[r] =
 * x[r] / outdeg[r] (0 when outdeg is 0) for the local rows, then -- with comm -- the same
 * all-gather into xs_all as a step.  Fields used: n_rows, n_cols, x, outdeg, xs_next, comm,
 * xs_all, slice_len. */
acsr_status acsr_pagerank_init(const acsr_pr_args *args, cudaStream_t stream);

/* The same fused step is Random Walk with Restart (Eq. 8):
 *   r' = c (W r) + (1 - c) e_i,  W_{vu} = 1/outdeg_u on every edge u -> v (reading R5)
 * with damping = c, teleport = 0, restart = i, restart_weight = 1 - c. */

/* xs[v] = outdeg[v] > 0 ? x[v] / outdeg[v] : 0 for v < n (IEEE division).
 * Builds the first scaled vector of Alg. 5 (PR^(0) = 1/n) or of a warm
 * start. */
acsr_status acsr_pagerank_scale(int64_t n, const double *x, const int32_t *outdeg, double *xs,
                                cudaStream_t stream);

/* ------------------------------------------------------------------------ */
/* Multi-GPU PageRank with the exchange FUSED into the step over peer memory
 * (§VIII row split, reading Q19; SURVEY §8(e) lever 1 / §8(f) N1).
 * Row-partitioned PageRank needs every rank's slice of xs' = PR'/outdeg in every
 * rank's replicated xs after each step.  Here the fused step kernel stores each
 * finished slice entry directly into all ranks' xs buffers (NVLink/NVSwitch P2P
 * stores, overlapped with the rest of the step), and its last CTA publishes the
 * push -- the Delta^2 partial and a release flag -- to every rank.  The next step
 * waits on those flags at entry; no host-side collective is involved.
 *
 * One acsr_peer per rank (single node, one process per GPU; several processes may
 * share a GPU).  The library owns one device region per rank: a state block and two
 * replicated xs buffers of xs_len doubles (alternating by push parity; zeroed at
 * create, so slots nobody writes -- e.g. the trailing always-zero slot of the
 * dangling-free layout -- read +0.0).  Protocol:
 *   1. acsr_peer_create on every rank -> ACSR_IPC_HANDLE_BYTES of HOST bytes;
 *   2. the caller all-gathers the handles (any host transport, rank order);
 *   3. acsr_peer_open maps every other rank's region (cudaIpcOpenMemHandle);
 *   4. acsr_peer_push: xs = x / outdeg of the local rows (first iterate, or a
 *      warm start), rows [0, slice_len) stored at slots slice_off + r of every
 *      rank's next buffer;
 *   5. per iteration: acsr_pagerank_step_peer (acsr_pagerank_step semantics; args->xs
 *      is ignored -- the step reads the buffer of the previous push; args->n_cols must
 *      equal xs_len; args->xs_next may be NULL, else it also receives the local xs';
 *      args->delta2 receives this rank's partial).  With args->ctrl, a step first
 *      waits for the previous push of every rank, adds their exact Delta^2 partials and,
 *      when the sum is <= eps2, sets ctrl[0] and does nothing (every rank decides
 *      alike): consecutive steps need no host round trip or extra launch.
 *   6. acsr_peer_delta2 whenever the host wants the GLOBAL Delta^2 of the last push.
 * Every rank must issue the same sequence of push / step calls.  Waits are bounded
 * (20 s, or ACSR_PEER_TIMEOUT_MS read at acsr_peer_open): a timed-out wait sets the
 * error word read by acsr_peer_query and the call proceeds with invalid results
 * rather than hanging the GPU.  Results are bitwise
 * identical to the same partition with a plain all-gather (the per-row sums do not
 * depend on where xs came from).  Not thread-safe; one stream per acsr_peer. */
enum { ACSR_PEER_MAX = 8, ACSR_IPC_HANDLE_BYTES = 64 };
typedef struct acsr_peer acsr_peer;

/* slice_off/slice_len: this rank's exchanged slots [slice_off, slice_off+slice_len)
 * of xs (local rows 0..slice_len-1 in order).  handle: HOST out, 64 bytes. */
acsr_status acsr_peer_create(acsr_peer **out, int nranks, int rank, int64_t xs_len,
                             int64_t slice_off, int64_t slice_len, void *handle);
/* handles: HOST, nranks * ACSR_IPC_HANDLE_BYTES in rank order (own entry ignored). */
acsr_status acsr_peer_open(acsr_peer *p, const void *handles);
/* synchronises the device, unmaps the peers, frees the region. */
acsr_status acsr_peer_destroy(acsr_peer *p);
/* x, outdeg: [n] local rows (n >= slice_len); xs_local: NULL or [n] (also gets xs). */
acsr_status acsr_peer_push(acsr_peer *p, int64_t n, const double *x, const int32_t *outdeg,
                           double *xs_local, cudaStream_t stream);
/* args->n_rows >= 1 and >= slice_len (every rank owns at least one row); RWR fields
 * (restart, restart_weight) work as in acsr_pagerank_step on the local rows. */
acsr_status acsr_pagerank_step_peer(const acsr_pr_args *args, acsr_peer *p, cudaStream_t stream);
/* delta2: [1] device out, the global sum of every rank's partial of the last push
 * (exact fixed-point partials: the same bits on every rank; 0 if the last push was
 * acsr_peer_push).  ctrl: NULL or [2] as in
 * acsr_pr_args -- ctrl[0] is set here when delta2 <= eps2 (every rank decides alike),
 * and a call with ctrl[0] set does nothing, so blocks of (step, delta2) pairs can be
 * enqueued between host synchronisations. */
acsr_status acsr_peer_delta2(acsr_peer *p, double *delta2, int32_t *ctrl, double eps2,
                             cudaStream_t stream);
/* HOST query (synchronous copy): pushes completed by this rank, the error word, and
 * the local buffer holding the last push (NULL before the first push). */
acsr_status acsr_peer_query(const acsr_peer *p, int64_t *pushes, int32_t *error,
                            const double **xs_current);
/* dst: [xs_len] device; receives (stream-ordered) this rank's replicated xs as left by
 * the last push (zeros before the first push). */
acsr_status acsr_peer_read_xs(const acsr_peer *p, double *dst, cudaStream_t stream);

/* ------------------------------------------------------------------------ */
/* HITS normalisation (Eq. 5-7).  The HITS step is one acsr_spmv on the
 * 2n x 2n pattern matrix [[0, A^T], [A, 0]] applied to v = [a; h] (Eq. 7); this call
 * then scales each half of y = [A^T h; A a] to unit Euclidean norm (reading R6; a zero
 * half stays zero) into v_next and writes dist2[0] = ||a' - a||^2, dist2[1] =
 * ||h' - h||^2 (the convergence test "until both ... converge", with the
 * Euclidean distance of P:326).  Deterministic (fixed reduction order).
 * y, v, v_next: [2n] device doubles; dist2: [2] device. */
size_t acsr_hits_workspace_bytes(int64_t n);
acsr_status acsr_hits_normalize(int64_t n, const double *y, const double *v, double *v_next,
                                double *dist2, void *ws, size_t ws_bytes, cudaStream_t stream);
/* The same with device-side convergence (as acsr_pr_args.ctrl): ctrl NULL or [2] device;
 * a call with ctrl[0] != 0 does nothing; otherwise ctrl[1] += 1 and ctrl[0] = 1 once both
 * dist2[0] and dist2[1] are <= eps2.  Lets the host enqueue blocks of (acsr_spmv,
 * acsr_hits_normalize_ctrl) iterations between synchronisations with the results of a test
 * after every iteration (the iterate after k executed iterations is in buffer k mod 2). */
acsr_status acsr_hits_normalize_ctrl(int64_t n, const double *y, const double *v, double *v_next,
                                     double *dist2, int32_t *ctrl, double eps2, void *ws, size_t ws_bytes,
                                     cudaStream_t stream);

/* ------------------------------------------------------------------------ */
/* Degree-ordered vertex relabelling of a PageRank in-link graph (an application-level
 * preprocessing option for large graphs -- C4 -- not part of ACSR).  Alg. 5 (P:279-291,
 * reading Q12) gathers xs[u] = x_u / outdeg_u for every in-link u -> v; renumbering the
 * vertices by decreasing out-degree packs the most gathered entries of xs at the front of
 * the vector, where they stay in L2.  Rows and columns get the same permutation (P A P^T),
 * so every kernel runs unchanged and PR in the original numbering is x'[perm[v]].  The
 * graph persists across the dynamic-graph epochs, so the relabel is paid once.
 *   row_ptr [n+1], col_idx [nnz]   the in-link CSR (standard; row v = sources of v)
 *   outdeg [n]                     out-degree of every vertex
 *   row_ptr_out [n+1], col_out [nnz], outdeg_out [n]   the relabelled graph
 *   perm_out [n]                   perm_out[v] = new id of old vertex v
 * Order: decreasing out-degree, ties by increasing old id (stable).  Entry j of old row u
 * becomes entry j of new row perm[u] (column order inside a row kept), or -- with flag
 * ACSR_RELABEL_SORT_ROWS -- every new row's columns are sorted ascending (the hot, now small,
 * column ids of a row sit together: fewer 128-byte lines per warp gather).  col_idx/col_out
 * may be NULL (permutation and row pointers only).  Outputs must not alias the inputs.
 * nnz = row_ptr[n] (sizes the workspace of the row sort).  Everything runs on `stream` (CUB
 * radix sort + scan, two copy kernels, CUB segmented sort; no host sync).  Unknown flag
 * bits -> ACSR_ERR_INVALID_VALUE. */
enum { ACSR_RELABEL_SORT_ROWS = 1u };
size_t acsr_relabel_workspace_bytes(int64_t n, int64_t nnz, unsigned flags);
acsr_status acsr_degree_relabel(int64_t n, int64_t nnz, const int32_t *row_ptr, const int32_t *col_idx,
                                const int32_t *outdeg, int32_t *row_ptr_out, int32_t *col_out, int32_t *outdeg_out,
                                int32_t *perm_out, unsigned flags, void *ws, size_t ws_bytes, cudaStream_t stream);

/* ------------------------------------------------------------------------ */
/* Dynamic-graph update (§VII): for update i (row r = upd_rows[i],
 * upd_rows strictly increasing) delete every entry whose column is in
 * del_cols[del_ptr[i] .. del_ptr[i+1]) (sorted, non-decreasing), compact the
 * row keeping order ("compresses (shifts columns) the row"), then append
 * ins_cols[ins_ptr[i] .. ins_ptr[i+1]) in order (with ins_vals, or 1 for a
 * pattern matrix).  outdeg (nullable, [n_cols]) gets -1 per removed and +1 per
 * inserted entry.  Reading Q13: the batch is all-or-nothing -- it is first
 * validated for every i in order:
 *   (a) 0 <= upd_rows[i] < n_rows and upd_rows[i] > upd_rows[i-1]   INVALID_VALUE
 *   (b) delete list non-decreasing                                   INVALID_VALUE
 *   (c) 0 <= insert column < n_cols                                  INVALID_VALUE
 *   (d) kept + inserted <= row_cap[r]                                CAPACITY
 * status[0] = code of the smallest failing i (ACSR_OK if none), status[1] = that
 * i (or -1).  On failure nothing is modified (bitwise).  del_ptr/del_cols may be
 * NULL (insert-only batch).  Re-run acsr_bin afterwards. */
size_t acsr_update_workspace_bytes(int64_t n_upd);

acsr_status acsr_update_edges(acsr_dtype dt, int64_t n_rows, int64_t n_cols,
                              const int32_t *row_begin, int32_t *row_end, const int32_t *row_cap,
                              int32_t *col_idx, void *values /* NULL => pattern */,
                              int64_t n_upd, const int32_t *upd_rows,
                              const int32_t *del_ptr, const int32_t *del_cols,
                              const int32_t *ins_ptr, const int32_t *ins_cols,
                              const void *ins_vals /* NULL => ones */,
                              int32_t *outdeg /* NULL or [n_cols] */,
                              int32_t *status /* [2] out */,
                              void *ws, size_t ws_bytes, cudaStream_t stream);

/* acsr_update_edges with the batch size read on the DEVICE: n_upd_dev[0] (int64) updates
 * are applied, n_upd_max (>= it) sizes the launch and the workspace.  The launch
 * configuration no longer depends on the batch, so the per-batch sequence (update ->
 * acsr_bin -> ... -> acsr_spmv) can be captured into a CUDA graph once and replayed for
 * every batch with the change lists copied into fixed buffers (CUDA graphs
 * for the C5 update + re-bin + SpMV sequence).  A device count outside [0, n_upd_max]
 * rejects the batch (status {ACSR_ERR_INVALID_VALUE, 0}, nothing modified). */
acsr_status acsr_update_edges_dev(acsr_dtype dt, int64_t n_rows, int64_t n_cols,
                                  const int32_t *row_begin, int32_t *row_end, const int32_t *row_cap,
                                  int32_t *col_idx, void *values /* NULL => pattern */,
                                  int64_t n_upd_max, const int64_t *n_upd_dev /* [1] device */,
                                  const int32_t *upd_rows,
                                  const int32_t *del_ptr, const int32_t *del_cols,
                                  const int32_t *ins_ptr, const int32_t *ins_cols,
                                  const void *ins_vals /* NULL => ones */,
                                  int32_t *outdeg /* NULL or [n_cols] */,
                                  int32_t *status /* [2] out */,
                                  void *ws, size_t ws_bytes, cudaStream_t stream);

/* Re-layout of a slack CSR (§VII keeps "some additional memory ... at the end of
 * each CSR row"; what happens when a row outgrows it is unstated -- reading
 * R4 in DESIGN.md: after a CAPACITY rejection the caller re-lays the matrix out with
 * larger capacities and re-submits the batch).  Row r is copied, in order, from
 * [old_begin[r], old_end[r]) to [new_begin[r], new_begin[r] + len); new_end[r] is
 * set.  new_begin (with the capacities it implies) is chosen by the caller; the
 * new arrays must not overlap the old ones.  Values are moved as opaque 4/8-byte
 * items (NULL/NULL = pattern). */
acsr_status acsr_relayout(acsr_dtype dt, int64_t n_rows,
                          const int32_t *old_begin, const int32_t *old_end,
                          const int32_t *old_col, const void *old_val,
                          const int32_t *new_begin, int32_t *new_end,
                          int32_t *new_col, void *new_val, cudaStream_t stream);

/* The grown layout of reading R4, on the device: for every row
 *   new_cap[r]   = max(cap_r + max(min_slack, ceil(cap_r / frac)),
 *                      len_r + max(min_slack, ceil(len_r / frac)))      (every row grows)
 *   new_begin[r] = sum_{r' < r} new_cap[r']                             (exclusive prefix)
 * and total[0] = sum of new_cap (int64, DEVICE; the caller allocates total entries for the
 * new col / val arrays and checks total < 2^31 before acsr_relayout).  min_slack >= 1,
 * frac >= 1.  ws: acsr_grow_workspace_bytes(n_rows) bytes. */
size_t acsr_grow_workspace_bytes(int64_t n_rows);
acsr_status acsr_grow_layout(int64_t n_rows, const int32_t *row_begin, const int32_t *row_end,
                             const int32_t *row_cap, int32_t min_slack, int32_t frac, int32_t *new_begin,
                             int32_t *new_cap, int64_t *total, void *ws, size_t ws_bytes, cudaStream_t stream);

/* ------------------------------------------------------------------------ */
const char *acsr_status_string(acsr_status s);
const char *acsr_last_error(void); /* thread-local detail of the last failure */
int acsr_version(void);             /* 100 * major + minor */

#ifdef __cplusplus
}
#endif
#endif /* ACSR_H */
