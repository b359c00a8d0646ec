/* capi_smoke.c -- drives libacsr.so through the plain C ABI (include/acsr.h) with no
 * Python/torch: a 6-row CSR covering several bins, acsr_bin + acsr_spmv on a stream,
 * result checked against a hand-computed y = A x.  Exit code 0 = pass. */
#include <math.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <cuda_runtime_api.h>

#include "../../include/acsr.h"

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { printf("cuda %s\n", cudaGetErrorString(e_)); return 2; } } while (0)
#define AK(x) do { acsr_status s_ = (x); if (s_ != ACSR_OK) { printf("acsr %s: %s\n", acsr_status_string(s_), acsr_last_error()); return 3; } } while (0)

int main(void)
{
    /* rows: lengths 0, 1, 3, 5, 70, 1500 (bins 0, 1, 2, 3, 7, 11 -> split rows) */
    const int lens[6] = {0, 1, 3, 5, 70, 1500};
    const int n = 6, n_cols = 2000;
    int rp[7];
    rp[0] = 0;
    for (int r = 0; r < n; r++) rp[r + 1] = rp[r] + lens[r];
    const int nnz = rp[n];
    int *col = (int *)malloc(sizeof(int) * nnz);
    double *val = (double *)malloc(sizeof(double) * nnz), *x = (double *)malloc(sizeof(double) * n_cols);
    for (int k = 0; k < nnz; k++) {
        col[k] = (k * 37) % n_cols;
        val[k] = (double)((k % 7) - 3);
    }
    for (int c = 0; c < n_cols; c++) x[c] = (double)((c % 5) - 2);
    double y_ref[6];
    for (int r = 0; r < n; r++) {
        y_ref[r] = 0.0;
        for (int k = rp[r]; k < rp[r + 1]; k++) y_ref[r] += val[k] * x[col[k]]; /* integers: exact */
    }
    int *d_rp, *d_col, *d_bins, *d_off;
    double *d_val, *d_x, *d_y;
    void *d_ws;
    size_t ws_bytes = acsr_bin_workspace_bytes(n, n_cols, nnz);
    CK(cudaMalloc((void **)&d_rp, sizeof(rp)));
    CK(cudaMalloc((void **)&d_col, sizeof(int) * nnz));
    CK(cudaMalloc((void **)&d_val, sizeof(double) * nnz));
    CK(cudaMalloc((void **)&d_x, sizeof(double) * n_cols));
    CK(cudaMalloc((void **)&d_y, sizeof(double) * n));
    CK(cudaMalloc((void **)&d_bins, sizeof(int) * n));
    CK(cudaMalloc((void **)&d_off, sizeof(int) * (ACSR_NBINS + 1)));
    CK(cudaMalloc(&d_ws, ws_bytes));
    CK(cudaMemcpy(d_rp, rp, sizeof(rp), cudaMemcpyHostToDevice));
    CK(cudaMemcpy(d_col, col, sizeof(int) * nnz, cudaMemcpyHostToDevice));
    CK(cudaMemcpy(d_val, val, sizeof(double) * nnz, cudaMemcpyHostToDevice));
    CK(cudaMemcpy(d_x, x, sizeof(double) * n_cols, cudaMemcpyHostToDevice));
    cudaStream_t st;
    CK(cudaStreamCreate(&st));
    AK(acsr_bin(n, n_cols, nnz, d_rp, NULL, d_col, d_bins, d_off, d_ws, ws_bytes, st));
    AK(acsr_spmv(ACSR_F64, n, n_cols, d_rp, NULL, d_col, d_val, d_x, d_y, d_bins, d_off, d_ws, ws_bytes, st));
    CK(cudaStreamSynchronize(st));
    double y[6];
    int off[ACSR_NBINS + 1], bins[6];
    CK(cudaMemcpy(y, d_y, sizeof(y), cudaMemcpyDeviceToHost));
    CK(cudaMemcpy(off, d_off, sizeof(off), cudaMemcpyDeviceToHost));
    CK(cudaMemcpy(bins, d_bins, sizeof(bins), cudaMemcpyDeviceToHost));
    const int exp_bins[6] = {0, 1, 2, 3, 4, 5}; /* rows are already in bin order here */
    int ok = off[ACSR_NBINS] == n;
    for (int r = 0; r < n; r++) ok &= (y[r] == y_ref[r]) && (bins[r] == exp_bins[r]);
    /* host-detected errors return synchronously */
    ok &= acsr_spmv(ACSR_F64, -1, 0, NULL, NULL, NULL, NULL, NULL, NULL, NULL, NULL, NULL, 0, st) == ACSR_ERR_INVALID_VALUE;
    ok &= acsr_bin(n, n_cols, nnz, d_rp, NULL, d_col, d_bins, d_off, d_ws, 8, st) == ACSR_ERR_WORKSPACE;

    /* the peer-exchange PageRank path, one rank: the same rows as an in-link pattern over
     * an xs of n_cols slots; this rank's slice = slots [0, n) */
    acsr_peer *peer = NULL;
    char handle[ACSR_IPC_HANDLE_BYTES];
    AK(acsr_peer_create(&peer, 1, 0, n_cols, 0, n, handle));
    AK(acsr_peer_open(peer, handle));
    const int od[6] = {1, 2, 3, 1, 2, 1};
    double x0[6], xn[6];
    for (int r = 0; r < n; r++) x0[r] = 1.0 / (r + 2);
    int *d_od;
    double *d_x0, *d_xn, *d_d2, *d_d2g, *d_xsr;
    CK(cudaMalloc((void **)&d_od, sizeof(od)));
    CK(cudaMalloc((void **)&d_x0, sizeof(x0)));
    CK(cudaMalloc((void **)&d_xn, sizeof(xn)));
    CK(cudaMalloc((void **)&d_d2, sizeof(double)));
    CK(cudaMalloc((void **)&d_d2g, sizeof(double)));
    CK(cudaMalloc((void **)&d_xsr, sizeof(double) * n_cols));
    CK(cudaMemcpy(d_od, od, sizeof(od), cudaMemcpyHostToDevice));
    CK(cudaMemcpy(d_x0, x0, sizeof(x0), cudaMemcpyHostToDevice));
    AK(acsr_peer_push(peer, n, d_x0, d_od, NULL, st));
    const double damping = 0.85, teleport = (1.0 - 0.85) / n;
    acsr_pr_args a;
    memset(&a, 0, sizeof(a));
    a.n_rows = n; a.n_cols = n_cols; a.row_begin = d_rp; a.col_idx = d_col;
    a.bin_rows = d_bins; a.bin_offsets = d_off; a.plan_ws = d_ws; a.plan_ws_bytes = ws_bytes;
    a.x = d_x0; a.outdeg = d_od; a.x_new = d_xn; a.xs_next = NULL;
    a.damping = damping; a.teleport = teleport; a.delta2 = d_d2; a.restart = -1; a.eps2 = -1.0;
    AK(acsr_pagerank_step_peer(&a, peer, st));
    AK(acsr_peer_delta2(peer, d_d2g, NULL, 0.0, st));
    AK(acsr_peer_read_xs(peer, d_xsr, st));
    CK(cudaStreamSynchronize(st));
    double *xsr = (double *)malloc(sizeof(double) * n_cols), d2g;
    CK(cudaMemcpy(xn, d_xn, sizeof(xn), cudaMemcpyDeviceToHost));
    CK(cudaMemcpy(xsr, d_xsr, sizeof(double) * n_cols, cudaMemcpyDeviceToHost));
    CK(cudaMemcpy(&d2g, d_d2g, sizeof(double), cudaMemcpyDeviceToHost));
    double d2_ref = 0.0;
    for (int r = 0; r < n; r++) {
        double s = 0.0, den = 0.0; /* Alg. 5 on the pattern: sum of xs over the row */
        for (int k = rp[r]; k < rp[r + 1]; k++) {
            const int c = col[k];
            const double xs = c < n ? x0[c] / od[c] : 0.0;
            s += xs;
            den += xs;
        }
        const double ref = teleport + damping * s;
        ok &= fabs(xn[r] - ref) <= 1e-12 * (teleport + damping * den);
        ok &= xsr[r] == xn[r] / od[r]; /* the pushed slice: IEEE division of x_new */
        d2_ref += (ref - x0[r]) * (ref - x0[r]);
    }
    for (int c = n; c < n_cols; c++) ok &= xsr[c] == 0.0; /* slots nobody owns stay +0.0 */
    ok &= fabs(d2g - d2_ref) <= 1e-12 * d2_ref;
    int64_t pushes = -1;
    int32_t perr = -1;
    const double *cur = NULL;
    AK(acsr_peer_query(peer, &pushes, &perr, &cur));
    ok &= pushes == 2 && perr == 0 && cur != NULL;
    ok &= acsr_peer_create(&peer, 9, 0, 10, 0, 5, handle) == ACSR_ERR_INVALID_VALUE;
    AK(acsr_peer_destroy(peer));

    /* the library-owned NCCL exchange, one rank: acsr_pagerank_init + acsr_pagerank_step
     * with comm (in-place all-gather of the slice, global Delta^2 from the exact partials)
     * gives the same x_new as the peer step above and the same Delta^2 */
    char uid[ACSR_COMM_ID_BYTES];
    acsr_comm *comm = NULL;
    AK(acsr_comm_get_unique_id(uid));
    AK(acsr_comm_init(&comm, 1, 0, uid));
    int nr = 0, rk = -1;
    AK(acsr_comm_query(comm, &nr, &rk));
    ok &= nr == 1 && rk == 0;
    double *d_xa, *d_xb, *d_xn2, *d_d2c;
    int32_t *d_ctrl;
    CK(cudaMalloc((void **)&d_xa, sizeof(double) * n_cols));
    CK(cudaMalloc((void **)&d_xb, sizeof(double) * n_cols));
    CK(cudaMalloc((void **)&d_xn2, sizeof(xn)));
    CK(cudaMalloc((void **)&d_d2c, sizeof(double)));
    CK(cudaMalloc((void **)&d_ctrl, 2 * sizeof(int32_t)));
    CK(cudaMemset(d_xa, 0, sizeof(double) * n_cols));
    CK(cudaMemset(d_xb, 0, sizeof(double) * n_cols));
    CK(cudaMemset(d_ctrl, 0, 2 * sizeof(int32_t)));
    acsr_pr_args c;
    memset(&c, 0, sizeof(c));
    c.n_rows = n; c.n_cols = n_cols; c.row_begin = d_rp; c.col_idx = d_col;
    c.bin_rows = d_bins; c.bin_offsets = d_off; c.plan_ws = d_ws; c.plan_ws_bytes = ws_bytes;
    c.x = d_x0; c.outdeg = d_od; c.xs_next = d_xa; c.comm = comm; c.xs_all = d_xa; c.slice_len = n;
    AK(acsr_pagerank_init(&c, st));
    c.xs = d_xa; c.x_new = d_xn2; c.xs_next = d_xb; c.xs_all = d_xb;
    c.damping = damping; c.teleport = teleport; c.delta2 = d_d2c; c.restart = -1;
    c.ctrl = d_ctrl; c.eps2 = 1e300; /* converges on the first step: ctrl[0] = 1, ctrl[1] = 1 */
    AK(acsr_pagerank_step(&c, st));
    CK(cudaStreamSynchronize(st));
    double xn2[6], d2c;
    int32_t ctrl[2];
    CK(cudaMemcpy(xn2, d_xn2, sizeof(xn2), cudaMemcpyDeviceToHost));
    CK(cudaMemcpy(&d2c, d_d2c, sizeof(double), cudaMemcpyDeviceToHost));
    CK(cudaMemcpy(ctrl, d_ctrl, sizeof(ctrl), cudaMemcpyDeviceToHost));
    for (int r = 0; r < n; r++) ok &= xn2[r] == xn[r];
    ok &= d2c == d2g && ctrl[0] == 1 && ctrl[1] == 1;
    /* with comm, xs_all is required */
    c.xs_all = NULL;
    ok &= acsr_pagerank_step(&c, st) == ACSR_ERR_INVALID_VALUE;
    /* all-gather-v with one rank: count 2 of a 3-double slice; the third entry untouched */
    double hsend[3] = {1.5, -2.5, 9.0}, hrecv[3] = {0.0, 0.0, 7.0};
    double *d_send, *d_recv;
    CK(cudaMalloc((void **)&d_send, sizeof(hsend)));
    CK(cudaMalloc((void **)&d_recv, sizeof(hrecv)));
    CK(cudaMemcpy(d_send, hsend, sizeof(hsend), cudaMemcpyHostToDevice));
    CK(cudaMemcpy(d_recv, hrecv, sizeof(hrecv), cudaMemcpyHostToDevice));
    const int64_t cnt_bytes[1] = {2 * sizeof(double)};
    AK(acsr_comm_allgatherv(comm, d_send, d_recv, sizeof(hrecv), cnt_bytes, st));
    CK(cudaStreamSynchronize(st));
    CK(cudaMemcpy(hrecv, d_recv, sizeof(hrecv), cudaMemcpyDeviceToHost));
    ok &= hrecv[0] == 1.5 && hrecv[1] == -2.5 && hrecv[2] == 7.0;
    AK(acsr_comm_destroy(comm));

    /* O8 partition on the device, and a valid plan reports ACSR_OK */
    int64_t *d_splits, splits[3];
    void *d_pws;
    size_t pws = acsr_partition_workspace_bytes(n);
    CK(cudaMalloc((void **)&d_splits, sizeof(splits)));
    CK(cudaMalloc(&d_pws, pws));
    AK(acsr_partition(n, d_rp, NULL, 4, 36, 2, 1, d_splits, d_pws, pws, st));
    CK(cudaStreamSynchronize(st));
    CK(cudaMemcpy(splits, d_splits, sizeof(splits), cudaMemcpyDeviceToHost));
    /* costs 36, 40, 48, 56, 316, 6036 (total 6532): the prefix before row r first reaches
     * ceil(6532 / 2) = 3266 at r = 6 (the last row holds most of the cost) */
    ok &= splits[0] == 0 && splits[1] == 6 && splits[2] == 6;
    AK(acsr_plan_status(d_ws, ws_bytes, st));
    printf("capi_smoke %s (version %d)\n", ok ? "OK" : "FAIL", acsr_version());
    return ok ? 0 : 1;
}
