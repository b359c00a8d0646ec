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
    printf("capi_smoke %s (version %d)\n", ok ? "OK" : "FAIL", acsr_version());
    return ok ? 0 : 1;
}
