/*
 * oracle/wino_oracle.c -- TEST INFRASTRUCTURE ONLY.
 *
 * Plain, slow, obviously-correct fp64 CPU reference for the fused batched
 * Winograd F(2x2,3x3) forward convolution of Yan, Wang & Chu, "Optimizing
 * Batched Winograd Convolution on GPUs" (PPoPP'20).  Citations are lines of
 * /root/reference/PAPER.md ("L<n>") plus the paper's section / equation.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / reference
 * arm may load this library.  It shares NO code, header, table or constant with
 * the CUDA path (paper_conf_ppopp_yanwc20_b200/csrc) and includes nothing from it.
 *
 * Layouts (Table 4), all dense, row-major, fp64 here:
 *   x  (C,H,W,N)  "CHWN", N contiguous
 *   w  (C,3,3,K)  "CRSK", K contiguous
 *   u  (C,4,4,K)  "CR'S'K", element (r',s') of G w G^T at index 4r'+s'
 *                 (reading R6 / SURVEY 8(c) c6)
 *   y  (K,H,W,N)  "KHWN"
 * Readings of the paper: pad = 1, stride = 1, output
 * H x W (Table 1), 0-based correlation without filter flip (Eq. 4
 * with 1-based r,s and the implicit zero padding of Sec. 3.5), ceil(H/2) x
 * ceil(W/2) output tiles whose out-of-range outputs are discarded (L1155).
 *
 * Parallelism: OpenMP over independent outputs only; every output value is a
 * sum evaluated in one fixed, documented order, so results are deterministic.
 */
#include <stddef.h>
#include <stdint.h>
#ifdef _OPENMP
#include <omp.h>
#endif

/* ---- Eq. 2-3 (L89-113), reconstructed from the garbled scrape as the
 *      Lavin-Gray F(2x2,3x3) matrices (readings R1, R2). ---------- */
static const double AT[2][4] = {{1.0, 1.0, 1.0, 0.0},
                                {0.0, 1.0, -1.0, -1.0}};
static const double G[4][3] = {{1.0, 0.0, 0.0},
                               {0.5, 0.5, 0.5},
                               {0.5, -0.5, 0.5},
                               {0.0, 0.0, 1.0}};
static const double BT[4][4] = {{1.0, 0.0, -1.0, 0.0},
                                {0.0, 1.0, 1.0, 0.0},
                                {0.0, -1.0, 1.0, 0.0},
                                {0.0, 1.0, 0.0, -1.0}};

int oracle_num_threads(void) {
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}

/* Thread count of the following calls (plumbing only: bench.py gives each of P ranks
 * sharing one host cores/P threads; torchrun's OMP_NUM_THREADS=1 would serialise it). */
void oracle_set_num_threads(int n) {
#ifdef _OPENMP
    if (n > 0) omp_set_num_threads(n);
#else
    (void)n;
#endif
}

/* x-hat of Eq. 4 with implicit zero padding (Sec. 3.5): x inside
 * [0,H) x [0,W), 0 outside. */
static inline double xhat(const double* x, int N, int H, int W, int c, int h, int w, int n) {
    if (h < 0 || h >= H || w < 0 || w >= W) return 0.0;
    return x[(((size_t)c * H + h) * W + w) * N + n];
}

/* ------------------------------------------------------------------------- *
 * Eq. 4 (Sec. 3.1): the batched direct 3x3 convolution,
 *   y[k,i,j,n] = sum_c sum_r sum_s xhat[c, i+r-1, j+s-1, n] * w[c,r,s,k]
 * for 0 <= i < H, 0 <= j < W.  Summation order: c outer, then r, then s.
 * ------------------------------------------------------------------------- */
void oracle_direct_conv(const double* x, const double* w, double* y,
                        int N, int C, int H, int W, int K) {
    long total = (long)K * H;
#pragma omp parallel for schedule(dynamic, 1)
    for (long ki = 0; ki < total; ++ki) {
        int k = (int)(ki / H), i = (int)(ki % H);
        for (int j = 0; j < W; ++j) {
            double* yrow = y + (((size_t)k * H + i) * W + j) * N;
            for (int n = 0; n < N; ++n) yrow[n] = 0.0;
            for (int c = 0; c < C; ++c)
                for (int r = 0; r < 3; ++r)
                    for (int s = 0; s < 3; ++s) {
                        int h = i + r - 1, ww = j + s - 1;
                        if (h < 0 || h >= H || ww < 0 || ww >= W) continue; /* xhat = 0 */
                        double f = w[(((size_t)c * 3 + r) * 3 + s) * K + k];
                        const double* xrow = x + (((size_t)c * H + h) * W + ww) * N;
                        for (int n = 0; n < N; ++n) yrow[n] += xrow[n] * f;
                    }
        }
    }
}

/* Eq. 4 evaluated at selected output points only; idx holds n_pts quadruples
 * (k, i, j, n).  Same summation order as oracle_direct_conv, so results are
 * bit-identical to the corresponding entries of the full computation. */
void oracle_direct_sample(const double* x, const double* w,
                          int N, int C, int H, int W, int K,
                          const int64_t* idx, long n_pts, double* out) {
#pragma omp parallel for schedule(static)
    for (long p = 0; p < n_pts; ++p) {
        int k = (int)idx[4 * p + 0], i = (int)idx[4 * p + 1];
        int j = (int)idx[4 * p + 2], n = (int)idx[4 * p + 3];
        double acc = 0.0;
        for (int c = 0; c < C; ++c)
            for (int r = 0; r < 3; ++r)
                for (int s = 0; s < 3; ++s) {
                    int h = i + r - 1, ww = j + s - 1;
                    if (h < 0 || h >= H || ww < 0 || ww >= W) continue;
                    acc += x[(((size_t)c * H + h) * W + ww) * N + n] *
                           w[(((size_t)c * 3 + r) * 3 + s) * K + k];
                }
        (void)K;
        out[p] = acc;
    }
}

/* ------------------------------------------------------------------------- *
 * Eq. 5 (L191): filter transform (FTF) U[c,k] = G * w[c,:,:,k] * G^T,
 * written out as two plain matrix products.  Output in (C,4,4,K).
 * ------------------------------------------------------------------------- */
static void ftf_tile(const double g[3][3], double u[4][4]) {
    double t[4][3]; /* t = G g */
    for (int a = 0; a < 4; ++a)
        for (int b = 0; b < 3; ++b) {
            double s = 0.0;
            for (int m = 0; m < 3; ++m) s += G[a][m] * g[m][b];
            t[a][b] = s;
        }
    for (int a = 0; a < 4; ++a) /* u = t G^T */
        for (int b = 0; b < 4; ++b) {
            double s = 0.0;
            for (int m = 0; m < 3; ++m) s += t[a][m] * G[b][m];
            u[a][b] = s;
        }
}

void oracle_filter_transform(const double* w, double* u, int C, int K) {
#pragma omp parallel for schedule(static)
    for (long ck = 0; ck < (long)C * K; ++ck) {
        int c = (int)(ck / K), k = (int)(ck % K);
        double g[3][3], t[4][4];
        for (int r = 0; r < 3; ++r)
            for (int s = 0; s < 3; ++s) g[r][s] = w[(((size_t)c * 3 + r) * 3 + s) * K + k];
        ftf_tile(g, t);
        for (int a = 0; a < 4; ++a)
            for (int b = 0; b < 4; ++b) u[(((size_t)c * 4 + a) * 4 + b) * K + k] = t[a][b];
    }
}

/* Eq. 6 (L193-195): input transform V = B^T d B of one 4x4 tile. */
static void itf_tile(const double d[4][4], double v[4][4]) {
    double t[4][4]; /* t = B^T d */
    for (int a = 0; a < 4; ++a)
        for (int b = 0; b < 4; ++b) {
            double s = 0.0;
            for (int m = 0; m < 4; ++m) s += BT[a][m] * d[m][b];
            t[a][b] = s;
        }
    for (int a = 0; a < 4; ++a) /* v = t B, B[m][b] = BT[b][m] */
        for (int b = 0; b < 4; ++b) {
            double s = 0.0;
            for (int m = 0; m < 4; ++m) s += t[a][m] * BT[b][m];
            v[a][b] = s;
        }
}

/* Eq. 8 (L205-207): output transform Y = A^T M A of one 4x4 tile. */
static void otf_tile(const double m[4][4], double o[2][2]) {
    double t[2][4]; /* t = A^T m */
    for (int a = 0; a < 2; ++a)
        for (int b = 0; b < 4; ++b) {
            double s = 0.0;
            for (int q = 0; q < 4; ++q) s += AT[a][q] * m[q][b];
            t[a][b] = s;
        }
    for (int a = 0; a < 2; ++a) /* o = t A, A[q][b] = AT[b][q] */
        for (int b = 0; b < 2; ++b) {
            double s = 0.0;
            for (int q = 0; q < 4; ++q) s += t[a][q] * AT[b][q];
            o[a][b] = s;
        }
}

/* Single-tile entry points (test pins on the transforms themselves). */
void oracle_ftf_tile(const double* g9, double* u16) {
    double g[3][3], u[4][4];
    for (int i = 0; i < 9; ++i) g[i / 3][i % 3] = g9[i];
    ftf_tile(g, u);
    for (int i = 0; i < 16; ++i) u16[i] = u[i / 4][i % 4];
}
void oracle_itf_tile(const double* d16, double* v16) {
    double d[4][4], v[4][4];
    for (int i = 0; i < 16; ++i) d[i / 4][i % 4] = d16[i];
    itf_tile(d, v);
    for (int i = 0; i < 16; ++i) v16[i] = v[i / 4][i % 4];
}
void oracle_otf_tile(const double* m16, double* o4) {
    double m[4][4], o[2][2];
    for (int i = 0; i < 16; ++i) m[i / 4][i % 4] = m16[i];
    otf_tile(m, o);
    for (int i = 0; i < 4; ++i) o4[i] = o[i / 2][i % 2];
}

/* ------------------------------------------------------------------------- *
 * Naive Winograd convolution, Eq. 5-8 (L191-207) in the paper's order:
 *   1. U[c,k]          = G w[c,k] G^T                        (Eq. 5)
 *   2. V[c,th,tw,n]    = B^T d B, d = xhat[c, 2th-1..2th+2, 2tw-1..2tw+2, n] (Eq. 6)
 *   3. M[k,th,tw,n]    = sum_c U[c,k] (.) V[c,th,tw,n]          (Eq. 7)
 *   4. Y               = A^T M A, scattered to y[k, 2th+a, 2tw+b, n],
 *                        dropping 2th+a >= H or 2tw+b >= W      (Eq. 8)
 * u_out (optional, may be NULL) receives U in (C,4,4,K).
 * Parallel over tile positions (th,tw); each tile's V for all (c,n) is kept in
 * a per-thread buffer of 16*C*N doubles.
 * ------------------------------------------------------------------------- */
#include <stdlib.h>
int oracle_winograd_conv(const double* x, const double* w, double* y, double* u_out,
                         int N, int C, int H, int W, int K) {
    double* U = u_out ? u_out : (double*)malloc(sizeof(double) * 16 * (size_t)C * K);
    if (!U) return 1;
    oracle_filter_transform(w, U, C, K);
    int TH = (H + 1) / 2, TW = (W + 1) / 2;
    int failed = 0;
#pragma omp parallel
    {
        double* V = (double*)malloc(sizeof(double) * 16 * (size_t)C * N);
        if (!V) {
#pragma omp atomic write
            failed = 1;
        }
#pragma omp for schedule(dynamic, 1)
        for (long t = 0; t < (long)TH * TW; ++t) {
            if (!V) continue;
            int th = (int)(t / TW), tw = (int)(t % TW);
            for (int c = 0; c < C; ++c)
                for (int n = 0; n < N; ++n) {
                    double d[4][4], v[4][4];
                    for (int a = 0; a < 4; ++a)
                        for (int b = 0; b < 4; ++b)
                            d[a][b] = xhat(x, N, H, W, c, 2 * th - 1 + a, 2 * tw - 1 + b, n);
                    itf_tile(d, v);
                    for (int e = 0; e < 16; ++e) V[((size_t)c * N + n) * 16 + e] = v[e / 4][e % 4];
                }
            for (int k = 0; k < K; ++k)
                for (int n = 0; n < N; ++n) {
                    double m[4][4], o[2][2];
                    for (int e = 0; e < 16; ++e) m[e / 4][e % 4] = 0.0;
                    for (int c = 0; c < C; ++c)
                        for (int e = 0; e < 16; ++e)
                            m[e / 4][e % 4] += U[((size_t)c * 16 + e) * K + k] *
                                               V[((size_t)c * N + n) * 16 + e];
                    otf_tile(m, o);
                    for (int a = 0; a < 2; ++a)
                        for (int b = 0; b < 2; ++b) {
                            int i = 2 * th + a, j = 2 * tw + b;
                            if (i < H && j < W) y[(((size_t)k * H + i) * W + j) * N + n] = o[a][b];
                        }
                }
        }
        free(V);
    }
    if (!u_out) free(U);
    return failed;
}

/* ========================================================================= *
 * NEXT row N1: Winograd F(4x4,3x3).  PAPER.md only points to
 * the matrices ("the transformation matrices for ... F(4x4,3x3) ... are also
 * given in [11, 26]", L117; "We expect greater speedup in the future if the
 * fused F(4x4,3x3) is well optimized", L1271).  The matrices below are the
 * Lavin-Gray F(4x4,3x3) ones (interpolation points 0, +-1, +-2, inf); they are
 * pinned by the exact-rational identity tests (tests/test_oracle.py), not by
 * the paper's text.  Same steps as Eq. 5-8 with alpha = 6, 4x4 outputs per tile.
 * ========================================================================= */
static const double AT4[4][6] = {{1, 1, 1, 1, 1, 0},
                                 {0, 1, -1, 2, -2, 0},
                                 {0, 1, 1, 4, 4, 0},
                                 {0, 1, -1, 8, -8, 1}};
static const double G4[6][3] = {{1.0 / 4, 0, 0},
                                {-1.0 / 6, -1.0 / 6, -1.0 / 6},
                                {-1.0 / 6, 1.0 / 6, -1.0 / 6},
                                {1.0 / 24, 1.0 / 12, 1.0 / 6},
                                {1.0 / 24, -1.0 / 12, 1.0 / 6},
                                {0, 0, 1}};
static const double BT4[6][6] = {{4, 0, -5, 0, 1, 0},
                                 {0, -4, -4, 1, 1, 0},
                                 {0, 4, -4, -1, 1, 0},
                                 {0, -2, -1, 2, 1, 0},
                                 {0, 2, -1, -2, 1, 0},
                                 {0, 4, 0, -5, 0, 1}};

/* U = G4 g G4^T (6x6) */
void oracle_ftf4_tile(const double* g9, double* u36) {
    double t[6][3];
    for (int a = 0; a < 6; ++a)
        for (int b = 0; b < 3; ++b) {
            double s = 0.0;
            for (int m = 0; m < 3; ++m) s += G4[a][m] * g9[m * 3 + b];
            t[a][b] = s;
        }
    for (int a = 0; a < 6; ++a)
        for (int b = 0; b < 6; ++b) {
            double s = 0.0;
            for (int m = 0; m < 3; ++m) s += t[a][m] * G4[b][m];
            u36[a * 6 + b] = s;
        }
}
/* V = BT4 d BT4^T (6x6) */
void oracle_itf4_tile(const double* d36, double* v36) {
    double t[6][6];
    for (int a = 0; a < 6; ++a)
        for (int b = 0; b < 6; ++b) {
            double s = 0.0;
            for (int m = 0; m < 6; ++m) s += BT4[a][m] * d36[m * 6 + b];
            t[a][b] = s;
        }
    for (int a = 0; a < 6; ++a)
        for (int b = 0; b < 6; ++b) {
            double s = 0.0;
            for (int m = 0; m < 6; ++m) s += t[a][m] * BT4[b][m];
            v36[a * 6 + b] = s;
        }
}
/* Y = AT4 M AT4^T (4x4) */
void oracle_otf4_tile(const double* m36, double* o16) {
    double t[4][6];
    for (int a = 0; a < 4; ++a)
        for (int b = 0; b < 6; ++b) {
            double s = 0.0;
            for (int q = 0; q < 6; ++q) s += AT4[a][q] * m36[q * 6 + b];
            t[a][b] = s;
        }
    for (int a = 0; a < 4; ++a)
        for (int b = 0; b < 4; ++b) {
            double s = 0.0;
            for (int q = 0; q < 6; ++q) s += t[a][q] * AT4[b][q];
            o16[a * 4 + b] = s;
        }
}

/* U4 (C,6,6,K) */
void oracle_filter_transform_f4(const double* w, double* u, int C, int K) {
#pragma omp parallel for schedule(static)
    for (long ck = 0; ck < (long)C * K; ++ck) {
        int c = (int)(ck / K), k = (int)(ck % K);
        double g[9], t[36];
        for (int e = 0; e < 9; ++e) g[e] = w[((size_t)c * 9 + e) * K + k];
        oracle_ftf4_tile(g, t);
        for (int e = 0; e < 36; ++e) u[((size_t)c * 36 + e) * K + k] = t[e];
    }
}

/* Naive F(4x4,3x3) Winograd conv, pad 1: windows start at (4th-1, 4tw-1). */
int oracle_winograd_f4_conv(const double* x, const double* w, double* y, int N, int C, int H, int W, int K) {
    double* U = (double*)malloc(sizeof(double) * 36 * (size_t)C * K);
    if (!U) return 1;
    oracle_filter_transform_f4(w, U, C, K);
    int TH = (H + 3) / 4, TW = (W + 3) / 4;
    int failed = 0;
#pragma omp parallel
    {
        double* V = (double*)malloc(sizeof(double) * 36 * (size_t)C * N);
        if (!V) {
#pragma omp atomic write
            failed = 1;
        }
#pragma omp for schedule(dynamic, 1)
        for (long t = 0; t < (long)TH * TW; ++t) {
            if (!V) continue;
            int th = (int)(t / TW), tw = (int)(t % TW);
            for (int c = 0; c < C; ++c)
                for (int n = 0; n < N; ++n) {
                    double d[36];
                    for (int a = 0; a < 6; ++a)
                        for (int b = 0; b < 6; ++b) d[a * 6 + b] = xhat(x, N, H, W, c, 4 * th - 1 + a, 4 * tw - 1 + b, n);
                    oracle_itf4_tile(d, V + ((size_t)c * N + n) * 36);
                }
            for (int k = 0; k < K; ++k)
                for (int n = 0; n < N; ++n) {
                    double m[36], o[16];
                    for (int e = 0; e < 36; ++e) m[e] = 0.0;
                    for (int c = 0; c < C; ++c)
                        for (int e = 0; e < 36; ++e) m[e] += U[((size_t)c * 36 + e) * K + k] * V[((size_t)c * N + n) * 36 + e];
                    oracle_otf4_tile(m, o);
                    for (int a = 0; a < 4; ++a)
                        for (int b = 0; b < 4; ++b) {
                            int i = 4 * th + a, j = 4 * tw + b;
                            if (i < H && j < W) y[(((size_t)k * H + i) * W + j) * N + n] = o[a * 4 + b];
                        }
                }
        }
        free(V);
    }
    free(U);
    return failed;
}
