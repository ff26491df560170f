/*
 * oracle.c -- TEST INFRASTRUCTURE ONLY.  Plain, slow, obviously-correct CPU
 * definitions of the unprotected kernels the paper evaluates (PAPER.md P:157,
 * Fig. 2 axis P:237-255) plus the BJ-added MatrixTranspose.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference leg may load this library.  It shares no code, header,
 * table or constant generator with the CUDA path (paper_conf_isca_waddenlgss14_b200/csrc).
 *
 * Citations: "P:NNN" = /root/reference/PAPER.md line NNN.  The paper names the
 * kernels only (they are AMD APP SDK samples, ref [5] P:931); each
 * definition below is the textbook one, with the readings recorded in
 * DESIGN.md section "Readings" (R-xx tags below).  RMT itself never changes a
 * result: "all redundant values that leave the SoR must be compared ... before
 * a single correct copy is allowed to leave", so the oracle of every
 * RMT variant's output is the unprotected definition.
 *
 * Precision: fp64 for floating point, exact integers otherwise.
 * The one exception is orc_fwt_f32dag, which evaluates the FWT's butterfly DAG
 * in fp32 in the normative stage order (reading R-FWT2) so that the GPU can be
 * checked bit-exactly.
 *
 * Parity pins live in tests/test_oracle_pins.py (closed forms, invariants,
 * brute force, an independent algorithm).
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#ifdef _OPENMP
#include <omp.h>
#endif

int orc_num_threads(void) {
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}

/* Thread count for the timing legs (bench.py's 1-thread cpu_baseline run). */
void orc_set_threads(int n) {
#ifdef _OPENMP
    omp_set_num_threads(n > 0 ? n : 1);
#else
    (void)n;
#endif
}

/* ------------------------------------------------------------------------ */
/* BlackScholes  (P:157 / Fig.2 "BlkSch"; R-BS1 input mapping, R-BS2 CND)    */
/* ------------------------------------------------------------------------ */

/* Cumulative normal distribution, Abramowitz & Stegun 26.2.17 polynomial
 * (reading R-BS2): k = 1/(1+0.2316419|x|),
 * N(x) = 1 - phi(x) * k*(a1 + k*(a2 + k*(a3 + k*(a4 + k*a5)))) for x >= 0,
 * N(x) = 1 - N(-x) for x < 0. */
double orc_cnd(double x) {
    const double a1 = 0.319381530, a2 = -0.356563782, a3 = 1.781477937;
    const double a4 = -1.821255978, a5 = 1.330274429;
    double ax = fabs(x);
    double k = 1.0 / (1.0 + 0.2316419 * ax);
    double phi = exp(-0.5 * ax * ax) / sqrt(2.0 * M_PI);
    double w = 1.0 - phi * k * (a1 + k * (a2 + k * (a3 + k * (a4 + k * a5))));
    return x < 0.0 ? 1.0 - w : w;
}

/* European call / put, textbook Black-Scholes:
 *   d1 = (ln(S/K) + (R + sigma^2/2) T) / (sigma sqrt T),  d2 = d1 - sigma sqrt T
 *   C = S N(d1) - K e^{-RT} N(d2),  P = K e^{-RT} N(-d2) - S N(-d1). */
void orc_bs_price(double S, double K, double T, double R, double V, double* call, double* put) {
    double sT = V * sqrt(T);
    double d1 = (log(S / K) + (R + 0.5 * V * V) * T) / sT;
    double d2 = d1 - sT;
    double disc = K * exp(-R * T);
    *call = S * orc_cnd(d1) - disc * orc_cnd(d2);
    *put = disc * orc_cnd(-d2) - S * orc_cnd(-d1);
}

/* R-BS1 (APP-SDK-style workload): one uniform r per option,
 *   S = 10r + 100(1-r), K = 10r + 100(1-r), T = 1r + 10(1-r),
 *   R = 0.01r + 0.05(1-r), sigma = 0.01r + 0.10(1-r). */
void orc_bs_params(double r, double* S, double* K, double* T, double* R, double* V) {
    *S = 10.0 * r + 100.0 * (1.0 - r);
    *K = 10.0 * r + 100.0 * (1.0 - r);
    *T = 1.0 * r + 10.0 * (1.0 - r);
    *R = 0.01 * r + 0.05 * (1.0 - r);
    *V = 0.01 * r + 0.10 * (1.0 - r);
}

void orc_blackscholes(const float* r, int64_t n, double* call, double* put) {
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n; ++i) {
        double S, K, T, R, V;
        orc_bs_params((double)r[i], &S, &K, &T, &R, &V);
        orc_bs_price(S, K, T, R, V, &call[i], &put[i]);
    }
}

/* Independent parameters (reading R-BS4, SURVEY 8(c) "bs_indep"): option i has
 * S = prm[i], K = prm[n+i], T = prm[2n+i], R = prm[3n+i], sigma = prm[4n+i].
 * Besides the prices, returns the conditioning scale of each price, the sum of
 * the magnitudes of its two terms: |S N(d1)| + |K e^{-RT} N(d2)| for the call,
 * |K e^{-RT} N(-d2)| + |S N(-d1)| for the put (the fp32 error of a difference
 * scales with the terms, not with the difference). */
void orc_blackscholes_indep(const float* prm, int64_t n, double* call, double* put, double* call_scale,
                            double* put_scale) {
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n; ++i) {
        double S = prm[i], K = prm[n + i], T = prm[2 * n + i], R = prm[3 * n + i], V = prm[4 * n + i];
        double sT = V * sqrt(T);
        double d1 = (log(S / K) + (R + 0.5 * V * V) * T) / sT;
        double d2 = d1 - sT;
        double disc = K * exp(-R * T);
        orc_bs_price(S, K, T, R, V, &call[i], &put[i]);
        call_scale[i] = fabs(S * orc_cnd(d1)) + fabs(disc * orc_cnd(d2));
        put_scale[i] = fabs(disc * orc_cnd(-d2)) + fabs(S * orc_cnd(-d1));
    }
}

/* ------------------------------------------------------------------------ */
/* BinarySearch (Fig.2 "BinS"; reading R-BIN1: batched lower_bound)   */
/* ------------------------------------------------------------------------ */
/* idx[j] = #{ i : A[i] < q[j] } for sorted A, found by plain bisection. */
void orc_binarysearch(const uint32_t* A, int64_t N, const uint32_t* q, int64_t Q, uint32_t* idx) {
#pragma omp parallel for schedule(static)
    for (int64_t j = 0; j < Q; ++j) {
        int64_t lo = 0, hi = N; /* invariant: A[<lo] < key <= A[>=hi] */
        uint32_t key = q[j];
        while (lo < hi) {
            int64_t mid = lo + (hi - lo) / 2;
            if (A[mid] < key) lo = mid + 1; else hi = mid;
        }
        idx[j] = (uint32_t)lo;
    }
}

/* ------------------------------------------------------------------------ */
/* FastWalshTransform (Fig.2 "FWT"; R-FWT1 natural order, unnormalised) */
/* ------------------------------------------------------------------------ */
/* y = H_N x: log2 N radix-2 stages, step h = 1, 2, 4, ..., N/2; for every
 * i with (i & h) == 0: (a, b) = (x[i], x[i+h]) -> (a + b, a - b). */
void orc_fwt_f64(const float* x, int64_t N, double* y) {
    for (int64_t i = 0; i < N; ++i) y[i] = (double)x[i];
    for (int64_t h = 1; h < N; h <<= 1) {
#pragma omp parallel for schedule(static)
        for (int64_t i = 0; i < N; ++i) {
            if (i & h) continue;
            double a = y[i], b = y[i + h];
            y[i] = a + b;
            y[i + h] = a - b;
        }
    }
}

/* Same DAG, evaluated in fp32 (R-FWT2: the stage order is normative, so the
 * fp32 result is unique and the GPU must match it bit for bit). */
void orc_fwt_f32dag(const float* x, int64_t N, float* y) {
    for (int64_t i = 0; i < N; ++i) y[i] = x[i];
    for (int64_t h = 1; h < N; h <<= 1) {
#pragma omp parallel for schedule(static)
        for (int64_t i = 0; i < N; ++i) {
            if (i & h) continue;
            volatile float a = y[i], b = y[i + h];
            y[i] = a + b;
            y[i + h] = a - b;
        }
    }
}

/* ------------------------------------------------------------------------ */
/* PrefixSum ("PS"; R-PS1 inclusive, R-PS2 u32 mod 2^32)              */
/* ------------------------------------------------------------------------ */
void orc_prefixsum_u32(const uint32_t* x, int64_t n, uint32_t* y) {
    uint32_t acc = 0;
    for (int64_t i = 0; i < n; ++i) { acc += x[i]; y[i] = acc; }
}

/* Exclusive form (SURVEY 8(c) PrefixSum reading (1): "inclusive, with an
 * exclusive flag"; exclusive = shift): y_i = sum_{j<i} x_j mod 2^32. */
void orc_prefixsum_u32_excl(const uint32_t* x, int64_t n, uint32_t* y) {
    uint32_t acc = 0;
    for (int64_t i = 0; i < n; ++i) { y[i] = acc; acc += x[i]; }
}

/* fp32 secondary (SURVEY 8(c) PrefixSum reading (2): the SDK scan is fp32): the
 * definition in fp64, y_i = sum_{j<=i} x_j (exclusive: j < i), plus the
 * conditioning bound b_i = sum |x_j| over the same range, against which the
 * kernel's fixed-association fp32 scan is checked (|dy_i| <= 1e-5 b_i). */
void orc_prefixsum_f64(const float* x, int64_t n, int exclusive, double* y, double* b) {
    double acc = 0.0, abs_acc = 0.0;
    for (int64_t i = 0; i < n; ++i) {
        if (exclusive) { y[i] = acc; b[i] = abs_acc; }
        acc += (double)x[i];
        abs_acc += fabs((double)x[i]);
        if (!exclusive) { y[i] = acc; b[i] = abs_acc; }
    }
}

/* ------------------------------------------------------------------------ */
/* Reduction ("R"; R-RED1 u32 inputs, exact u64 result)               */
/* ------------------------------------------------------------------------ */
uint64_t orc_reduction_u32(const uint32_t* x, int64_t n) {
    uint64_t s = 0;
#pragma omp parallel for reduction(+ : s) schedule(static)
    for (int64_t i = 0; i < n; ++i) s += x[i];
    return s;
}

/* ------------------------------------------------------------------------ */
/* MatrixTranspose (BJ configs[1]; not one of the paper's 16)    */
/* ------------------------------------------------------------------------ */
/* B[j][i] = A[i][j], A is H x W row-major; moves 32-bit words. */
void orc_transpose_u32(const uint32_t* A, int64_t H, int64_t W, uint32_t* B) {
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < H; ++i)
        for (int64_t j = 0; j < W; ++j) B[j * H + i] = A[i * W + j];
}

/* ------------------------------------------------------------------------ */
/* SobelFilter ("SF"; R-SOB1..5)                                      */
/* ------------------------------------------------------------------------ */
static uint32_t orc_isqrt(uint64_t s) { /* largest r with r*r <= s, by bisection */
    uint64_t lo = 0, hi = 1u << 16;
    while (lo < hi) {
        uint64_t mid = (lo + hi + 1) / 2;
        if (mid * mid <= s) lo = mid; else hi = mid - 1;
    }
    return (uint32_t)lo;
}

/* I, O: H x W pixels of 4 channels (uchar4).  For interior pixels, per channel
 *   Gx = i(-1,-1) + 2 i(0,-1) + i(1,-1) - i(-1,1) - 2 i(0,1) - i(1,1)
 *   Gy = i(-1,-1) - i(1,-1) + 2 i(-1,0) - 2 i(1,0) + i(-1,1) - i(1,1)
 * with i(dx,dy) = I[y+dy][x+dx], and O = min(255, floor(isqrt(Gx^2+Gy^2) / 2)).
 * Border pixels are 0 (R-SOB3). */
void orc_sobel(const uint8_t* I, int64_t H, int64_t W, uint8_t* O) {
#pragma omp parallel for schedule(static)
    for (int64_t y = 0; y < H; ++y) {
        for (int64_t x = 0; x < W; ++x) {
            for (int c = 0; c < 4; ++c) {
                uint8_t out = 0;
                if (x >= 1 && x < W - 1 && y >= 1 && y < H - 1) {
#define PIX(dx, dy) ((int64_t)I[((y + (dy)) * W + (x + (dx))) * 4 + c])
                    int64_t gx = PIX(-1, -1) + 2 * PIX(0, -1) + PIX(1, -1)
                               - PIX(-1, 1) - 2 * PIX(0, 1) - PIX(1, 1);
                    int64_t gy = PIX(-1, -1) - PIX(1, -1) + 2 * PIX(-1, 0)
                               - 2 * PIX(1, 0) + PIX(-1, 1) - PIX(1, 1);
#undef PIX
                    uint32_t m = orc_isqrt((uint64_t)(gx * gx + gy * gy)) / 2;
                    out = (uint8_t)(m > 255 ? 255 : m);
                }
                O[(y * W + x) * 4 + c] = out;
            }
        }
    }
}

/* ------------------------------------------------------------------------ */
/* FloydWarshall ("FW"; R-FW1..4)                                     */
/* ------------------------------------------------------------------------ */
/* In place, canonical k order: for k = 0..n-1, for all (i,j):
 *   if D[i][k] + D[k][j] < D[i][j] then D[i][j] = D[i][k] + D[k][j], P[i][j] = k.
 * P must be initialised by the caller (R-FW2: P[i][j] = i). */
void orc_floydwarshall(uint32_t* D, uint32_t* P, int64_t n) {
    for (int64_t k = 0; k < n; ++k) {
#pragma omp parallel for schedule(static)
        for (int64_t i = 0; i < n; ++i) {
            uint64_t dik = D[i * n + k];
            for (int64_t j = 0; j < n; ++j) {
                uint64_t cand = dik + D[k * n + j];
                if (cand < D[i * n + j]) { D[i * n + j] = (uint32_t)cand; P[i * n + j] = (uint32_t)k; }
            }
        }
    }
}

/* Independent check (not FW): O(n^2) Dijkstra from `src` on the dense weight matrix. */
void orc_dijkstra_row(const uint32_t* Wm, int64_t n, int64_t src, uint32_t* dist) {
    uint8_t* done = (uint8_t*)calloc((size_t)n, 1);
    uint64_t* d = (uint64_t*)malloc((size_t)n * sizeof(uint64_t));
    for (int64_t v = 0; v < n; ++v) d[v] = UINT64_MAX;
    d[src] = 0;
    for (int64_t it = 0; it < n; ++it) {
        int64_t u = -1;
        for (int64_t v = 0; v < n; ++v)
            if (!done[v] && (u < 0 || d[v] < d[u])) u = v;
        if (u < 0 || d[u] == UINT64_MAX) break;
        done[u] = 1;
        for (int64_t v = 0; v < n; ++v) {
            uint64_t c = d[u] + Wm[u * n + v];
            if (c < d[v]) d[v] = c;
        }
    }
    for (int64_t v = 0; v < n; ++v) dist[v] = (uint32_t)d[v];
    free(done);
    free(d);
}

/* ------------------------------------------------------------------------ */
/* DCT ("DCT"; R-DCT1..4: forward orthonormal 8x8 DCT-II)             */
/* ------------------------------------------------------------------------ */
/* Per 8x8 block X (rows x, cols y): Y[u][v] = sum_x sum_y C[u][x] X[x][y] C[v][y],
 * C[u][x] = alpha(u) cos((2x+1) u pi / 16), alpha(0) = sqrt(1/8), alpha(u>0) = 1/2. */
static double orc_dct_c(int u, int x) {
    double a = (u == 0) ? sqrt(1.0 / 8.0) : 0.5;
    return a * cos((2.0 * x + 1.0) * u * M_PI / 16.0);
}

void orc_dct8x8(const float* X, int64_t H, int64_t W, double* Y) {
    double C[8][8];
    for (int u = 0; u < 8; ++u)
        for (int x = 0; x < 8; ++x) C[u][x] = orc_dct_c(u, x);
#pragma omp parallel for schedule(static)
    for (int64_t by = 0; by < H / 8; ++by) {
        for (int64_t bx = 0; bx < W / 8; ++bx) {
            for (int u = 0; u < 8; ++u) {
                for (int v = 0; v < 8; ++v) {
                    double s = 0.0;
                    for (int x = 0; x < 8; ++x)
                        for (int y = 0; y < 8; ++y)
                            s += C[u][x] * (double)X[(by * 8 + x) * W + bx * 8 + y] * C[v][y];
                    Y[(by * 8 + u) * W + bx * 8 + v] = s;
                }
            }
        }
    }
}

/* Componentwise condition bound (|C| |X| |C|^T)_uv used by the DCT tolerance (R-DCT3). */
void orc_dct8x8_absbound(const float* X, int64_t H, int64_t W, double* Yabs) {
    double C[8][8];
    for (int u = 0; u < 8; ++u)
        for (int x = 0; x < 8; ++x) C[u][x] = fabs(orc_dct_c(u, x));
#pragma omp parallel for schedule(static)
    for (int64_t by = 0; by < H / 8; ++by)
        for (int64_t bx = 0; bx < W / 8; ++bx)
            for (int u = 0; u < 8; ++u)
                for (int v = 0; v < 8; ++v) {
                    double s = 0.0;
                    for (int x = 0; x < 8; ++x)
                        for (int y = 0; y < 8; ++y)
                            s += C[u][x] * fabs((double)X[(by * 8 + x) * W + bx * 8 + y]) * C[v][y];
                    Yabs[(by * 8 + u) * W + bx * 8 + v] = s;
                }
}

/* ------------------------------------------------------------------------ */
/* MatrixMultiplication ("MM"; R-MM1 bf16 operands, fp32 result)      */
/* ------------------------------------------------------------------------ */
static double orc_bf16(uint16_t b) {
    uint32_t u = (uint32_t)b << 16;
    float f;
    memcpy(&f, &u, 4);
    return (double)f;
}

/* C[i][j] = sum_k A[i][k] * Bt[j][k]  (A: M x K row-major, Bt: N x K row-major,
 * i.e. B = Bt^T), exact fp64 dot products of the bf16 values. */
void orc_matmul_bf16(const uint16_t* A, const uint16_t* Bt, int64_t M, int64_t N, int64_t K, double* C) {
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < M; ++i)
        for (int64_t j = 0; j < N; ++j) {
            double s = 0.0;
            for (int64_t k = 0; k < K; ++k) s += orc_bf16(A[i * K + k]) * orc_bf16(Bt[j * K + k]);
            C[i * N + j] = s;
        }
}

/* Sampled elements: out[s] = C[rows[s]][cols[s]] (same definition, one dot each). */
void orc_matmul_bf16_sampled(const uint16_t* A, const uint16_t* Bt, int64_t K, int64_t nsamp,
                             const int64_t* rows, const int64_t* cols, double* out, double* absout) {
#pragma omp parallel for schedule(static)
    for (int64_t s = 0; s < nsamp; ++s) {
        double acc = 0.0, aacc = 0.0;
        for (int64_t k = 0; k < K; ++k) {
            double p = orc_bf16(A[rows[s] * K + k]) * orc_bf16(Bt[cols[s] * K + k]);
            acc += p;
            aacc += fabs(p);
        }
        out[s] = acc;
        absout[s] = aacc;
    }
}

/* ======================================================================== */
/* the paper's communication-stress kernels              */
/* ======================================================================== */

/* ------------------------------------------------------------------------ */
/* BitonicSort (P:157 / Fig.2 "BitS"; memory-bound P:567, Inter 9.48x P:695, */
/* P:807; reading R-BIT1: ascending u32 keys, N a power of two).  A sorting  */
/* network's result is the sorted sequence, which is unique for keys, so the */
/* oracle is that definition: a library sort of a copy.                      */
/* ------------------------------------------------------------------------ */
static int orc_cmp_u32(const void* a, const void* b) {
    uint32_t x = *(const uint32_t*)a, y = *(const uint32_t*)b;
    return (x > y) - (x < y);
}
void orc_sort_u32(const uint32_t* keys, int64_t n, uint32_t* out) {
    memcpy(out, keys, (size_t)n * sizeof(uint32_t));
    qsort(out, (size_t)n, sizeof(uint32_t), orc_cmp_u32);
}

/* ------------------------------------------------------------------------ */
/* DwtHaar1D (P:157 / Fig.2 "DWT"; memory-bound yet communication-heavy,     */
/* P:571-575).  Readings R-DWT1/2: full orthonormal Haar decomposition of N = */
/* 2^L samples, level by level: a_i = (c_{2i} + c_{2i+1}) / sqrt2,            */
/* d_i = (c_{2i} - c_{2i+1}) / sqrt2 of the previous level's approximation c. */
/* Layout: y[0] = final approximation a_L, y[2^(L-k) .. 2^(L-k+1)) = level-k */
/* details (k = 1 finest: y[N/2 .. N)).                                      */
/* ------------------------------------------------------------------------ */
void orc_dwthaar1d_f64(const float* x, int64_t N, double* y) {
    double* c = (double*)malloc((size_t)N * sizeof(double));
    for (int64_t i = 0; i < N; ++i) c[i] = (double)x[i];
    for (int64_t len = N; len > 1; len >>= 1) {
        int64_t half = len >> 1;
        for (int64_t i = 0; i < half; ++i) {
            double a = (c[2 * i] + c[2 * i + 1]) * M_SQRT1_2;
            double d = (c[2 * i] - c[2 * i + 1]) * M_SQRT1_2;
            y[half + i] = d;
            c[i] = a; /* i < 2i: the in-place overwrite reads nothing later needed */
        }
    }
    if (N >= 1) y[0] = c[0];
    free(c);
}

/* Same DAG in fp32 (R-DWT2: per level a = RN(RN(c0 + c1) * s), d = RN(RN(c0 -
 * c1) * s), s = RN32(1/sqrt2); the level order fixes every rounding, so the GPU
 * is checked bit for bit against this). */
void orc_dwthaar1d_f32dag(const float* x, int64_t N, float* y) {
    float* c = (float*)malloc((size_t)N * sizeof(float));
    const float s = (float)M_SQRT1_2;
    memcpy(c, x, (size_t)N * sizeof(float));
    for (int64_t len = N; len > 1; len >>= 1) {
        int64_t half = len >> 1;
        for (int64_t i = 0; i < half; ++i) {
            volatile float sum = c[2 * i] + c[2 * i + 1];
            volatile float dif = c[2 * i] - c[2 * i + 1];
            volatile float a = sum * s;
            volatile float d = dif * s;
            y[half + i] = d;
            c[i] = a;
        }
    }
    if (N >= 1) y[0] = c[0];
    free(c);
}

/* ------------------------------------------------------------------------ */
/* BinomialOption (P:157 / Fig.2 "BO"; LDS-bound, -LDS trades compute for    */
/* communication P:575; FAST swizzle beneficiary P:853).  Readings R-BO1/2:   */
/* European call on a Cox-Ross-Rubinstein lattice of NSTEPS = 254 steps,     */
/* R = 0.02, sigma = 0.30; one U[0,1) draw r per option mapped to            */
/* S = 5(1-r) + 30r, K = (1-r) + 100r, T = 0.25(1-r) + 10r [APP-SDK?].        */
/* dt = T/N, u = e^{sigma sqrt dt}, d = 1/u, p = (e^{R dt} - d)/(u - d);      */
/* leaves V_i = max(S u^{2i-N} - K, 0), i = 0..N; N backward steps           */
/* V_i <- e^{-R dt} (p V_{i+1} + (1-p) V_i); the price is V_0.               */
/* ------------------------------------------------------------------------ */
#define ORC_BO_STEPS 254
#define ORC_BO_R 0.02
#define ORC_BO_V 0.30

double orc_crr_price(double S, double K, double T, double R, double V, int64_t N, int call) {
    double dt = T / (double)N;
    double u = exp(V * sqrt(dt)), d = 1.0 / u;
    double p = (exp(R * dt) - d) / (u - d);
    double disc = exp(-R * dt);
    double* v = (double*)malloc((size_t)(N + 1) * sizeof(double));
    for (int64_t i = 0; i <= N; ++i) {
        double price = S * pow(u, (double)(2 * i - N));
        double pay = call ? price - K : K - price;
        v[i] = pay > 0.0 ? pay : 0.0;
    }
    for (int64_t j = N; j > 0; --j)
        for (int64_t i = 0; i < j; ++i) v[i] = disc * (p * v[i + 1] + (1.0 - p) * v[i]);
    double out = v[0];
    free(v);
    return out;
}

void orc_bo_params(double r, double* S, double* K, double* T) {
    *S = 5.0 * (1.0 - r) + 30.0 * r;
    *K = 1.0 * (1.0 - r) + 100.0 * r;
    *T = 0.25 * (1.0 - r) + 10.0 * r;
}

void orc_binomialoption(const float* r, int64_t n, double* call) {
#pragma omp parallel for schedule(dynamic, 64)
    for (int64_t i = 0; i < n; ++i) {
        double S, K, T;
        orc_bo_params((double)r[i], &S, &K, &T);
        call[i] = orc_crr_price(S, K, T, ORC_BO_R, ORC_BO_V, ORC_BO_STEPS, 1);
    }
}
