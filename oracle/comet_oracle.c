/*
 * comet_oracle.c -- CPU oracle for the COMET W4Ax hot path.  TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference
 * leg may load this library.  It shares no code, header, table or constant generator
 * with the CUDA path (paper_conf_asplos_liu0rxpwl0w25_b200/csrc); neither side includes
 * or links the other.
 *
 * What it computes is written out from the paper (COMET, ASPLOS'25, /root/reference/PAPER.md,
 * cited as P:Lnnn) in the paper's order, with the readings of DESIGN.md §3 where the
 * paper is silent:
 *
 *   1. FMPQ block quantisation of activations ("divide the activation tensor into
 *      multiple sub-tensors with a channel size of k ... setting k to 128"; "any block
 *      that contains outliers will require 8-bit quantization"; P:L126 min-max quantisation;
 *      P:L242 "block-wise mixed-precision (INT4 and INT8) quantization for activations").
 *      Readings R1-R5: one scale per (token, block), symmetric, qmax = 7 / 127,
 *      s = amax/qmax and r = qmax/amax in IEEE binary32, q = clamp(rint_half_even(x*r)).
 *   2. The integer GEMM per 128-channel block, accumulated exactly (int64, checked to fit
 *      int32) (P:L164 tile accumulation; P:L166 W4A4 / W4A8 mma with INT32 accumulators).
 *   3. Dequantisation: y[m,n] = s_w[n] * sum_b s_a[m,b] * acc_b[m,n] in binary64, b ascending
 *      ("reduction operator to accumulate the compute results of different tiles";
 *      P:L206 the scale absorbs the conversion factor).  Reading R7: per-output-channel s_w.
 *
 * Build: gcc -O2 -fno-fast-math -ffp-contract=off -fopenmp -shared -fPIC
 * (-ffp-contract=off: x*r must be one correctly-rounded binary32 product, never an FMA).
 * Every loop below is the plain definition; the only parallelism is OpenMP over rows,
 * which does not change any result (each row is independent).
 */
#include <stdint.h>
#include <string.h>
#include <math.h>

#define COMET_ORACLE_BLOCK 128   /* k = 128 channels per block */

/* ---- exact conversions of the 16-bit inputs to binary32 -------------------------------- */

/* IEEE binary16 -> binary32 (exact; every binary16 value is a binary32 value). */
static float oracle_f16_to_f32(uint16_t h) {
    uint32_t sign = (uint32_t)(h >> 15) << 31;
    uint32_t exp = (h >> 10) & 0x1F;
    uint32_t man = h & 0x3FF;
    uint32_t bits;
    if (exp == 0) {
        if (man == 0) {
            bits = sign;
        } else {                         /* subnormal binary16: man * 2^-24, normal in binary32 */
            int e = -1;
            do { man <<= 1; e++; } while ((man & 0x400) == 0);
            man &= 0x3FF;
            bits = sign | ((uint32_t)(127 - 15 - e) << 23) | (man << 13);
        }
    } else if (exp == 31) {
        bits = sign | 0x7F800000u | (man << 13);
    } else {
        bits = sign | ((exp - 15 + 127) << 23) | (man << 13);
    }
    float f;
    memcpy(&f, &bits, 4);
    return f;
}

/* bfloat16 -> binary32 (exact: bf16 is the top half of a binary32). */
static float oracle_bf16_to_f32(uint16_t h) {
    uint32_t bits = (uint32_t)h << 16;
    float f;
    memcpy(&f, &bits, 4);
    return f;
}

static float oracle_load_x(const uint16_t* x, int64_t idx, int x_is_bf16) {
    return x_is_bf16 ? oracle_bf16_to_f32(x[idx]) : oracle_f16_to_f32(x[idx]);
}

/* ---- 1. FMPQ quantisation of one (token m, block b) ----------------------------------- */
/*
 * For block b of row m (channels 128b .. 128b+127):
 *   amax = max_k |x_k|                              (min-max quantisation)
 *   qmax = 127 if tags[b] (outlier block -> INT8) else 7 (INT4)
 *   amax == 0        -> s = 0, every code 0         (reading R5)
 *   otherwise        -> s = amax / qmax, r = qmax / amax (binary32, correctly rounded)
 *                       t_k = x_k * r (binary32);  q_k = clamp(rint(t_k), -qmax, qmax)
 *                       (rint = round half to even, reading R3; t_k NaN (0*inf when r
 *                        overflows for a binary32-subnormal amax) gives code 0, reading R5)
 */
static void oracle_quantize_block(const uint16_t* x, int x_is_bf16, int64_t row_off, int64_t b,
                                  int is_int8, int8_t* codes_row, float* scale_out) {
    const int64_t k0 = b * COMET_ORACLE_BLOCK;
    float amax = 0.0f;
    for (int64_t k = 0; k < COMET_ORACLE_BLOCK; ++k) {
        float v = fabsf(oracle_load_x(x, row_off + k0 + k, x_is_bf16));
        if (v > amax) amax = v;
    }
    const float qmax = is_int8 ? 127.0f : 7.0f;
    if (amax == 0.0f) {
        *scale_out = 0.0f;
        for (int64_t k = 0; k < COMET_ORACLE_BLOCK; ++k) codes_row[k0 + k] = 0;
        return;
    }
    volatile float s = amax / qmax;   /* volatile: force a binary32 rounding step */
    volatile float r = qmax / amax;
    *scale_out = s;
    for (int64_t k = 0; k < COMET_ORACLE_BLOCK; ++k) {
        float xv = oracle_load_x(x, row_off + k0 + k, x_is_bf16);
        volatile float t = xv * r;
        float q;
        if (t != t) {
            q = 0.0f;
        } else {
            q = rintf(t);
            if (q > qmax) q = qmax;
            if (q < -qmax) q = -qmax;
        }
        codes_row[k0 + k] = (int8_t)q;
    }
}

/* Quantise X[M][K] (row-major, leading dimension K) -> codes[M][K] (int8) and
 * scales[M][K/128] (binary32, row-major: scales[m*nb + b]). Returns 0, or -1 on bad args. */
int oracle_quantize(const uint16_t* x, int x_is_bf16, int64_t M, int64_t K, const uint8_t* tags,
                    int8_t* codes, float* scales) {
    if (M < 0 || K <= 0 || (K % COMET_ORACLE_BLOCK) != 0) return -1;
    const int64_t nb = K / COMET_ORACLE_BLOCK;
#pragma omp parallel for schedule(static)
    for (int64_t m = 0; m < M; ++m) {
        for (int64_t b = 0; b < nb; ++b) {
            oracle_quantize_block(x, x_is_bf16, m * K, b, tags[b] != 0, codes + m * K,
                                  scales + m * nb + b);
        }
    }
    return 0;
}

/* ---- 2. integer GEMM per block ----------------------------------------------------------- */
/*
 * acc[b][m][n] = sum_{k in block b} q[m][k] * w[n][k]   (exact, int64)
 * rows[] selects which token rows to compute (out is [nb][nrows][N]).
 * Returns 0, -1 on bad args, -2 if some accumulator does not fit int32.
 */
int oracle_gemm_blocks(const int8_t* q, const int8_t* w, int64_t M, int64_t N, int64_t K,
                       const int64_t* rows, int64_t nrows, int64_t* acc) {
    if (K <= 0 || (K % COMET_ORACLE_BLOCK) != 0 || N <= 0) return -1;
    const int64_t nb = K / COMET_ORACLE_BLOCK;
    int overflow = 0;
#pragma omp parallel for schedule(static) reduction(| : overflow)
    for (int64_t i = 0; i < nrows; ++i) {
        const int64_t m = rows[i];
        if (m < 0 || m >= M) { overflow |= 4; continue; }
        for (int64_t b = 0; b < nb; ++b) {
            for (int64_t n = 0; n < N; ++n) {
                int64_t s = 0;
                for (int64_t k = b * COMET_ORACLE_BLOCK; k < (b + 1) * COMET_ORACLE_BLOCK; ++k)
                    s += (int64_t)q[m * K + k] * (int64_t)w[n * K + k];
                if (s > INT32_MAX || s < INT32_MIN) overflow |= 1;
                acc[(b * nrows + i) * N + n] = s;
            }
        }
    }
    if (overflow & 4) return -1;
    return overflow ? -2 : 0;
}

/* ---- 3. dequantisation ------------------------------------------------------------------- */
/*
 * y[i][n] = s_w[n] * sum_{b ascending} s_a[rows[i]][b] * acc[b][i][n]     (binary64)
 */
int oracle_dequant(const int64_t* acc, const float* s_a, const float* s_w, int64_t N, int64_t nb,
                   const int64_t* rows, int64_t nrows, double* y) {
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < nrows; ++i) {
        const int64_t m = rows[i];
        for (int64_t n = 0; n < N; ++n) {
            double t = 0.0;
            for (int64_t b = 0; b < nb; ++b)
                t += (double)s_a[m * nb + b] * (double)acc[(b * nrows + i) * N + n];
            y[i * N + n] = (double)s_w[n] * t;
        }
    }
    return 0;
}

/* ---- whole path for a sample of rows (bounded memory at full sizes) ---------------------- */
/*
 * For each selected row m: quantise the row (step 1), then for every output channel n the
 * per-block integer dot products (step 2) and the binary64 dequantised sum (step 3).
 * Outputs: y[i][n] (binary64), acc_sum[i][n] = sum_b acc_b (int64), codes_out[i][K] and
 * scales_out[i][nb] of the quantised rows.  Same arithmetic as the three functions above,
 * row by row; used for BASELINE-sized configurations where [nb][M][N] does not fit.
 */
int oracle_w4ax_rows(const uint16_t* x, int x_is_bf16, int64_t M, int64_t K, const uint8_t* tags,
                     const int8_t* w, const float* s_w, int64_t N, const int64_t* rows,
                     int64_t nrows, double* y, int64_t* acc_sum, int8_t* codes_out,
                     float* scales_out) {
    if (K <= 0 || (K % COMET_ORACLE_BLOCK) != 0 || N <= 0) return -1;
    const int64_t nb = K / COMET_ORACLE_BLOCK;
    int bad = 0;
    for (int64_t i = 0; i < nrows; ++i) {
        const int64_t m = rows[i];
        if (m < 0 || m >= M) return -1;
        int8_t* qrow = codes_out + i * K;
        float* srow = scales_out + i * nb;
        for (int64_t b = 0; b < nb; ++b)
            oracle_quantize_block(x, x_is_bf16, m * K, b, tags[b] != 0, qrow, srow + b);
#pragma omp parallel for schedule(static) reduction(| : bad)
        for (int64_t n = 0; n < N; ++n) {
            double t = 0.0;
            int64_t total = 0;
            for (int64_t b = 0; b < nb; ++b) {
                int64_t s = 0;
                for (int64_t k = b * COMET_ORACLE_BLOCK; k < (b + 1) * COMET_ORACLE_BLOCK; ++k)
                    s += (int64_t)qrow[k] * (int64_t)w[n * K + k];
                if (s > INT32_MAX || s < INT32_MIN) bad = 1;
                t += (double)srow[b] * (double)s;
                total += s;
            }
            y[i * N + n] = (double)s_w[n] * t;
            acc_sum[i * N + n] = total;
        }
    }
    return bad ? -2 : 0;
}

/* Threads OpenMP will use (reported as cpu_baseline.cores). */
#ifdef _OPENMP
#include <omp.h>
int oracle_num_threads(void) { return omp_get_max_threads(); }
#else
int oracle_num_threads(void) { return 1; }
#endif
