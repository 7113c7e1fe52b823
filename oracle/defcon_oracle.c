/*
 * defcon_oracle.c -- fp64 CPU oracle for the DEFCON inference hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load this library.
 * It shares no code, header, table or helper with the CUDA product path
 * (paper_conf_ipps_jayaweeralwrk24_b200/csrc) and never calls it.
 *
 * Citations are to /root/reference/PAPER.md as "P:<line>" (section / equation).
 * Where the paper is silent we follow DESIGN.md "Readings" R1..R19 (same
 * numbering as SURVEY.md section 8(c)).
 *
 * Plain C99, fp64 throughout, no intrinsics.  OpenMP parallelises over the
 * (n, ho) output rows only; every output value is computed by one thread in
 * a fixed order, so results are deterministic.
 *
 * Layouts (all row-major, channel-last):
 *   x       [N][H][W][Cin]
 *   offset  [N][Ho][Wo][G][Kh*Kw][2]      (dy, dx) per tap, R4
 *   mask    [N][Ho][Wo][G][Kh*Kw]         already through the sigmoid, R6
 *   weight  [Cout][Kh][Kw][Cin]
 *   bias    [Cout]
 *   y       [N][Ho][Wo][Cout]
 *
 * Functions
 *   oracle_bilinear_f64         Eq.3 for one plane location
 *   oracle_dcn_forward_f64      Eq.2 (+DCNv2 mask) over the whole grid  P:56-59, R1-R9
 *   oracle_dcn_pixels_f64       same, for a list of output pixels
 *   oracle_offset_branch_f64    lightweight offset branch (dw3x3, BN, ReLU, 1x1) P:170
 *   oracle_dcn_forward_texq_f64 Eq.2 with the texture unit's fixed-point filter
 *                               weights (texture model; NOT from the paper, R14)
 *   oracle_bound_offsets_f64    bounded deformation, P x P window (R12)
 *   oracle_round_f16_array      16-bit offsets / mask of tex2D++ (R13)
 */
#include <math.h>
#include <stddef.h>
#include <stdint.h>
#include <stdlib.h>

#ifdef _OPENMP
#include <omp.h>
#endif

#define ORACLE_ABI_VERSION 1

int oracle_abi_version(void) { return ORACLE_ABI_VERSION; }

/* Number of OpenMP threads a parallel region will use (1 without OpenMP). */
int oracle_num_threads(void) {
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}

/* Set the thread count for subsequent calls (no-op without OpenMP). */
void oracle_set_num_threads(int n) {
#ifdef _OPENMP
    if (n > 0) omp_set_num_threads(n);
#else
    (void)n;
#endif
}

/* g(a, b) = max(0, 1 - |a - b|)  -- the 1-D bilinear kernel */
static double g_kernel(double a, double b) {
    double v = 1.0 - fabs(a - b);
    return v > 0.0 ? v : 0.0;
}

/*
 * Eq.3: x(p) = sum_q G(p, q) x(q), G(p,q) = g(p_x,q_x) g(p_y,q_y),
 * q over all integral locations of the plane.  Only the four neighbours
 * q in {floor(p), floor(p)+1}^2 can have G != 0, so the sum is taken
 * over exactly those; a neighbour outside [0,H)x[0,W) contributes zero
 * (R8).  floor() (not truncation) is used for negative p (R9).
 *
 * plane points at x[n][0][0][c]; pixel stride is `pix_stride` doubles.
 */
double oracle_bilinear_f64(const double *plane, int H, int W, long pix_stride,
                           double py, double px) {
    double y0 = floor(py), x0 = floor(px);
    double acc = 0.0;
    for (int a = 0; a < 2; ++a) {
        double qy = y0 + a;
        if (qy < 0.0 || qy > (double)(H - 1)) continue;
        for (int b = 0; b < 2; ++b) {
            double qx = x0 + b;
            if (qx < 0.0 || qx > (double)(W - 1)) continue;
            double G = g_kernel(px, qx) * g_kernel(py, qy);
            long idx = ((long)qy * W + (long)qx) * pix_stride;
            acc += G * plane[idx];
        }
    }
    return acc;
}

/* Texture-unit model (R14, CUDA programming guide "linear filtering"):
 * the fractional part is held in 9-bit fixed point with 8 fractional bits.
 * quant_mode: 1 = round to nearest 1/256, 2 = truncate to 1/256, 3 = the measured half4 filter
 * (bilinear_texq below). */
static double quant_frac(double f, int quant_mode) {
    if (quant_mode == 1) return floor(f * 256.0 + 0.5) / 256.0;
    if (quant_mode == 2) return floor(f * 256.0) / 256.0;
    return f;
}

/* Round to the nearest binary16 value, ties to even (normal and subnormal range; beyond the
 * largest finite value 65504 -- after rounding -- +-infinity, as IEEE binary16 does).  The
 * texels of the half4 texture are binary16, and so is the filter's result (R14); so are the
 * 16-bit offsets / mask of tex2D++ (R13). */
static double round_to_f16(double v) {
    if (v == 0.0 || v != v) return v;
    int e;
    frexp(v, &e);                          /* |v| = m * 2^e, 0.5 <= m < 1 */
    double q = ldexp(1.0, (e - 1 >= -14 ? e - 1 : -14) - 10);   /* 11 significant bits */
    double r = rint(v / q) * q;            /* default rounding mode: to nearest, ties to even */
    if (fabs(r) > 65504.0) r = copysign(INFINITY, v);
    return r;
}

/* quant_mode 3 ("hw", the half4-texel filter as measured on B200, R14): both fractions and
 * each of the four products (1-a)(1-b), a(1-b), (1-a)b, ab rounded to the nearest 1/256
 * (ties to even), the weighted sum of the four binary16 texels rounded to binary16. */
static double bilinear_texq(const double *plane, int H, int W, long pix_stride,
                            double py, double px, int quant_mode) {
    double y0 = floor(py), x0 = floor(px);
    double ay = quant_mode == 3 ? rint((py - y0) * 256.0) / 256.0 : quant_frac(py - y0, quant_mode);
    double ax = quant_mode == 3 ? rint((px - x0) * 256.0) / 256.0 : quant_frac(px - x0, quant_mode);
    double wy[2] = {1.0 - ay, ay}, wx[2] = {1.0 - ax, ax};
    double acc = 0.0;
    for (int a = 0; a < 2; ++a) {
        double qy = y0 + a;
        if (qy < 0.0 || qy > (double)(H - 1)) continue;
        for (int b = 0; b < 2; ++b) {
            double qx = x0 + b;
            if (qx < 0.0 || qx > (double)(W - 1)) continue;
            long idx = ((long)qy * W + (long)qx) * pix_stride;
            double w = wy[a] * wx[b];
            if (quant_mode == 3) w = rint(w * 256.0) / 256.0;
            acc += w * plane[idx];
        }
    }
    return quant_mode == 3 ? round_to_f16(acc) : acc;
}

/* Output size "computed similarly to a regular convolution" (R3). */
int oracle_out_size(int in, int k, int stride, int pad, int dil) {
    int span = in + 2 * pad - dil * (k - 1) - 1;
    if (span < 0 || stride <= 0) return 0; /* floor of a negative quotient: no output */
    return span / stride + 1;
}

/*
 * One output pixel (n, ho, wo) of Eq.2 with the DCNv2 modulation (R6):
 *   y[co] = b[co] + sum_{i,j} sum_ci W[co][i][j][ci] * m[g][k] * x(p_o + p_k + dp_k)
 * with k = i*Kw + j (all Kh*Kw taps, R1/R2), g = ci / (Cin/G) (R5),
 * p_o + p_k = (ho*s_h - pad_h + i*d_h, wo*s_w - pad_w + j*d_w) (R3),
 * dp_k = (offset[..][g][k][0], offset[..][g][k][1]) = (dy, dx) (R4).
 * Built as col[k][ci] first, then one dot product per co.
 */
/* The sampled column of one output pixel: col[k*Cin + ci] = m[g][k] * X(p_o + p_k + dp_k)
 * (Eq.3 with the mask, R6); the deformable analogue of an im2col row ("two-step"). */
static void dcn_pixel_col(const double *x, int H, int W, int Cin,
                          const double *off_px, const double *mask_px,
                          int Kh, int Kw, int sh, int sw, int ph, int pw, int dh, int dw,
                          int G, int n, int ho, int wo, int quant_mode, double *col) {
    const int KK = Kh * Kw;
    const int Cg = Cin / G;
    const double *img = x + (long)n * H * W * Cin;
    for (int i = 0; i < Kh; ++i) {
        for (int j = 0; j < Kw; ++j) {
            int k = i * Kw + j;
            for (int ci = 0; ci < Cin; ++ci) {
                int g = ci / Cg;
                double dy = off_px[((long)g * KK + k) * 2 + 0];
                double dx = off_px[((long)g * KK + k) * 2 + 1];
                double py = (double)(ho * sh - ph + i * dh) + dy;
                double px = (double)(wo * sw - pw + j * dw) + dx;
                double m = mask_px ? mask_px[(long)g * KK + k] : 1.0;
                double v = quant_mode
                               ? bilinear_texq(img + ci, H, W, Cin, py, px, quant_mode)
                               : oracle_bilinear_f64(img + ci, H, W, Cin, py, px);
                col[(long)k * Cin + ci] = m * v;
            }
        }
    }
}

static void dcn_one_pixel(const double *x, int H, int W, int Cin,
                          const double *off_px, const double *mask_px,
                          const double *weight, const double *bias, int Cout,
                          int Kh, int Kw, int sh, int sw, int ph, int pw, int dh, int dw,
                          int G, int n, int ho, int wo, int quant_mode,
                          double *col, double *y_px) {
    const int KK = Kh * Kw;
    dcn_pixel_col(x, H, W, Cin, off_px, mask_px, Kh, Kw, sh, sw, ph, pw, dh, dw, G, n, ho, wo,
                  quant_mode, col);
    for (int co = 0; co < Cout; ++co) {
        const double *wr = weight + (long)co * KK * Cin; /* [Kh][Kw][Cin] == [k][ci] */
        double acc = 0.0;
        for (long t = 0; t < (long)KK * Cin; ++t) acc += wr[t] * col[t];
        y_px[co] = (bias ? bias[co] : 0.0) + acc;
    }
}

static int dcn_check(int N, int H, int W, int Cin, int Cout, int Kh, int Kw,
                     int sh, int sw, int dh, int dw, int G, int Ho, int Wo) {
    if (N <= 0 || H <= 0 || W <= 0 || Cin <= 0 || Cout <= 0 || Kh <= 0 || Kw <= 0) return 1;
    if (sh <= 0 || sw <= 0 || dh <= 0 || dw <= 0 || G <= 0 || Cin % G != 0) return 1;
    if (Ho <= 0 || Wo <= 0) return 1;
    return 0;
}

static int dcn_grid(const double *x, int N, int H, int W, int Cin,
                    const double *offset, const double *mask,
                    const double *weight, const double *bias, int Cout,
                    int Kh, int Kw, int sh, int sw, int ph, int pw, int dh, int dw,
                    int G, int quant_mode, double *y) {
    int Ho = oracle_out_size(H, Kh, sh, ph, dh);
    int Wo = oracle_out_size(W, Kw, sw, pw, dw);
    if (dcn_check(N, H, W, Cin, Cout, Kh, Kw, sh, sw, dh, dw, G, Ho, Wo)) return 1;
    const int KK = Kh * Kw;
    int fail = 0;
#pragma omp parallel
    {
        double *col = (double *)malloc(sizeof(double) * (size_t)KK * Cin);
        if (!col) {
#pragma omp atomic write
            fail = 1;
        }
#pragma omp for schedule(dynamic, 1)
        for (long row = 0; row < (long)N * Ho; ++row) {
            if (!col) continue;
            int n = (int)(row / Ho), ho = (int)(row % Ho);
            for (int wo = 0; wo < Wo; ++wo) {
                long pix = ((long)n * Ho + ho) * Wo + wo;
                dcn_one_pixel(x, H, W, Cin, offset + pix * G * KK * 2,
                              mask ? mask + pix * G * KK : NULL, weight, bias, Cout,
                              Kh, Kw, sh, sw, ph, pw, dh, dw, G, n, ho, wo, quant_mode,
                              col, y + pix * Cout);
            }
        }
        free(col);
    }
    return fail ? 2 : 0;
}

/* Whole-grid DCN forward, Eq.2 + Eq.3 (+ DCNv2 mask when mask != NULL).
 * Returns 0 on success, 1 on invalid arguments, 2 on allocation failure. */
int oracle_dcn_forward_f64(const double *x, int N, int H, int W, int Cin,
                           const double *offset, const double *mask,
                           const double *weight, const double *bias, int Cout,
                           int Kh, int Kw, int sh, int sw, int ph, int pw, int dh, int dw,
                           int G, double *y) {
    return dcn_grid(x, N, H, W, Cin, offset, mask, weight, bias, Cout, Kh, Kw,
                    sh, sw, ph, pw, dh, dw, G, 0, y);
}

/* Texture-filter model of the same layer (R14): identical to
 * oracle_dcn_forward_f64 except that the two fractional parts of each
 * sampling position are quantised to 1/256 (quant_mode 1 = round,
 * 2 = truncate) before forming the bilinear weights. */
int oracle_dcn_forward_texq_f64(const double *x, int N, int H, int W, int Cin,
                                const double *offset, const double *mask,
                                const double *weight, const double *bias, int Cout,
                                int Kh, int Kw, int sh, int sw, int ph, int pw, int dh, int dw,
                                int G, int quant_mode, double *y) {
    if (quant_mode < 1 || quant_mode > 3) return 1;
    return dcn_grid(x, N, H, W, Cin, offset, mask, weight, bias, Cout, Kh, Kw,
                    sh, sw, ph, pw, dh, dw, G, quant_mode, y);
}

/* The same definition evaluated only at `n_pix` flattened output pixels
 * pix_idx[t] = (n*Ho + ho)*Wo + wo; y_out is [n_pix][Cout].  Lets the tests
 * check full-size GPU launches on sampled outputs. */
static int dcn_pixels(const double *x, int N, int H, int W, int Cin,
                      const double *offset, const double *mask,
                      const double *weight, const double *bias, int Cout,
                      int Kh, int Kw, int sh, int sw, int ph, int pw, int dh, int dw,
                      int G, const int64_t *pix_idx, int n_pix, int quant_mode, double *y_out) {
    int Ho = oracle_out_size(H, Kh, sh, ph, dh);
    int Wo = oracle_out_size(W, Kw, sw, pw, dw);
    if (dcn_check(N, H, W, Cin, Cout, Kh, Kw, sh, sw, dh, dw, G, Ho, Wo)) return 1;
    const int KK = Kh * Kw;
    for (int t = 0; t < n_pix; ++t)
        if (pix_idx[t] < 0 || pix_idx[t] >= (int64_t)N * Ho * Wo) return 1;
    int fail = 0;
#pragma omp parallel
    {
        double *col = (double *)malloc(sizeof(double) * (size_t)KK * Cin);
        if (!col) {
#pragma omp atomic write
            fail = 1;
        }
#pragma omp for schedule(dynamic, 1)
        for (int t = 0; t < n_pix; ++t) {
            if (!col) continue;
            long pix = (long)pix_idx[t];
            int wo = (int)(pix % Wo);
            int ho = (int)((pix / Wo) % Ho);
            int n = (int)(pix / ((long)Wo * Ho));
            dcn_one_pixel(x, H, W, Cin, offset + pix * G * KK * 2,
                          mask ? mask + pix * G * KK : NULL, weight, bias, Cout,
                          Kh, Kw, sh, sw, ph, pw, dh, dw, G, n, ho, wo, quant_mode,
                          col, y_out + (long)t * Cout);
        }
        free(col);
    }
    return fail ? 2 : 0;
}

int oracle_dcn_pixels_f64(const double *x, int N, int H, int W, int Cin,
                          const double *offset, const double *mask,
                          const double *weight, const double *bias, int Cout,
                          int Kh, int Kw, int sh, int sw, int ph, int pw, int dh, int dw,
                          int G, const int64_t *pix_idx, int n_pix, double *y_out) {
    return dcn_pixels(x, N, H, W, Cin, offset, mask, weight, bias, Cout, Kh, Kw, sh, sw, ph, pw,
                      dh, dw, G, pix_idx, n_pix, 0, y_out);
}

/* The texture-filter model (R14, as oracle_dcn_forward_texq_f64) at sampled output pixels,
 * so full-size texture-sampler launches can be checked against it. */
int oracle_dcn_pixels_texq_f64(const double *x, int N, int H, int W, int Cin,
                               const double *offset, const double *mask,
                               const double *weight, const double *bias, int Cout,
                               int Kh, int Kw, int sh, int sw, int ph, int pw, int dh, int dw,
                               int G, int quant_mode, const int64_t *pix_idx, int n_pix,
                               double *y_out) {
    if (quant_mode < 1 || quant_mode > 3) return 1;
    return dcn_pixels(x, N, H, W, Cin, offset, mask, weight, bias, Cout, Kh, Kw, sh, sw, ph, pw,
                      dh, dw, G, pix_idx, n_pix, quant_mode, y_out);
}

/*
 * Lightweight offset branch, P:170 (W1: C x 1 x 3 x 3 depthwise, W2: OC x C x 1 x 1)
 * and P:180 (BN + ReLU after the depthwise conv only; the 1x1 is linear).
 * BN is folded to a per-channel affine (scale, shift) at inference (R10).
 *
 *   t[c]   = max(0, scale[c] * sum_{a,b<3} W1[c][a][b] * x[n][ho*s-pad+a*d][wo*s-pad+b*d][c] + shift[c])
 *            (zero padding outside the image)
 *   u[o]   = pw_b[o] + sum_c W2[o][c] * t[c],   o < OC = G*K*K*(with_mask ? 3 : 2)   (R11)
 *   offset[n][ho][wo][:] = u[0 : 2*G*K*K]                     (layout [G][K*K][2], R4)
 *   mask  [n][ho][wo][:] = 1 / (1 + exp(-u[2*G*K*K : 3*G*K*K])) (layout [G][K*K], R6)
 *
 * The grid (Ho, Wo) uses the dw conv's own stride/pad/dil with kernel 3 (R10).
 */
int oracle_offset_branch_f64(const double *x, int N, int H, int W, int C,
                             const double *dw_w, const double *dw_scale, const double *dw_shift,
                             const double *pw_w, const double *pw_b,
                             int K, int G, int with_mask,
                             int s, int pad, int dil,
                             double *offset, double *mask) {
    if (N <= 0 || H <= 0 || W <= 0 || C <= 0 || K <= 0 || G <= 0 || s <= 0 || dil <= 0) return 1;
    if (with_mask && !mask) return 1;
    int Ho = oracle_out_size(H, 3, s, pad, dil);
    int Wo = oracle_out_size(W, 3, s, pad, dil);
    if (Ho <= 0 || Wo <= 0) return 1;
    const int KK = K * K;
    const int n_off = 2 * G * KK;
    const int n_msk = with_mask ? G * KK : 0;
    const int OC = n_off + n_msk;
    int fail = 0;
#pragma omp parallel
    {
        double *t = (double *)malloc(sizeof(double) * (size_t)C);
        if (!t) {
#pragma omp atomic write
            fail = 1;
        }
#pragma omp for schedule(dynamic, 1)
        for (long row = 0; row < (long)N * Ho; ++row) {
            if (!t) continue;
            int n = (int)(row / Ho), ho = (int)(row % Ho);
            const double *img = x + (long)n * H * W * C;
            for (int wo = 0; wo < Wo; ++wo) {
                long pix = ((long)n * Ho + ho) * Wo + wo;
                for (int c = 0; c < C; ++c) {
                    double acc = 0.0;
                    for (int a = 0; a < 3; ++a) {
                        int yy = ho * s - pad + a * dil;
                        if (yy < 0 || yy >= H) continue;
                        for (int b = 0; b < 3; ++b) {
                            int xx = wo * s - pad + b * dil;
                            if (xx < 0 || xx >= W) continue;
                            acc += dw_w[(long)c * 9 + a * 3 + b] * img[((long)yy * W + xx) * C + c];
                        }
                    }
                    double v = dw_scale[c] * acc + dw_shift[c];
                    t[c] = v > 0.0 ? v : 0.0;
                }
                for (int o = 0; o < OC; ++o) {
                    double u = pw_b ? pw_b[o] : 0.0;
                    for (int c = 0; c < C; ++c) u += pw_w[(long)o * C + c] * t[c];
                    if (o < n_off)
                        offset[pix * n_off + o] = u;
                    else
                        mask[pix * n_msk + (o - n_off)] = 1.0 / (1.0 + exp(-u));
                }
            }
        }
        free(t);
    }
    return fail ? 2 : 0;
}

/* Deformable columns (the sampling step alone, P:69-76 / Eq.3 + mask): for each flattened
 * output pixel pix_idx[t] = (n*Ho + ho)*Wo + wo, cols[t][k*Cin + ci] as in dcn_pixel_col.
 * Returns 0 on success, 1 on invalid arguments. */
int oracle_deform_columns_f64(const double *x, int N, int H, int W, int Cin,
                              const double *offset, const double *mask,
                              int Kh, int Kw, int sh, int sw, int ph, int pw, int dh, int dw,
                              int G, const int64_t *pix_idx, long n_pix, double *cols) {
    int Ho = oracle_out_size(H, Kh, sh, ph, dh);
    int Wo = oracle_out_size(W, Kw, sw, pw, dw);
    if (dcn_check(N, H, W, Cin, 1, Kh, Kw, sh, sw, dh, dw, G, Ho, Wo)) return 1;
    const long KKC = (long)Kh * Kw * Cin;
    for (long t = 0; t < n_pix; ++t)
        if (pix_idx[t] < 0 || pix_idx[t] >= (long)N * Ho * Wo) return 1;
#pragma omp parallel for schedule(dynamic, 16)
    for (long t = 0; t < n_pix; ++t) {
        long pix = pix_idx[t];
        int n = (int)(pix / ((long)Ho * Wo));
        int rem = (int)(pix % ((long)Ho * Wo));
        int ho = rem / Wo, wo = rem % Wo;
        dcn_pixel_col(x, H, W, Cin, offset + pix * G * Kh * Kw * 2,
                      mask ? mask + pix * G * Kh * Kw : NULL, Kh, Kw, sh, sw, ph, pw, dh, dw, G,
                      n, ho, wo, 0, cols + t * KKC);
    }
    return 0;
}

/* Bounded deformation (section III-A-c, reading R12): before the deformable kernel is
 * applied, each learned offset is restricted so that the sampling point of tap (i, j) stays in
 * the P x P window centred on the output pixel's centre tap.  Written per axis: with the tap's
 * regular displacement from the centre tap r = (i - (Kh-1)/2) * dh (resp. (j - (Kw-1)/2) * dw)
 * and h = (P - 1) / 2, the bounded offset is clamp(r + d, -h, h) - r.  P <= 0: unbounded (the
 * offsets are copied).  A NaN offset stays NaN.  offset / out: [n_pix][G][Kh*Kw][2] (dy, dx);
 * out may alias offset.  Returns 0, or 1 on invalid arguments. */
int oracle_bound_offsets_f64(const double *offset, long n_pix, int G, int Kh, int Kw, int dh, int dw,
                             int P, double *out) {
    if (n_pix < 0 || G <= 0 || Kh <= 0 || Kw <= 0 || dh <= 0 || dw <= 0) return 1;
    const double h = 0.5 * (P - 1);
    for (long p = 0; p < n_pix; ++p)
        for (int g = 0; g < G; ++g)
            for (int i = 0; i < Kh; ++i)
                for (int j = 0; j < Kw; ++j) {
                    const long e = ((p * G + g) * Kh * Kw + (long)i * Kw + j) * 2;
                    const double ry = (i - 0.5 * (Kh - 1)) * dh;   /* regular displacement */
                    const double rx = (j - 0.5 * (Kw - 1)) * dw;
                    double dy = offset[e], dx = offset[e + 1];
                    if (P > 0) {
                        double sy = ry + dy, sx = rx + dx;        /* point relative to the centre */
                        if (sy < -h) sy = -h;
                        if (sy > h) sy = h;
                        if (sx < -h) sx = -h;
                        if (sx > h) sx = h;
                        dy = sy - ry;
                        dx = sx - rx;
                    }
                    out[e] = dy;
                    out[e + 1] = dx;
                }
    return 0;
}

/* tex2D++ (reading R13): the offsets and mask stored in 16 bits -- IEEE binary16, round to
 * nearest even (round_to_f16 above) -- before the deformable kernel forms its coordinates.
 * out may alias in.  Returns 0. */
int oracle_round_f16_array(const double *in, long n, double *out) {
    for (long i = 0; i < n; ++i) out[i] = round_to_f16(in[i]);
    return 0;
}
