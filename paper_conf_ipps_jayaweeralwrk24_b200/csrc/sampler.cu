// sampler.cu -- the sampling step alone ("two-step" deformable conv):
//   cols[m][k*Cin + ci] = m_k * X(p_o + p_k + dp_k)     Eq.3, zero outside,
// i.e. the deformable im2col rows, written to HBM.  It is the unfused baseline's first
// step (columns + a library GEMM) and the measurement of the sampling stage on its own
// (HBM-bound, GB/s and elements/clk/SM).  The fused kernel
// (dcn_tc_bf16.cu) produces the same values into shared memory and never writes them.
//
// Thread = one 32-byte piece (16 bf16 / 8 fp32 channels) of one (pixel, tap) row segment
// (256-bit corner gathers and column stores); the linear index runs piece-fastest, then
// tap, then pixel, so the column writes are contiguous and the corner gathers of
// neighbouring threads are contiguous runs of the same NHWC pixel.  Needs (Cin/G) * ES a
// multiple of 32 bytes (bf16 Cin/G % 16, fp32 % 8).  fp32 weights and lerp (FFMA2); bf16
// output RNE.
#include <cstdlib>

#include "common.cuh"
#include "kernels.h"

namespace defcon {
namespace {

struct ColArgs {
    const void* x;
    const float* offset;
    const float* mask;
    void* cols;
    int H, W, Cin, Kw, Ho, Wo;
    int sh, sw, ph, pw, dh, dw;
    int G, Cg, M, KK;
    float bound_h;       // bounded deformation half-window (R12); < 0: unbounded
    int off_f16;         // offsets / mask in binary16 (tex2D++, R13)
    int pieces;          // 32-byte pieces per (pixel, tap) row = Cin * ES / 32
    long long total;     // M * KK * pieces
};

// One piece of one (pixel, tap) row: fp32 bilinear sum of CPP channels (32 bytes of x).
template <bool BF16>
struct Piece {
    static constexpr int ES = BF16 ? 2 : 4;
    static constexpr int CPP = 32 / ES;                // channels per 32-byte piece
    U8x32 v[4];
    float w[4];
};

template <bool BF16>
__device__ __forceinline__ void piece_issue(const ColArgs& a, long long u, Piece<BF16>& P, long& dst_off) {
    constexpr int CPP = Piece<BF16>::CPP, ES = Piece<BF16>::ES;
    const int piece = (int)(u % a.pieces);
    const long long mk = u / a.pieces;
    const int k = (int)(mk % a.KK);
    const int m = (int)(mk / a.KK);
    const int c0 = piece * CPP;
    const int g = c0 / a.Cg;
    const int hw = a.Ho * a.Wo;
    const int n = m / hw;
    const int rem = m - n * hw;
    const int ho = rem / a.Wo;
    const int wo = rem - ho * a.Wo;
    const int i = k / a.Kw, j = k - (k / a.Kw) * a.Kw;
    const long pix = (long)m * a.G + g;
    float2 d = ld_offset2(a.offset, (pix * a.KK + k) * 2, a.off_f16);
    d.x = bound_offset(d.x, (i - 0.5f * (a.KK / a.Kw - 1)) * a.dh, a.bound_h);   // P:182, R12
    d.y = bound_offset(d.y, (j - 0.5f * (a.Kw - 1)) * a.dw, a.bound_h);
    const float mv = a.mask ? ld_mask1(a.mask, pix * a.KK + k, a.off_f16) : 1.f;
    float py = (float)(ho * a.sh - a.ph + i * a.dh) + d.x;
    float px = (float)(wo * a.sw - a.pw + j * a.dw) + d.y;
    py = fminf(fmaxf(py, -2.f), (float)a.H + 1.f);     // beyond one pixel out: zeros only
    px = fminf(fmaxf(px, -2.f), (float)a.W + 1.f);
    const uint8_t* img = reinterpret_cast<const uint8_t*>(a.x) + ((long)n * a.H * a.W * a.Cin + c0) * ES;
    long off[4] = {0, 0, 0, 0};
#pragma unroll
    for (int q = 0; q < 4; ++q) P.w[q] = 0.f;
    if (py == py && px == px) {
        const float fy = floorf(py), fx = floorf(px);
        const float ly = py - fy, lx = px - fx;
        const int y0 = (int)fy, x0 = (int)fx;
        const float wq[4] = {(1.f - ly) * (1.f - lx) * mv, (1.f - ly) * lx * mv, ly * (1.f - lx) * mv, ly * lx * mv};
#pragma unroll
        for (int q = 0; q < 4; ++q) {
            const int yy = y0 + (q >> 1), xx = x0 + (q & 1);
            if (yy >= 0 && yy < a.H && xx >= 0 && xx < a.W) {   // else: weight 0, harmless in-image load
                P.w[q] = wq[q];
                off[q] = ((long)yy * a.W + xx) * a.Cin * ES;
            }
        }
    }
#pragma unroll
    for (int q = 0; q < 4; ++q) P.v[q] = ldg_nc_v8(img + off[q]);
    dst_off = (((long)m * a.KK + k) * a.Cin + c0) * ES;
}

template <bool BF16>
__device__ __forceinline__ void piece_store(const ColArgs& a, const Piece<BF16>& P, long dst_off) {
    uint8_t* dst = static_cast<uint8_t*>(a.cols) + dst_off;
    uint32_t o[8];
    if (BF16) {
        uint64_t acc[8];
#pragma unroll
        for (int q = 0; q < 4; ++q) {
            const uint64_t w2 = f32x2_pack(P.w[q], P.w[q]);
#pragma unroll
            for (int h = 0; h < 8; ++h) {
                const uint64_t c = bf16x2_to_f32x2(P.v[q].w[h]);
                acc[h] = q == 0 ? f32x2_mul(c, w2) : f32x2_fma(c, w2, acc[h]);
            }
        }
#pragma unroll
        for (int h = 0; h < 8; ++h) o[h] = f32x2_to_bf16x2(acc[h]);
    } else {
        uint64_t acc[4];
#pragma unroll
        for (int q = 0; q < 4; ++q) {
            const uint64_t w2 = f32x2_pack(P.w[q], P.w[q]);
#pragma unroll
            for (int h = 0; h < 4; ++h) {
                const uint64_t c = ((uint64_t)P.v[q].w[2 * h + 1] << 32) | P.v[q].w[2 * h];
                acc[h] = q == 0 ? f32x2_mul(c, w2) : f32x2_fma(c, w2, acc[h]);
            }
        }
#pragma unroll
        for (int h = 0; h < 4; ++h) {
            o[2 * h] = (uint32_t)(acc[h] & 0xFFFFFFFFull);
            o[2 * h + 1] = (uint32_t)(acc[h] >> 32);
        }
    }
    asm volatile("st.global.v8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(dst), "r"(o[0]), "r"(o[1]), "r"(o[2]),
                 "r"(o[3]), "r"(o[4]), "r"(o[5]), "r"(o[6]), "r"(o[7])
                 : "memory");
}

// Two pieces in flight per thread (the second's gathers issued before the first is
// finished); grid-stride over all pieces.
template <bool BF16>
__global__ void __launch_bounds__(256) deform_columns_kernel(const ColArgs a) {
    griddep_wait();
    griddep_launch_dependents();
    const long long stride = (long long)gridDim.x * blockDim.x;
    for (long long u = (long long)blockIdx.x * blockDim.x + threadIdx.x; u < a.total; u += 2 * stride) {
        Piece<BF16> P0, P1;
        long d0, d1 = 0;
        piece_issue<BF16>(a, u, P0, d0);
        const bool two = u + stride < a.total;
        if (two) piece_issue<BF16>(a, u + stride, P1, d1);
        piece_store<BF16>(a, P0, d0);
        if (two) piece_store<BF16>(a, P1, d1);
    }
}

// Row-mapped variant: a (pixel, tap) row is PIECES consecutive lanes (32 / PIECES rows per warp),
// all index math 32-bit and done once per row (each lane of the row recomputes it from the same
// broadcast offset / mask loads -- no 64-bit divisions), two rows in flight per thread.
// The row's (dy, dx, mask) -- loaded one iteration ahead of its use (software pipelining), so
// a row costs one dependent memory round trip (the corner gathers), not two.
struct RowMeta {
    float2 d;
    float mv;
};

template <bool BF16>
__device__ __forceinline__ RowMeta row_meta(const ColArgs& a, int r, int piece) {
    RowMeta q;
    q.d = make_float2(0.f, 0.f);
    q.mv = 0.f;
    if (r >= a.M * a.KK) return q;
    const int m = r / a.KK, k = r - (r / a.KK) * a.KK;
    const int g = piece * Piece<BF16>::CPP / a.Cg;
    const int pix = m * a.G + g;
    q.d = ld_offset2(a.offset, ((long)pix * a.KK + k) * 2, a.off_f16);
    q.mv = a.mask ? ld_mask1(a.mask, (long)pix * a.KK + k, a.off_f16) : 1.f;
    return q;
}

template <bool BF16, int PIECES>
__device__ __forceinline__ void row_issue(const ColArgs& a, int r, int piece, const RowMeta& rm, Piece<BF16>& P,
                                          long& dst_off) {
    constexpr int CPP = Piece<BF16>::CPP, ES = Piece<BF16>::ES;
    const int m = r / a.KK, k = r - (r / a.KK) * a.KK;
    const int c0 = piece * CPP;
    const int hw = a.Ho * a.Wo;
    const int n = m / hw;
    const int rem = m - n * hw;
    const int ho = rem / a.Wo;
    const int wo = rem - ho * a.Wo;
    const int i = k / a.Kw, j = k - (k / a.Kw) * a.Kw;
    float2 d = rm.d;
    d.x = bound_offset(d.x, (i - 0.5f * (a.KK / a.Kw - 1)) * a.dh, a.bound_h);   // P:182, R12
    d.y = bound_offset(d.y, (j - 0.5f * (a.Kw - 1)) * a.dw, a.bound_h);
    const float mv = rm.mv;
    float py = (float)(ho * a.sh - a.ph + i * a.dh) + d.x;
    float px = (float)(wo * a.sw - a.pw + j * a.dw) + d.y;
    py = fminf(fmaxf(py, -2.f), (float)a.H + 1.f);     // beyond one pixel out: zeros only
    px = fminf(fmaxf(px, -2.f), (float)a.W + 1.f);
    const uint8_t* img = reinterpret_cast<const uint8_t*>(a.x) + ((size_t)n * a.H * a.W * a.Cin + c0) * ES;
    int off[4] = {0, 0, 0, 0};
#pragma unroll
    for (int q = 0; q < 4; ++q) P.w[q] = 0.f;
    if (py == py && px == px) {
        const float fy = floorf(py), fx = floorf(px);
        const float ly = py - fy, lx = px - fx;
        const int y0 = (int)fy, x0 = (int)fx;
        const float wq[4] = {(1.f - ly) * (1.f - lx) * mv, (1.f - ly) * lx * mv, ly * (1.f - lx) * mv, ly * lx * mv};
#pragma unroll
        for (int q = 0; q < 4; ++q) {
            const int yy = y0 + (q >> 1), xx = x0 + (q & 1);
            if (yy >= 0 && yy < a.H && xx >= 0 && xx < a.W) {   // else: weight 0, harmless in-image load
                P.w[q] = wq[q];
                off[q] = (yy * a.W + xx) * a.Cin;
            }
        }
    }
#pragma unroll
    for (int q = 0; q < 4; ++q) P.v[q] = ldg_nc_v8(img + (size_t)off[q] * ES);
    dst_off = ((long)r * a.Cin + c0) * ES;
}

template <bool BF16, int PIECES>
__global__ void __launch_bounds__(256) deform_columns_rows_kernel(const ColArgs a) {
    griddep_wait();
    griddep_launch_dependents();
    constexpr int RPW = 32 / PIECES;                       // rows per warp per step
    const int lane = threadIdx.x & 31;
    const int piece = lane % PIECES, sub = lane / PIECES;
    const int warps = gridDim.x * (blockDim.x >> 5);
    const int gw = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
    const int rows = a.M * a.KK;
    const int stride = warps * RPW;
    int r = gw * RPW + sub;
    RowMeta q0 = row_meta<BF16>(a, r, piece), q1 = row_meta<BF16>(a, r + stride, piece);
    for (; r < rows; r += 2 * stride) {
        Piece<BF16> P0, P1;
        long d0, d1 = 0;
        row_issue<BF16, PIECES>(a, r, piece, q0, P0, d0);
        const bool two = r + stride < rows;
        if (two) row_issue<BF16, PIECES>(a, r + stride, piece, q1, P1, d1);
        q0 = row_meta<BF16>(a, r + 2 * stride, piece);      // next iteration's rows
        q1 = row_meta<BF16>(a, r + 3 * stride, piece);
        piece_store<BF16>(a, P0, d0);
        if (two) piece_store<BF16>(a, P1, d1);
    }
}

}  // namespace

cudaError_t launch_deform_columns(const DcnGeom& g, const void* x, const float* offset, const float* mask,
                                  bool bf16, void* cols, cudaStream_t stream) {
    ColArgs a;
    a.x = x; a.offset = offset; a.mask = mask; a.cols = cols;
    a.H = g.H; a.W = g.W; a.Cin = g.Cin; a.Kw = g.Kw; a.Ho = g.Ho; a.Wo = g.Wo;
    a.sh = g.sh; a.sw = g.sw; a.ph = g.ph; a.pw = g.pw; a.dh = g.dh; a.dw = g.dw;
    a.G = g.G; a.Cg = g.Cg; a.M = g.M; a.KK = g.KK;
    a.bound_h = g.bound_h;
    a.off_f16 = g.off_f16;
    a.pieces = g.Cin * (bf16 ? 2 : 4) / 32;
    a.total = (long long)g.M * g.KK * a.pieces;
    int dev = 0, nsm = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    const long long blocks = (a.total + 255) / 256;
    const int grid = (int)(blocks < (long long)nsm * 8 ? blocks : (long long)nsm * 8);
    // row-mapped kernel when a row is 8 / 16 / 32 pieces and every index fits 32 bits
    const bool rows32 = (long long)g.M * g.KK * g.Cin < (1ll << 31) &&
                        (long long)g.N * g.H * g.W * g.Cin < (1ll << 31);
    if (rows32 && (a.pieces == 8 || a.pieces == 16 || a.pieces == 32)) {
        auto pick = [&](auto kb, auto kf) { return bf16 ? kb : kf; };
        void (*kern)(ColArgs) =
            a.pieces == 8 ? pick(deform_columns_rows_kernel<true, 8>, deform_columns_rows_kernel<false, 8>)
            : a.pieces == 16 ? pick(deform_columns_rows_kernel<true, 16>, deform_columns_rows_kernel<false, 16>)
                             : pick(deform_columns_rows_kernel<true, 32>, deform_columns_rows_kernel<false, 32>);
        return launch_pdl(kern, dim3(nsm * 2), dim3(256), 0, stream, a);   // 2 blocks per SM resident
    }
    return bf16 ? launch_pdl(deform_columns_kernel<true>, dim3(grid), dim3(256), 0, stream, a)
                : launch_pdl(deform_columns_kernel<false>, dim3(grid), dim3(256), 0, stream, a);
}

}  // namespace defcon
