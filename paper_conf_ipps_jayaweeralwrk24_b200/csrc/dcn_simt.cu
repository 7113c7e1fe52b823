// dcn_simt.cu -- deformable convolution forward on the CUDA cores (FFMA), the simple
// anchor for the fp32 path and the general fallback for shapes the tensor-core kernel
// does not tile (e.g. Cin/G not a multiple of 64).
//
// Same computation as dcn_tc_bf16.cu: Eq.2 + Eq.3, zero
// outside the image, offset groups, DCNv2 mask (R6).  A classic smem-tiled
// SIMT GEMM whose A tile (64 pixels x 32 kd) is produced by in-block bilinear gathers
// (fp32 weights and lerp) and whose B tile is the weight slice; fp32 accumulation.
#include <cstdlib>

#include "common.cuh"
#include "kernels.h"

namespace defcon {
namespace {

constexpr int TM = 64;    // output pixels per block
constexpr int TN = 64;    // output channels per block
constexpr int TK = 32;    // kd per step
constexpr int THREADS = 256;

struct SimtArgs {
    const void* x;
    const float* offset;
    const float* mask;
    const void* weight;
    const float* bias;
    void* y;
    DcnGeom g;
};

template <bool BF16>
__device__ __forceinline__ void load4(const void* base, long idx, float (&v)[4]) {
    if (BF16) {
        const uint2 u = *reinterpret_cast<const uint2*>(static_cast<const __nv_bfloat16*>(base) + idx);
        v[0] = bf16lo_to_f32(u.x);
        v[1] = bf16hi_to_f32(u.x);
        v[2] = bf16lo_to_f32(u.y);
        v[3] = bf16hi_to_f32(u.y);
    } else {
        const float4 f = *reinterpret_cast<const float4*>(static_cast<const float*>(base) + idx);
        v[0] = f.x; v[1] = f.y; v[2] = f.z; v[3] = f.w;
    }
}

template <bool BF16>
__global__ void __launch_bounds__(THREADS) dcn_fwd_simt_kernel(const SimtArgs a) {
    const DcnGeom& g = a.g;
    __shared__ float As[TK][TM + 4];
    __shared__ float Bs[TK][TN + 4];
    const int t = threadIdx.x;
    const int m0 = blockIdx.x * TM;
    const int n0 = blockIdx.y * TN;
    const int Kd = g.KK * g.Cin;
    const int tx = t & 15, ty = t >> 4;   // 16 x 16 threads, 4 x 4 outputs each

    float acc[4][4];
#pragma unroll
    for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[i][j] = 0.f;

    for (int k0 = 0; k0 < Kd; k0 += TK) {
        // ---- A: 64 pixels x 32 kd, each thread 2 groups of 4 consecutive kd
#pragma unroll
        for (int r = 0; r < 2; ++r) {
            const int e = t + r * THREADS;        // 0..511
            const int pl = e >> 3;                // pixel in tile 0..63
            const int kq = (e & 7) * 4;           // kd offset 0..28
            const int kd = k0 + kq;
            const int m = m0 + pl;
            float v[4] = {0.f, 0.f, 0.f, 0.f};
            if (m < g.M && kd < Kd) {
                const int tap = kd / g.Cin;
                const int ci = kd - tap * g.Cin;
                const int grp = ci / g.Cg;
                const int hw = g.Ho * g.Wo;
                const int n = m / hw;
                const int rem = m - n * hw;
                const int ho = rem / g.Wo, wo = rem - (rem / g.Wo) * g.Wo;
                const int i = tap / g.Kw, j = tap - (tap / g.Kw) * g.Kw;
                const long pix = (long)m * g.G + grp;
                const float2 d = ld_offset2(a.offset, (pix * g.KK + tap) * 2, g.off_f16);
                const float dy = bound_offset(d.x, (i - 0.5f * (g.Kh - 1)) * g.dh,
                                              g.bound_h);   // bounded deformation (R12)
                const float dx = bound_offset(d.y, (j - 0.5f * (g.Kw - 1)) * g.dw, g.bound_h);
                const float mk = a.mask ? ld_mask1(a.mask, pix * g.KK + tap, g.off_f16) : 1.f;
                float py = (float)(ho * g.sh - g.ph + i * g.dh) + dy;
                float px = (float)(wo * g.sw - g.pw + j * g.dw) + dx;
                py = fminf(fmaxf(py, -2.f), (float)g.H + 1.f);
                px = fminf(fmaxf(px, -2.f), (float)g.W + 1.f);
                if (py == py && px == px) {
                    const float fy = floorf(py), fx = floorf(px);
                    const float ly = py - fy, lx = px - fx;
                    const int y0 = (int)fy, x0 = (int)fx;
#pragma unroll
                    for (int q = 0; q < 4; ++q) {
                        const int yy = y0 + (q >> 1), xx = x0 + (q & 1);
                        if (yy < 0 || yy >= g.H || xx < 0 || xx >= g.W) continue;
                        const float wq = ((q >> 1) ? ly : 1.f - ly) * ((q & 1) ? lx : 1.f - lx) * mk;
                        float c[4];
                        load4<BF16>(a.x, ((long)(n * g.H + yy) * g.W + xx) * g.Cin + ci, c);
#pragma unroll
                        for (int u = 0; u < 4; ++u) v[u] = fmaf(wq, c[u], v[u]);
                    }
                }
            }
#pragma unroll
            for (int u = 0; u < 4; ++u) As[kq + u][pl] = v[u];
        }
        // ---- B: 64 cout x 32 kd
#pragma unroll
        for (int r = 0; r < 2; ++r) {
            const int e = t + r * THREADS;
            const int nl = e >> 3;
            const int kq = (e & 7) * 4;
            const int co = n0 + nl;
            const int kd = k0 + kq;
            float v[4] = {0.f, 0.f, 0.f, 0.f};
            if (co < g.Cout && kd < Kd) load4<BF16>(a.weight, (long)co * Kd + kd, v);
#pragma unroll
            for (int u = 0; u < 4; ++u) Bs[kq + u][nl] = v[u];
        }
        __syncthreads();
#pragma unroll 8
        for (int kk = 0; kk < TK; ++kk) {
            float av[4], bv[4];
#pragma unroll
            for (int i = 0; i < 4; ++i) av[i] = As[kk][ty * 4 + i];
#pragma unroll
            for (int j = 0; j < 4; ++j) bv[j] = Bs[kk][tx * 4 + j];
#pragma unroll
            for (int i = 0; i < 4; ++i)
#pragma unroll
                for (int j = 0; j < 4; ++j) acc[i][j] = fmaf(av[i], bv[j], acc[i][j]);
        }
        __syncthreads();
    }
    // ---- epilogue
#pragma unroll
    for (int i = 0; i < 4; ++i) {
        const int m = m0 + ty * 4 + i;
        if (m >= g.M) continue;
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            const int co = n0 + tx * 4 + j;
            if (co >= g.Cout) continue;
            const float v = acc[i][j] + (a.bias ? a.bias[co] : 0.f);
            if (BF16)
                static_cast<__nv_bfloat16*>(a.y)[(long)m * g.Cout + co] = __float2bfloat16_rn(v);
            else
                static_cast<float*>(a.y)[(long)m * g.Cout + co] = v;
        }
    }
}

// ------------------------------------------------------------------ fp32 path, register-tiled
// The fp32 storage path on the CUDA cores (the FP32 FFMA pipe, 128 FMA/clk/SM, is its bound).
// Block tile = 80 output pixels x 256 output channels (one gather of A serves all of Cout <= 256),
// K walked tap-outer in 16-channel steps.  Gathers: thread t < 160 owns pixel t/2 and 8 of the 16
// channels of each step; its sampling metadata (4 corner offsets, 4 mask-scaled fp32 weights,
// Eq.3) lives in registers and is rebuilt only when the tap or the offset group changes.
// GEMM: warps 2 (pixels) x 4 (channels), lanes 4 x 8, each thread 10 pixels x 8 channels, so
// every shared-memory fragment load is a broadcast of 1 wavefront (FFMA-bound, not LDS-bound).
// (Packed FFMA2 over channel pairs measured slower: 789 vs 728 us at C4 -- it does not raise
// the FP32 pipe's FMA rate and costs an operand pack per pixel.)
constexpr int FT_M = 80;
constexpr int FT_N = 256;
constexpr int FT_K = 16;
constexpr int FT_PX = 10;                  // pixels per thread
constexpr int FT_BS = FT_N + 4;            // Bs row stride

__global__ void __launch_bounds__(THREADS, 2) dcn_fwd_f32_tiled_kernel(const SimtArgs a) {
    const DcnGeom& g = a.g;
    __shared__ __align__(16) float As[FT_K][FT_M];
    __shared__ __align__(16) float Bs[FT_K][FT_BS];
    const int t = threadIdx.x, warp = t >> 5, lane = t & 31;
    const int m0 = blockIdx.x * FT_M;
    const int n0 = blockIdx.y * FT_N;
    const int Kd = g.KK * g.Cin;
    const float* x = static_cast<const float*>(a.x);
    const float* w = static_cast<const float*>(a.weight);
    // gather role
    const bool gat = t < 2 * FT_M;
    const int gpx = t >> 1, ghalf = t & 1;
    const int gm = m0 + gpx;
    const bool gok = gat && gm < g.M;
    int gn = 0, gyb = 0, gxb = 0;
    if (gok) {
        const int hw = g.Ho * g.Wo;
        gn = gm / hw;
        const int rem = gm - gn * hw;
        const int ho = rem / g.Wo;
        gyb = ho * g.sh - g.ph;
        gxb = (rem - ho * g.Wo) * g.sw - g.pw;
    }
    int ctap = -1, cgrp = -1;
    int off[4] = {0, 0, 0, 0};
    float wt[4] = {0.f, 0.f, 0.f, 0.f};
    // GEMM role
    const int wp = warp >> 2, wc = warp & 3;
    const int pg = lane >> 3, cg = lane & 7;
    const int px0 = wp * 40 + pg * FT_PX;
    const int co0 = wc * 64 + cg * 8;
    float acc[FT_PX][8];
#pragma unroll
    for (int i = 0; i < FT_PX; ++i)
#pragma unroll
        for (int j = 0; j < 8; ++j) acc[i][j] = 0.f;

    for (int k0 = 0; k0 < Kd; k0 += FT_K) {
        const int tap = k0 / g.Cin;
        const int ci0 = k0 - tap * g.Cin;
        // ---- A: this thread's 8 channels of pixel gpx
        if (gat) {
            const int grp = ci0 / g.Cg;
            if (tap != ctap || grp != cgrp) {      // rebuild the sampling metadata (Eq.3)
                ctap = tap;
                cgrp = grp;
#pragma unroll
                for (int q = 0; q < 4; ++q) { off[q] = 0; wt[q] = 0.f; }
                if (gok) {
                    const long pix = (long)gm * g.G + grp;
                    const int i = tap / g.Kw, j = tap - (tap / g.Kw) * g.Kw;
                    const float2 d = ld_offset2(a.offset, (pix * g.KK + tap) * 2, g.off_f16);
                    const float dy = bound_offset(d.x, (i - 0.5f * (g.Kh - 1)) * g.dh, g.bound_h);   // P:182, R12
                    const float dx = bound_offset(d.y, (j - 0.5f * (g.Kw - 1)) * g.dw, g.bound_h);
                    const float mk = a.mask ? ld_mask1(a.mask, pix * g.KK + tap, g.off_f16) : 1.f;
                    float py = (float)(gyb + i * g.dh) + dy;
                    float px = (float)(gxb + j * g.dw) + dx;
                    py = fminf(fmaxf(py, -2.f), (float)g.H + 1.f);
                    px = fminf(fmaxf(px, -2.f), (float)g.W + 1.f);
                    if (py == py && px == px) {
                        const float fy = floorf(py), fx = floorf(px);
                        const float ly = py - fy, lx = px - fx;
                        const int y0 = (int)fy, x0 = (int)fx;
#pragma unroll
                        for (int q = 0; q < 4; ++q) {
                            const int yy = y0 + (q >> 1), xx = x0 + (q & 1);
                            if (yy < 0 || yy >= g.H || xx < 0 || xx >= g.W) continue;
                            wt[q] = ((q >> 1) ? ly : 1.f - ly) * ((q & 1) ? lx : 1.f - lx) * mk;
                            off[q] = ((gn * g.H + yy) * g.W + xx) * g.Cin;
                        }
                    }
                }
            }
            const int c = ci0 + ghalf * 8;
            float v[8];
#pragma unroll
            for (int u = 0; u < 8; ++u) v[u] = 0.f;
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                const float4* src = reinterpret_cast<const float4*>(x + off[q] + c);
                const float4 c0 = __ldg(src), c1 = __ldg(src + 1);
                v[0] = fmaf(wt[q], c0.x, v[0]); v[1] = fmaf(wt[q], c0.y, v[1]);
                v[2] = fmaf(wt[q], c0.z, v[2]); v[3] = fmaf(wt[q], c0.w, v[3]);
                v[4] = fmaf(wt[q], c1.x, v[4]); v[5] = fmaf(wt[q], c1.y, v[5]);
                v[6] = fmaf(wt[q], c1.z, v[6]); v[7] = fmaf(wt[q], c1.w, v[7]);
            }
#pragma unroll
            for (int u = 0; u < 8; ++u) As[ghalf * 8 + u][gpx] = v[u];
        }
        // ---- B: 16 kd x 256 co, float4 along kd
#pragma unroll
        for (int r = 0; r < FT_K * FT_N / 4 / THREADS; ++r) {
            const int e = t + r * THREADS;
            const int nl = e >> 2, kq = (e & 3) * 4;
            const int co = n0 + nl;
            float4 b = make_float4(0.f, 0.f, 0.f, 0.f);
            if (co < g.Cout) b = __ldg(reinterpret_cast<const float4*>(w + (long)co * Kd + k0 + kq));
            Bs[kq][nl] = b.x; Bs[kq + 1][nl] = b.y; Bs[kq + 2][nl] = b.z; Bs[kq + 3][nl] = b.w;
        }
        __syncthreads();
#pragma unroll 4
        for (int kk = 0; kk < FT_K; ++kk) {
            float av[FT_PX], bv[8];
#pragma unroll
            for (int i = 0; i < FT_PX; i += 2) {
                const float2 f = *reinterpret_cast<const float2*>(&As[kk][px0 + i]);
                av[i] = f.x; av[i + 1] = f.y;
            }
            const float4 b0 = *reinterpret_cast<const float4*>(&Bs[kk][co0]);
            const float4 b1 = *reinterpret_cast<const float4*>(&Bs[kk][co0 + 4]);
            bv[0] = b0.x; bv[1] = b0.y; bv[2] = b0.z; bv[3] = b0.w;
            bv[4] = b1.x; bv[5] = b1.y; bv[6] = b1.z; bv[7] = b1.w;
#pragma unroll
            for (int i = 0; i < FT_PX; ++i)
#pragma unroll
                for (int j = 0; j < 8; ++j) acc[i][j] = fmaf(av[i], bv[j], acc[i][j]);
        }
        __syncthreads();
    }
    // ---- epilogue: + bias, fp32 NHWC
    float bb[8];
#pragma unroll
    for (int j = 0; j < 8; ++j) {
        const int co = n0 + co0 + j;
        bb[j] = (a.bias && co < g.Cout) ? __ldg(a.bias + co) : 0.f;
    }
    float* y = static_cast<float*>(a.y);
    const bool full8 = n0 + co0 + 8 <= g.Cout;
#pragma unroll
    for (int i = 0; i < FT_PX; ++i) {
        const int m = m0 + px0 + i;
        if (m >= g.M) continue;
        if (full8) {
            float4* dst = reinterpret_cast<float4*>(y + (long)m * g.Cout + n0 + co0);
            dst[0] = make_float4(acc[i][0] + bb[0], acc[i][1] + bb[1], acc[i][2] + bb[2], acc[i][3] + bb[3]);
            dst[1] = make_float4(acc[i][4] + bb[4], acc[i][5] + bb[5], acc[i][6] + bb[6], acc[i][7] + bb[7]);
        } else {
#pragma unroll
            for (int j = 0; j < 8; ++j)
                if (n0 + co0 + j < g.Cout) y[(long)m * g.Cout + n0 + co0 + j] = acc[i][j] + bb[j];
        }
    }
}

}  // namespace

cudaError_t launch_dcn_simt(const DcnGeom& g, const DcnPtrs& p, bool bf16, cudaStream_t stream) {
    SimtArgs a{p.x, p.offset, p.mask, p.weight, p.bias, p.y, g};
    // fp32: the register-tiled kernel when the 16-channel steps stay inside one tap and one offset
    // group and the 16-byte vector loads are aligned (Cin, Cg multiples of 16; Cout multiple of 4);
    // otherwise the simple anchor kernel below.
    if (!bf16 && g.Cin % FT_K == 0 && g.Cg % FT_K == 0 && g.Cout % 4 == 0) {
        dim3 grid((g.M + FT_M - 1) / FT_M, (g.Cout + FT_N - 1) / FT_N);
        dcn_fwd_f32_tiled_kernel<<<grid, THREADS, 0, stream>>>(a);
        return cudaGetLastError();
    }
    dim3 grid((g.M + TM - 1) / TM, (g.Cout + TN - 1) / TN);
    if (bf16)
        dcn_fwd_simt_kernel<true><<<grid, THREADS, 0, stream>>>(a);
    else
        dcn_fwd_simt_kernel<false><<<grid, THREADS, 0, stream>>>(a);
    return cudaGetLastError();
}

}  // namespace defcon
