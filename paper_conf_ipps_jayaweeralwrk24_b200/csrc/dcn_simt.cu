// dcn_simt.cu -- deformable convolution forward on the CUDA cores (FFMA), the simple
// anchor for the fp32 path and the general fallback for shapes the tensor-core kernel
// does not tile (e.g. Cin/G not a multiple of 64).
//
// Same computation as dcn_tc_bf16.cu: Eq.2 + Eq.3, zero
// outside the image, offset groups, DCNv2 mask (R6).  A classic smem-tiled
// SIMT GEMM whose A tile (64 pixels x 32 kd) is produced by in-block bilinear gathers
// (fp32 weights and lerp) and whose B tile is the weight slice; fp32 accumulation.
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
                const float dy = a.offset[(pix * g.KK + tap) * 2];
                const float dx = a.offset[(pix * g.KK + tap) * 2 + 1];
                const float mk = a.mask ? a.mask[pix * g.KK + tap] : 1.f;
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

}  // namespace

cudaError_t launch_dcn_simt(const DcnGeom& g, const DcnPtrs& p, bool bf16, cudaStream_t stream) {
    SimtArgs a{p.x, p.offset, p.mask, p.weight, p.bias, p.y, g};
    dim3 grid((g.M + TM - 1) / TM, (g.Cout + TN - 1) / TN);
    if (bf16)
        dcn_fwd_simt_kernel<true><<<grid, THREADS, 0, stream>>>(a);
    else
        dcn_fwd_simt_kernel<false><<<grid, THREADS, 0, stream>>>(a);
    return cudaGetLastError();
}

}  // namespace defcon
