// offset_branch.cu -- the paper's lightweight offset branch,
// fused into one NHWC pass:
//   t[c] = ReLU(scale[c] * sum_{3x3} W1[c] * x + shift[c])    depthwise 3x3 + folded BN
//   u[o] = b2[o] + sum_c W2[o][c] * t[c]                      1x1 to OC = G*K*K*(2|3)
//   offset = u[0 : 2GK^2] ([G][K*K][2] = (dy, dx), R4),  mask = sigmoid(u[2GK^2 :]) (R6)
// One block handles PIX consecutive output pixels: phase 1 computes t for all C channels
// into shared memory (coalesced along C), phase 2 the 1x1 projection with W2 staged
// through shared memory in chunks.  fp32 arithmetic throughout.
#include "common.cuh"
#include "kernels.h"

namespace defcon {
namespace {

constexpr int THREADS = 256;
constexpr int MAXO = 16;       // 1x1 outputs per thread: OC * PIX <= THREADS * MAXO
constexpr int CCH = 64;        // W2 channel chunk staged in smem

struct BranchArgs {
    const void* x;
    const float* dw_w;
    const float* dw_scale;
    const float* dw_shift;
    const float* pw_w;
    const float* pw_b;
    float* offset;
    float* mask;
    int N, H, W, C, Ho, Wo, M;
    int sh, sw, ph, pw, dh, dw;
    int n_off, n_msk, OC;
};

template <bool BF16>
__device__ __forceinline__ float ld_x(const void* x, long idx) {
    if (BF16) return __bfloat162float(static_cast<const __nv_bfloat16*>(x)[idx]);
    return static_cast<const float*>(x)[idx];
}

template <bool BF16, int PIX>
__global__ void __launch_bounds__(THREADS) offset_branch_kernel(const BranchArgs a) {
    extern __shared__ float sm[];
    float* t_s = sm;                              // [PIX][C + 1]
    float* w_s = sm + PIX * (a.C + 1);            // [OC][CCH + 1]
    const int m0 = blockIdx.x * PIX;
    const int tid = threadIdx.x;
    const int ts = a.C + 1;

    // ---- phase 1: depthwise 3x3 + BN + ReLU
    for (int e = tid; e < PIX * a.C; e += THREADS) {
        const int p = e / a.C;
        const int c = e - p * a.C;
        const int m = m0 + p;
        float v = 0.f;
        if (m < a.M) {
            const int hw = a.Ho * a.Wo;
            const int n = m / hw;
            const int rem = m - n * hw;
            const int ho = rem / a.Wo, wo = rem - (rem / a.Wo) * a.Wo;
            float acc = 0.f;
#pragma unroll
            for (int i = 0; i < 3; ++i) {
                const int yy = ho * a.sh - a.ph + i * a.dh;
                if (yy < 0 || yy >= a.H) continue;
#pragma unroll
                for (int j = 0; j < 3; ++j) {
                    const int xx = wo * a.sw - a.pw + j * a.dw;
                    if (xx < 0 || xx >= a.W) continue;
                    acc = fmaf(__ldg(a.dw_w + c * 9 + i * 3 + j),
                               ld_x<BF16>(a.x, ((long)(n * a.H + yy) * a.W + xx) * a.C + c), acc);
                }
            }
            v = fmaxf(fmaf(__ldg(a.dw_scale + c), acc, __ldg(a.dw_shift + c)), 0.f);
        }
        t_s[p * ts + c] = v;
    }

    // ---- phase 2: 1x1 projection, thread -> (o, p) pairs, W2 chunks in smem
    const int n_out = a.OC * PIX;
    float acc[MAXO];
#pragma unroll
    for (int r = 0; r < MAXO; ++r) acc[r] = 0.f;
    for (int c0 = 0; c0 < a.C; c0 += CCH) {
        const int cn = min(CCH, a.C - c0);
        __syncthreads();   // t_s complete (first pass) / previous w_s chunk consumed
        for (int e = tid; e < a.OC * cn; e += THREADS) {
            const int o = e / cn, c = e - (e / cn) * cn;
            w_s[o * (CCH + 1) + c] = __ldg(a.pw_w + (long)o * a.C + c0 + c);
        }
        __syncthreads();
#pragma unroll
        for (int r = 0; r < MAXO; ++r) {
            const int e = tid + r * THREADS;
            if (e < n_out) {
                const int o = e / PIX, p = e - (e / PIX) * PIX;
                const float* wr = w_s + o * (CCH + 1);
                const float* tr = t_s + p * ts + c0;
                float s = acc[r];
                for (int c = 0; c < cn; ++c) s = fmaf(wr[c], tr[c], s);
                acc[r] = s;
            }
        }
    }
#pragma unroll
    for (int r = 0; r < MAXO; ++r) {
        const int e = tid + r * THREADS;
        if (e >= n_out) continue;
        const int o = e / PIX, p = e - (e / PIX) * PIX;
        const int m = m0 + p;
        if (m >= a.M) continue;
        const float u = acc[r] + (a.pw_b ? __ldg(a.pw_b + o) : 0.f);
        if (o < a.n_off)
            a.offset[(long)m * a.n_off + o] = u;
        else
            a.mask[(long)m * a.n_msk + (o - a.n_off)] = 1.f / (1.f + __expf(-u));
    }
}

}  // namespace

cudaError_t launch_offset_branch(const void* x, bool x_bf16, int N, int H, int W, int C,
                                 const float* dw_w, const float* dw_scale, const float* dw_shift,
                                 const float* pw_w, const float* pw_b, int K, int G, bool with_mask,
                                 int s_h, int s_w, int p_h, int p_w, int d_h, int d_w, int Ho, int Wo,
                                 float* offset, float* mask, cudaStream_t stream) {
    BranchArgs a;
    a.x = x; a.dw_w = dw_w; a.dw_scale = dw_scale; a.dw_shift = dw_shift;
    a.pw_w = pw_w; a.pw_b = pw_b; a.offset = offset; a.mask = mask;
    a.N = N; a.H = H; a.W = W; a.C = C; a.Ho = Ho; a.Wo = Wo; a.M = N * Ho * Wo;
    a.sh = s_h; a.sw = s_w; a.ph = p_h; a.pw = p_w; a.dh = d_h; a.dw = d_w;
    a.n_off = 2 * G * K * K;
    a.n_msk = with_mask ? G * K * K : 0;
    a.OC = a.n_off + a.n_msk;
    int dev = 0, max_smem = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&max_smem, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
    auto smem_for = [&](int pix) {
        return sizeof(float) * ((size_t)pix * (C + 1) + (size_t)a.OC * (CCH + 1));
    };
    const int n_blocks32 = (a.M + 31) / 32, n_blocks8 = (a.M + 7) / 8;
    cudaError_t e;
    if (a.OC * 32 <= THREADS * MAXO && smem_for(32) <= (size_t)max_smem) {
        auto kern = x_bf16 ? offset_branch_kernel<true, 32> : offset_branch_kernel<false, 32>;
        e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem_for(32));
        if (e != cudaSuccess) return e;
        kern<<<n_blocks32, THREADS, smem_for(32), stream>>>(a);
    } else if (a.OC * 8 <= THREADS * MAXO && smem_for(8) <= (size_t)max_smem) {
        auto kern = x_bf16 ? offset_branch_kernel<true, 8> : offset_branch_kernel<false, 8>;
        e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem_for(8));
        if (e != cudaSuccess) return e;
        kern<<<n_blocks8, THREADS, smem_for(8), stream>>>(a);
    } else {
        return cudaErrorInvalidValue;   // api.cu maps this to DEFCON_ERR_LIMIT
    }
    return cudaGetLastError();
}

}  // namespace defcon
