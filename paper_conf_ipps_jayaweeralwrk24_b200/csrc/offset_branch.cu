// offset_branch.cu -- the paper's lightweight offset branch,
// fused into one NHWC pass:
//   t[c] = ReLU(scale[c] * sum_{3x3} W1[c] * x + shift[c])    depthwise 3x3 + folded BN
//   u[o] = b2[o] + sum_c W2[o][c] * t[c]                      1x1 to OC = G*K*K*(2|3)
//   offset = u[0 : 2GK^2] ([G][K*K][2] = (dy, dx), R4),  mask = sigmoid(u[2GK^2 :]) (R6)
// One block owns PIX = 64 consecutive output pixels and walks the channels in chunks
// of 64: phase 1 computes the chunk of t (16-byte vector loads of x, 8 channels per
// task) into shared memory, phase 2 accumulates the 1x1 projection for the chunk with
// a 4-pixel x OCT-output register tile per thread.  t never leaves the SM; x is read
// once from HBM (the 3x3 halo re-reads hit L1/L2).  fp32 arithmetic throughout.
#include "common.cuh"
#include "kernels.h"

namespace defcon {
namespace {

constexpr int THREADS = 256;
constexpr int PIX = 64;        // output pixels per block
constexpr int CCH = 64;        // channels per chunk
constexpr int TS = PIX + 4;    // t_s row stride (floats), keeps float4 alignment

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
__device__ __forceinline__ void load8(const void* x, long idx, float (&v)[8]) {
    if (BF16) {
        const uint4 u = __ldg(reinterpret_cast<const uint4*>(static_cast<const __nv_bfloat16*>(x) + idx));
        v[0] = bf16lo_to_f32(u.x); v[1] = bf16hi_to_f32(u.x);
        v[2] = bf16lo_to_f32(u.y); v[3] = bf16hi_to_f32(u.y);
        v[4] = bf16lo_to_f32(u.z); v[5] = bf16hi_to_f32(u.z);
        v[6] = bf16lo_to_f32(u.w); v[7] = bf16hi_to_f32(u.w);
    } else {
        const float4* p = reinterpret_cast<const float4*>(static_cast<const float*>(x) + idx);
        const float4 a = __ldg(p), b = __ldg(p + 1);
        v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w;
        v[4] = b.x; v[5] = b.y; v[6] = b.z; v[7] = b.w;
    }
}

// OCT = outputs per thread along OC; 16 threads span OCP = 16 * OCT >= OC outputs.
template <bool BF16, int OCT>
__global__ void __launch_bounds__(THREADS) offset_branch_kernel(const BranchArgs a) {
    constexpr int OCP = 16 * OCT;
    extern __shared__ __align__(16) float smem_f[];
    float* t_s = smem_f;                                   // [CCH][TS]   t, pixel-minor
    float* w_s = t_s + CCH * TS;                           // [CCH][OCP]  W2^T, zero padded
    float* dw_s = w_s + CCH * OCP;                         // [9][CCH]
    float* sc_s = dw_s + 9 * CCH;                          // [CCH]
    float* sf_s = sc_s + CCH;                              // [CCH]
    int4* pix_s = reinterpret_cast<int4*>(sf_s + CCH);     // [PIX] (n, ho, wo, valid)

    const int tid = threadIdx.x;
    const int m0 = blockIdx.x * PIX;
    if (tid < PIX) {
        const int m = m0 + tid;
        int4 q = make_int4(0, 0, 0, 0);
        if (m < a.M) {
            const int hw = a.Ho * a.Wo;
            q.x = m / hw;
            const int rem = m - q.x * hw;
            q.y = rem / a.Wo;
            q.z = rem - q.y * a.Wo;
            q.w = 1;
        }
        pix_s[tid] = q;
    }
    const int tp = tid >> 4;     // pixel group: pixels 4tp .. 4tp+3
    const int to = tid & 15;     // output group: outputs to*OCT .. to*OCT+OCT-1
    float acc[4][OCT];
#pragma unroll
    for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < OCT; ++j) acc[i][j] = 0.f;

    for (int c0 = 0; c0 < a.C; c0 += CCH) {
        const int cn = min(CCH, a.C - c0);     // multiple of 8
        __syncthreads();                        // previous chunk fully consumed
        for (int e = tid; e < cn * 9; e += THREADS) {
            const int c = e / 9, k = e - (e / 9) * 9;
            dw_s[k * CCH + c] = __ldg(a.dw_w + (long)(c0 + c) * 9 + k);
        }
        for (int e = tid; e < cn; e += THREADS) {
            sc_s[e] = __ldg(a.dw_scale + c0 + e);
            sf_s[e] = __ldg(a.dw_shift + c0 + e);
        }
        for (int e = tid; e < CCH * OCP; e += THREADS) {
            const int c = e / OCP, o = e - (e / OCP) * OCP;
            w_s[e] = (c < cn && o < a.OC) ? __ldg(a.pw_w + (long)o * a.C + c0 + c) : 0.f;
        }
        __syncthreads();

        // ---- phase 1: t[c][p] for this chunk, 8 channels per task
        const int nvec = cn >> 3;
        for (int task = tid; task < PIX * nvec; task += THREADS) {
            const int p = task & (PIX - 1);
            const int v = task >> 6;
            const int4 q = pix_s[p];
            float s[8];
#pragma unroll
            for (int u = 0; u < 8; ++u) s[u] = 0.f;
            if (q.w) {
#pragma unroll
                for (int i = 0; i < 3; ++i) {
                    const int yy = q.y * a.sh - a.ph + i * a.dh;
                    if (yy < 0 || yy >= a.H) continue;
#pragma unroll
                    for (int j = 0; j < 3; ++j) {
                        const int xx = q.z * a.sw - a.pw + j * a.dw;
                        if (xx < 0 || xx >= a.W) continue;
                        float xv[8];
                        load8<BF16>(a.x, ((long)(q.x * a.H + yy) * a.W + xx) * a.C + c0 + v * 8, xv);
                        const float4 w0 = *reinterpret_cast<const float4*>(dw_s + (i * 3 + j) * CCH + v * 8);
                        const float4 w1 = *reinterpret_cast<const float4*>(dw_s + (i * 3 + j) * CCH + v * 8 + 4);
                        s[0] = fmaf(w0.x, xv[0], s[0]); s[1] = fmaf(w0.y, xv[1], s[1]);
                        s[2] = fmaf(w0.z, xv[2], s[2]); s[3] = fmaf(w0.w, xv[3], s[3]);
                        s[4] = fmaf(w1.x, xv[4], s[4]); s[5] = fmaf(w1.y, xv[5], s[5]);
                        s[6] = fmaf(w1.z, xv[6], s[6]); s[7] = fmaf(w1.w, xv[7], s[7]);
                    }
                }
            }
#pragma unroll
            for (int u = 0; u < 8; ++u) {
                const int c = v * 8 + u;
                t_s[c * TS + p] = q.w ? fmaxf(fmaf(sc_s[c], s[u], sf_s[c]), 0.f) : 0.f;
            }
        }
        __syncthreads();

        // ---- phase 2: acc[p][o] += sum_c t[c][p] * W2[o][c]
#pragma unroll 4
        for (int c = 0; c < cn; ++c) {
            const float4 tv = *reinterpret_cast<const float4*>(t_s + c * TS + 4 * tp);
            float wv[OCT];
            if constexpr (OCT % 4 == 0) {
#pragma unroll
                for (int j = 0; j < OCT; j += 4) {
                    const float4 w4 = *reinterpret_cast<const float4*>(w_s + c * OCP + to * OCT + j);
                    wv[j] = w4.x; wv[j + 1] = w4.y; wv[j + 2] = w4.z; wv[j + 3] = w4.w;
                }
            } else {
#pragma unroll
                for (int j = 0; j < OCT; j += 2) {
                    const float2 w2 = *reinterpret_cast<const float2*>(w_s + c * OCP + to * OCT + j);
                    wv[j] = w2.x; wv[j + 1] = w2.y;
                }
            }
#pragma unroll
            for (int j = 0; j < OCT; ++j) {
                acc[0][j] = fmaf(tv.x, wv[j], acc[0][j]);
                acc[1][j] = fmaf(tv.y, wv[j], acc[1][j]);
                acc[2][j] = fmaf(tv.z, wv[j], acc[2][j]);
                acc[3][j] = fmaf(tv.w, wv[j], acc[3][j]);
            }
        }
    }

    // ---- outputs
#pragma unroll
    for (int i = 0; i < 4; ++i) {
        const int m = m0 + 4 * tp + i;
        if (m >= a.M) continue;
#pragma unroll
        for (int j = 0; j < OCT; ++j) {
            const int o = to * OCT + j;
            if (o >= a.OC) continue;
            const float u = acc[i][j] + (a.pw_b ? __ldg(a.pw_b + o) : 0.f);
            if (o < a.n_off)
                a.offset[(long)m * a.n_off + o] = u;
            else
                a.mask[(long)m * a.n_msk + (o - a.n_off)] = 1.f / (1.f + __expf(-u));
        }
    }
}

template <int OCT>
cudaError_t launch_oct(const BranchArgs& a, bool bf16, cudaStream_t stream) {
    const int blocks = (a.M + PIX - 1) / PIX;
    const size_t smem = sizeof(float) * ((size_t)CCH * TS + (size_t)CCH * 16 * OCT + 11 * CCH) +
                        sizeof(int4) * PIX;
    auto kern = bf16 ? offset_branch_kernel<true, OCT> : offset_branch_kernel<false, OCT>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    kern<<<blocks, THREADS, smem, stream>>>(a);
    return cudaGetLastError();
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
    if (a.OC <= 32) return launch_oct<2>(a, x_bf16, stream);
    if (a.OC <= 64) return launch_oct<4>(a, x_bf16, stream);
    if (a.OC <= 128) return launch_oct<8>(a, x_bf16, stream);
    if (a.OC <= 256) return launch_oct<16>(a, x_bf16, stream);
    return cudaErrorInvalidValue;   // api.cu maps this to DEFCON_ERR_LIMIT
}

}  // namespace defcon
