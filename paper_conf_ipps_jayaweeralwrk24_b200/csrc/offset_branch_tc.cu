// offset_branch_tc.cu -- the lightweight offset branch as ONE kernel:
//   t[c] = ReLU(scale[c] * sum_{3x3} W1[c] * x + shift[c])      depthwise 3x3 + folded BN (CUDA cores)
//   u[o] = b2[o] + sum_c W2[o][c] * t[c]                        1x1 projection (tensor cores)
//   offset = u[0 : 2GK^2] ((dy, dx) pairs, R4),  mask = sigmoid(u[2GK^2 :]) (R6, R11)
//
// Persistent CTAs walk tiles of TP = 64 output pixels.  Per tile and 32-channel chunk the
// 8 producer warps compute t on the CUDA cores (fp32, packed FFMA2; thread = pixel x 8
// channels, 9 taps of 16-byte x loads) and write it straight into shared memory in the
// canonical K-major SWIZZLE_128B layout as two tf32 operands, t_hi = t with the low 13
// mantissa bits cleared and t_lo = t - t_hi (both exact in fp32); W2's chunk is split the
// same way.  One thread issues tcgen05.mma kind::tf32 (M = 128 of which rows 0..63 are the
// tile, N = OC rounded up to 16, K = 8) three times per k-step -- lo*hi + hi*lo + hi*hi, the
// 3xTF32 scheme, fp32-level accuracy -- accumulating in TMEM.  t never leaves the SM; only
// offsets and mask are written.  Warps 0-1 (TMEM lanes 0..63) run the epilogue: + b2,
// sigmoid on mask channels, store.  Fixed summation order: deterministic.
#include <algorithm>
#include <cstdlib>

#include "common.cuh"
#include "kernels.h"

namespace defcon {
namespace {

constexpr int TP = 64;                    // pixels per tile (UMMA rows 0..63)
constexpr int KC = 32;                    // channels per chunk = one 128-byte tf32 row
constexpr int NPROD = 8;                  // producer warps
constexpr int OB_THREADS = (NPROD + 1) * 32;
constexpr int OB_STAGES = 2;
constexpr uint32_t TF32_MASK = 0xFFFFE000u;

struct ObArgs {
    const void* x;
    const float* dw_w;      // [C][9]
    const float* dw_scale;
    const float* dw_shift;
    const float* pw_w;      // [OC][C]
    const float* pw_b;      // [OC] or null
    float* offset;
    float* mask;
    int N, H, W, C, Ho, Wo, M;
    int sh, sw, ph, pw, dh, dw;
    int n_off, n_msk, OC, OCN;
    int tiles, nchunk;
};

// 32 zero bytes: the load target of taps in the zero padding (branch-free tap loop)
__device__ __align__(32) const uint32_t g_ob_zero[8] = {0, 0, 0, 0, 0, 0, 0, 0};

__host__ __device__ constexpr int ob_stage_bytes(int OCN) { return 2 * TP * 128 + 2 * OCN * 128; }

__device__ __forceinline__ void split_store(uint32_t hi_addr, uint32_t lo_addr, const float (&v)[4]) {
    uint32_t h[4], l[4];
#pragma unroll
    for (int i = 0; i < 4; ++i) {
        h[i] = __float_as_uint(v[i]) & TF32_MASK;
        l[i] = __float_as_uint(v[i] - __uint_as_float(h[i]));
    }
    st_shared_v4(hi_addr, h[0], h[1], h[2], h[3]);
    st_shared_v4(lo_addr, l[0], l[1], l[2], l[3]);
}

template <bool BF16>
__global__ void __launch_bounds__(OB_THREADS, 3) offset_branch_tc_kernel(const ObArgs a) {
    extern __shared__ __align__(1024) uint8_t ob_raw[];
    uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(ob_raw) + 1023) & ~uintptr_t(1023));
    const int SB = ob_stage_bytes(a.OCN);
    uint8_t* stages = smem;
    // + 8 KB of slack: the A_lo descriptor of the last stage spans 128 rows (rows 64..127
    // are don't-care and may read past the stage)
    float* wdw = reinterpret_cast<float*>(stages + OB_STAGES * SB + 8192);   // [9][C]
    float* sc = wdw + 9 * a.C;
    float* sf = sc + a.C;
    uint64_t* bars = reinterpret_cast<uint64_t*>(sf + a.C + 4);
    uint64_t* full = bars;                    // [OB_STAGES]
    uint64_t* empty = bars + OB_STAGES;       // [OB_STAGES]
    uint64_t* tmem_full = bars + 2 * OB_STAGES;
    uint64_t* tmem_empty = tmem_full + 1;
    uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tmem_empty + 1);

    const int tid = threadIdx.x;
    const int warp = tid >> 5, lane = tid & 31;
    if (tid == 0) {
        for (int s = 0; s < OB_STAGES; ++s) {
            mbar_init(&full[s], NPROD);
            mbar_init(&empty[s], 1);
        }
        mbar_init(tmem_full, 1);
        mbar_init(tmem_empty, 2);
        fence_barrier_init();
    }
    const int tcols = a.OCN <= 32 ? 32 : a.OCN <= 64 ? 64 : a.OCN <= 128 ? 128 : 256;
    if (warp == NPROD) {
        switch (tcols) {
            case 32: tmem_alloc<32>(tmem_slot); break;
            case 64: tmem_alloc<64>(tmem_slot); break;
            case 128: tmem_alloc<128>(tmem_slot); break;
            default: tmem_alloc<256>(tmem_slot); break;
        }
    }
    griddep_wait();                           // PDL: x (and our outputs' readers) are ordered
    griddep_launch_dependents();
    // [C][9] -> [9][C]: thread = channel, its 9 weights loaded together (one round trip)
    for (int c = tid; c < a.C; c += OB_THREADS) {
        float w9[9];
#pragma unroll
        for (int k = 0; k < 9; ++k) w9[k] = __ldg(a.dw_w + (long)c * 9 + k);
        const float s0 = __ldg(a.dw_scale + c), s1 = __ldg(a.dw_shift + c);
#pragma unroll
        for (int k = 0; k < 9; ++k) wdw[k * a.C + c] = w9[k];
        sc[c] = s0;
        sf[c] = s1;
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = *tmem_slot;
    constexpr int ES = BF16 ? 2 : 4;

    if (warp < NPROD) {
        // ============ producers (+ epilogue on warps 0, 1) ============
        const int p = tid >> 2;               // pixel of the tile
        const int v = tid & 3;                // 8-channel vector of the chunk
        const uint32_t st0 = smem_u32(stages);
        int q = 0;                            // running chunk counter (stage / phase)
        int tcount = 0;
#pragma unroll 1
        for (int tile = blockIdx.x; tile < a.tiles; tile += gridDim.x, ++tcount) {
            const int m = tile * TP + p;
            const bool ok = m < a.M;
            const uint8_t* base = reinterpret_cast<const uint8_t*>(a.x);
            uint32_t valid = 0;
            if (ok) {
                const int hw = a.Ho * a.Wo;
                const int n = m / hw;
                const int rem = m - n * hw;
                const int ho = rem / a.Wo;
                const int y0 = ho * a.sh - a.ph, x0 = (rem - ho * a.Wo) * a.sw - a.pw;
#pragma unroll
                for (int k = 0; k < 9; ++k) {
                    const int yy = y0 + (k / 3) * a.dh, xx = x0 + (k % 3) * a.dw;
                    if (yy >= 0 && yy < a.H && xx >= 0 && xx < a.W) valid |= 1u << k;
                }
                // may point outside x for padded taps; dereferenced only for valid ones
                base += (((long)n * a.H + y0) * a.W + x0) * (long)a.C * ES;
            }
#pragma unroll 1
            for (int ch = 0; ch < a.nchunk; ++ch, ++q) {
                const int s = q % OB_STAGES;
                const uint32_t sA = st0 + s * SB;                     // A_hi rows 0..63
                const uint32_t sAl = sA + TP * 128;                   // A_lo rows 0..63
                const uint32_t sBh = sA + 2 * TP * 128;               // W2 chunk, hi
                const uint32_t sBl = sBh + a.OCN * 128;               // W2 chunk, lo
                // ---- depthwise 3x3 + BN + ReLU for (pixel p, channels c0..c0+7)
                const int c0 = ch * KC + v * 8;
                float r[8];
#pragma unroll
                for (int u = 0; u < 8; ++u) r[u] = 0.f;
                if (ok && c0 < a.C) {
                    // all 9 loads issued before any use: padded taps read a zero page instead
                    // of branching (a branch per tap serialises the L2 round trips)
                    uint4 xv[9], xv2[9];
#pragma unroll
                    for (int k = 0; k < 9; ++k) {
                        const long toff = ((long)(k / 3) * a.dh * a.W + (k % 3) * a.dw) * a.C;
                        const uint4* src = ((valid >> k) & 1u)
                                               ? reinterpret_cast<const uint4*>(base + (toff + c0) * ES)
                                               : reinterpret_cast<const uint4*>(g_ob_zero);
                        xv[k] = __ldg(src);
                        if (!BF16) xv2[k] = __ldg(src + 1);
                    }
                    uint64_t acc[4] = {0ull, 0ull, 0ull, 0ull};
#pragma unroll
                    for (int k = 0; k < 9; ++k) {
                        uint64_t xp[4];
                        if (BF16) {
                            xp[0] = bf16x2_to_f32x2(xv[k].x); xp[1] = bf16x2_to_f32x2(xv[k].y);
                            xp[2] = bf16x2_to_f32x2(xv[k].z); xp[3] = bf16x2_to_f32x2(xv[k].w);
                        } else {
                            xp[0] = ((uint64_t)xv[k].y << 32) | xv[k].x;
                            xp[1] = ((uint64_t)xv[k].w << 32) | xv[k].z;
                            xp[2] = ((uint64_t)xv2[k].y << 32) | xv2[k].x;
                            xp[3] = ((uint64_t)xv2[k].w << 32) | xv2[k].z;
                        }
                        const float4 w0 = *reinterpret_cast<const float4*>(wdw + k * a.C + c0);
                        const float4 w1 = *reinterpret_cast<const float4*>(wdw + k * a.C + c0 + 4);
                        acc[0] = f32x2_fma(f32x2_pack(w0.x, w0.y), xp[0], acc[0]);
                        acc[1] = f32x2_fma(f32x2_pack(w0.z, w0.w), xp[1], acc[1]);
                        acc[2] = f32x2_fma(f32x2_pack(w1.x, w1.y), xp[2], acc[2]);
                        acc[3] = f32x2_fma(f32x2_pack(w1.z, w1.w), xp[3], acc[3]);
                    }
#pragma unroll
                    for (int u = 0; u < 4; ++u) {
                        r[2 * u] = __uint_as_float((uint32_t)(acc[u] & 0xFFFFFFFFull));
                        r[2 * u + 1] = __uint_as_float((uint32_t)(acc[u] >> 32));
                    }
#pragma unroll
                    for (int u = 0; u < 8; ++u) r[u] = fmaxf(fmaf(sc[c0 + u], r[u], sf[c0 + u]), 0.f);
                }
                // W2 chunk loads (rows o < OCN, zero beyond OC / C) before the stage wait
                float4 w2v[2];
#pragma unroll
                for (int i = 0; i < 2; ++i) {
                    const int e = tid + i * NPROD * 32;
                    const int o = e >> 3, c = ch * KC + (e & 7) * 4;
                    w2v[i] = make_float4(0.f, 0.f, 0.f, 0.f);
                    if (e < a.OCN * 8 && o < a.OC && c < a.C)
                        w2v[i] = __ldg(reinterpret_cast<const float4*>(a.pw_w + (long)o * a.C + c));
                }
                mbar_wait(&empty[s], ((uint32_t)(q / OB_STAGES) & 1u) ^ 1u);   // stage free
                {   // row p, 16-byte chunks 2v and 2v+1 of the 128-byte row, SW128
                    const uint32_t rowo = p * 128;
                    const uint32_t j0 = ((2 * v) ^ (p & 7)) << 4, j1 = ((2 * v + 1) ^ (p & 7)) << 4;
                    const float lo4[4] = {r[0], r[1], r[2], r[3]};
                    const float hi4[4] = {r[4], r[5], r[6], r[7]};
                    split_store(sA + rowo + j0, sAl + rowo + j0, lo4);
                    split_store(sA + rowo + j1, sAl + rowo + j1, hi4);
                }
                // ---- W2 chunk: 32 channels of rows o < OCN, split hi / lo, SW128
#pragma unroll
                for (int i = 0; i < 2; ++i) {
                    const int e = tid + i * NPROD * 32;
                    if (e < a.OCN * 8) {
                        const int o = e >> 3, j = e & 7;
                        const float w4[4] = {w2v[i].x, w2v[i].y, w2v[i].z, w2v[i].w};
                        const uint32_t off = o * 128 + ((j ^ (o & 7)) << 4);
                        split_store(sBh + off, sBl + off, w4);
                    }
                }
                for (int e = tid + 2 * NPROD * 32; e < a.OCN * 8; e += NPROD * 32) {   // OCN > 64
                    const int o = e >> 3, j = e & 7;
                    const int c = ch * KC + j * 4;
                    float w4[4] = {0.f, 0.f, 0.f, 0.f};
                    if (o < a.OC && c < a.C) {
                        const float4 wv = __ldg(reinterpret_cast<const float4*>(a.pw_w + (long)o * a.C + c));
                        w4[0] = wv.x; w4[1] = wv.y; w4[2] = wv.z; w4[3] = wv.w;
                    }
                    const uint32_t off = o * 128 + ((j ^ (o & 7)) << 4);
                    split_store(sBh + off, sBl + off, w4);
                }
                fence_proxy_async_smem();
                __syncwarp();
                if (lane == 0) mbar_arrive(&full[s]);
            }
            // ---- epilogue: TMEM lanes 0..63 = the tile's pixels
            if (warp < 2) {
                mbar_wait(tmem_full, (uint32_t)tcount & 1u);
                tc_fence_after();
                const int row = warp * 32 + lane;
                const int mm = tile * TP + row;
#pragma unroll 1
                for (int c = 0; c < a.OCN; c += 32) {
                    uint32_t vv[32];
                    tmem_ld_32x32b_x32(tmem + ((uint32_t)(warp * 32) << 16) + c, vv);
                    tmem_ld_wait();
                    if (mm < a.M) {
#pragma unroll
                        for (int u = 0; u < 32; ++u) {
                            const int o = c + u;
                            if (o >= a.OC) break;
                            const float val = __uint_as_float(vv[u]) + (a.pw_b ? __ldg(a.pw_b + o) : 0.f);
                            if (o < a.n_off)
                                a.offset[(long)mm * a.n_off + o] = val;
                            else
                                a.mask[(long)mm * a.n_msk + (o - a.n_off)] = 1.f / (1.f + __expf(-val));
                        }
                    }
                }
                tc_fence_before();
                __syncwarp();
                if (lane == 0) mbar_arrive(tmem_empty);
            }
        }
    } else if (lane == 0) {
        // ============ MMA issuer: 3xTF32 per k-step ============
        const uint32_t idesc = make_idesc(2u /*TF32*/, 128, (uint32_t)a.OCN);
        const uint32_t st0 = smem_u32(stages);
        int q = 0, tcount = 0;
#pragma unroll 1
        for (int tile = blockIdx.x; tile < a.tiles; tile += gridDim.x, ++tcount) {
            mbar_wait(tmem_empty, ((uint32_t)tcount & 1u) ^ 1u);
            tc_fence_after();
#pragma unroll 1
            for (int ch = 0; ch < a.nchunk; ++ch, ++q) {
                const int s = q % OB_STAGES;
                mbar_wait(&full[s], (uint32_t)(q / OB_STAGES) & 1u);
                tc_fence_after();
                const uint32_t sA = st0 + s * SB;
                const uint32_t sAl = sA + TP * 128;
                const uint32_t sBh = sA + 2 * TP * 128;
                const uint32_t sBl = sBh + a.OCN * 128;
#pragma unroll
                for (int kk = 0; kk < KC / 8; ++kk) {          // K = 8 tf32 = 32 bytes per step
                    const uint64_t ah = make_sw128_desc(sA + kk * 32), al = make_sw128_desc(sAl + kk * 32);
                    const uint64_t bh = make_sw128_desc(sBh + kk * 32), bl = make_sw128_desc(sBl + kk * 32);
                    mma_tf32_ss(tmem, al, bh, idesc, (ch | kk) != 0 ? 1u : 0u);
                    mma_tf32_ss(tmem, ah, bl, idesc, 1u);
                    mma_tf32_ss(tmem, ah, bh, idesc, 1u);
                }
                mma_commit(&empty[s]);
            }
            mma_commit(tmem_full);
        }
    }
    tc_fence_before();
    __syncthreads();
    if (warp == NPROD) {
        tc_fence_after();
        switch (tcols) {
            case 32: tmem_dealloc<32>(tmem); break;
            case 64: tmem_dealloc<64>(tmem); break;
            case 128: tmem_dealloc<128>(tmem); break;
            default: tmem_dealloc<256>(tmem); break;
        }
    }
}

size_t ob_smem_bytes(int C, int OCN) {
    return 1024 + (size_t)OB_STAGES * ob_stage_bytes(OCN) + 8192 + (size_t)(11 * C + 4) * 4 +
           (2 * OB_STAGES + 2) * 8 + 16;
}

}  // namespace

bool offset_branch_tc_supported(int C, int OC) {
    const int OCN = (OC + 15) & ~15;
    return C % 8 == 0 && OCN <= 256 && ob_smem_bytes(C, OCN) <= 227 * 1024;
}

cudaError_t launch_offset_branch_tc(const void* x, bool x_bf16, int N, int H, int W, int C,
                                    const float* dw_w, const float* dw_scale, const float* dw_shift,
                                    const float* pw_w, const float* pw_b, int n_off, int n_msk,
                                    int s_h, int s_w, int p_h, int p_w, int d_h, int d_w, int Ho, int Wo,
                                    float* offset, float* mask, cudaStream_t stream) {
    ObArgs a;
    a.x = x; a.dw_w = dw_w; a.dw_scale = dw_scale; a.dw_shift = dw_shift;
    a.pw_w = pw_w; a.pw_b = pw_b; a.offset = offset; a.mask = mask;
    a.N = N; a.H = H; a.W = W; a.C = C; a.Ho = Ho; a.Wo = Wo; a.M = N * Ho * Wo;
    a.sh = s_h; a.sw = s_w; a.ph = p_h; a.pw = p_w; a.dh = d_h; a.dw = d_w;
    a.n_off = n_off; a.n_msk = n_msk; a.OC = n_off + n_msk;
    a.OCN = (a.OC + 15) & ~15;
    if (a.OCN < 16) a.OCN = 16;
    a.tiles = (a.M + TP - 1) / TP;
    a.nchunk = (C + KC - 1) / KC;
    const size_t smem = ob_smem_bytes(C, a.OCN);
    auto kern = x_bf16 ? offset_branch_tc_kernel<true> : offset_branch_tc_kernel<false>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    int dev = 0, nsm = 148, smem_sm = 228 * 1024;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    cudaDeviceGetAttribute(&smem_sm, cudaDevAttrMaxSharedMemoryPerMultiprocessor, dev);
    cudaFuncAttributes fa;
    e = cudaFuncGetAttributes(&fa, kern);
    if (e != cudaSuccess) return e;
    // resident CTAs per SM from shared memory (+1 KB reserved each) and registers
    int per_sm = (int)(smem_sm / (smem + 1024));
    per_sm = std::min(per_sm, 65536 / std::max(1, fa.numRegs * OB_THREADS));
    per_sm = std::max(1, std::min(per_sm, 3));
    const int grid = std::min(a.tiles, per_sm * nsm);
    return launch_pdl(kern, dim3(grid), dim3(OB_THREADS), smem, stream, a);
}

}  // namespace defcon
