// offset_branch_fused.cu -- the lightweight offset branch as ONE
// kernel, t never leaves the SM:
//   t[c] = ReLU(scale[c] * sum_{3x3} W1[c] * x + shift[c])      depthwise 3x3 + folded BN
//   u[o] = b2[o] + sum_c W2[o][c] * t[c]                        1x1 projection
//   offset = u[0 : 2GK^2] ((dy, dx) pairs, R4),  mask = sigmoid(u[2GK^2 :]) (R6, R11)
//
// CTA = one output row (n, ho): all Wo pixels, all C channels, walked in chunks of 32
// channels.  8 producer warps + 1 MMA warp:
//   staging   per chunk ONE 4-D TMA box brings the 2*dil+1 input rows the row needs (from
//             y = ho*s - pad) x the Wc columns it touches (from x = -pad) into smem; the TMA
//             unit zero-fills everything outside the image, so the conv's zero padding costs
//             nothing.  Double-buffered: chunk k+2 is requested as soon as chunk k is read.
//   dw        thread = (16-byte channel vector, run of R adjacent output pixels); dw weights
//             transposed once per CTA into smem [9][C] (one 32-byte read per tap and vector);
//             with stride 1 / dilation 1 each staged column is read once
//             per run (R+2 columns for R outputs instead of 9R taps); packed FFMA2; BN + ReLU.
//   1x1       t is written straight into the K-major SWIZZLE_128B operand layout as two tf32
//             planes, hi = t with the low 13 mantissa bits cleared and lo = t - hi (both exact),
//             W2's chunk likewise; one thread issues tcgen05.mma kind::tf32 three times per
//             8-channel k-step (lo*hi + hi*lo + hi*hi: the 3xTF32 scheme, fp32-level accuracy),
//             M = 128 (rows = pixels), N = OC rounded to 16, accumulating in TMEM.
//   epilogue  warps 0-3 (TMEM lane quarters) + b2, sigmoid on the mask channels, store.
// Measured on B200: legacy mma.sync TF32 runs at roughly FFMA rate on sm_100a, so the 1x1 goes
// to tcgen05 (the two-launch path in offset_branch.cu keeps the mma.sync version).
// bf16 x is widened exactly; every sum is fp32; fixed summation order (deterministic).
#include <algorithm>

#include "common.cuh"
#include "kernels.h"

namespace defcon {
namespace {

constexpr int RT_NPROD = 8;                       // producer warps
constexpr int RT_THREADS = (RT_NPROD + 1) * 32;   // + MMA warp
constexpr int RT_KC = 32;                         // channels per chunk = one 128-byte tf32 row
constexpr uint32_t TF32_HI = 0xFFFFE000u;

struct RtArgs {
    const float* dw_w;      // [C][9]
    const float* dw_scale;
    const float* dw_shift;
    const float* pw_w;      // [OC][C]
    const float* pw_b;      // [OC] or null
    float* offset;
    float* mask;
    int H, W, C, Ho, Wo;
    int sh, sw, ph, pw, dh, dw;
    int n_off, n_msk, OC, OCN;
    int Wc, BR;             // TMA box: staged columns (input x = col - pw) and rows
    int xs_bytes;           // one x staging buffer (box + read slack), 1024-byte multiple
    int MR;                 // A rows allocated per plane (64 or 128; the MMA always reads 128)
    int ab_bytes;           // one operand stage: A hi, A lo, B hi, B lo
};

struct RtPlan {
    int R, Wc, BR, xs_bytes, MR, OCN, ab_bytes;
    size_t smem;
};

__host__ __device__ constexpr int rt_align1k(int b) { return (b + 1023) & ~1023; }

bool rt_plan(int C, int OC, int Wo, int sw, int dw, int dh, int ES, RtPlan* p) {
    if (Wo > 128 || C % 8 != 0) return false;
    p->Wc = (Wo - 1) * sw + 2 * dw + 1;
    p->BR = 2 * dh + 1;
    if (p->Wc > 256 || p->BR > 256) return false;        // TMA box limits
    const int cbb = RT_KC * ES;                          // staged bytes per pixel per chunk
    const int nvc = cbb / 16, nr = RT_NPROD * 32 / nvc;
    p->R = (Wo + nr - 1) / nr;
    if (p->R > 4) return false;
    // reads of runs past Wo may reach (R + 2) * sw + 2 * dw columns beyond the box: slack
    p->xs_bytes = rt_align1k((p->BR * p->Wc + (p->R + 2) * sw + 2 * dw) * cbb);
    p->MR = Wo <= 64 ? 64 : 128;
    p->OCN = std::max(16, (OC + 15) & ~15);
    if (p->OCN > 256) return false;
    p->ab_bytes = 2 * p->MR * 128 + 2 * p->OCN * 128;
    // 1 KB alignment + x buffers + operand stages + 8 KB slack (a 64-row plane is read as 128
    // rows by the M = 128 descriptor) + dw weights / BN [11][C] + barriers
    p->smem = 1024 + 2ull * p->xs_bytes + 2ull * p->ab_bytes + (p->MR == 64 ? 8192 : 0) + 11ull * C * 4 + 128;
    return p->smem <= 227 * 1024;
}

// 16 staged bytes -> fp32 pairs (bf16: 8 channels = 4 pairs; fp32: 4 channels = 2 pairs)
template <bool BF16>
__device__ __forceinline__ void unpack16(const uint4& u, uint64_t (&v)[BF16 ? 4 : 2]) {
    if constexpr (BF16) {
        v[0] = bf16x2_to_f32x2(u.x); v[1] = bf16x2_to_f32x2(u.y);
        v[2] = bf16x2_to_f32x2(u.z); v[3] = bf16x2_to_f32x2(u.w);
    } else {
        v[0] = f32x2_pack(__uint_as_float(u.x), __uint_as_float(u.y));
        v[1] = f32x2_pack(__uint_as_float(u.z), __uint_as_float(u.w));
    }
}

// 4 fp32 -> (hi, lo) tf32 planes at the same swizzled offset of two planes
__device__ __forceinline__ void store_split4(uint32_t hi_addr, uint32_t lo_addr, float a, float b, float c,
                                             float d) {
    const uint32_t h0 = __float_as_uint(a) & TF32_HI, h1 = __float_as_uint(b) & TF32_HI;
    const uint32_t h2 = __float_as_uint(c) & TF32_HI, h3 = __float_as_uint(d) & TF32_HI;
    st_shared_v4(hi_addr, h0, h1, h2, h3);
    st_shared_v4(lo_addr, __float_as_uint(a - __uint_as_float(h0)), __float_as_uint(b - __uint_as_float(h1)),
                 __float_as_uint(c - __uint_as_float(h2)), __float_as_uint(d - __uint_as_float(h3)));
}

template <bool BF16, bool S1, int R>
__global__ void __maxnreg__(112)
    offset_branch_row_tc_kernel(const __grid_constant__ CUtensorMap xmap, const RtArgs a) {
    constexpr int ES = BF16 ? 2 : 4;
    constexpr int VC = 16 / ES;                  // channels per 16-byte vector
    constexpr int VP = VC / 2;                   // fp32 pairs per vector
    constexpr int CBB = RT_KC * ES;              // staged bytes per pixel
    constexpr int NVC = CBB / 16;                // vectors per pixel per chunk
    extern __shared__ __align__(1024) uint8_t rt_raw[];
    uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(rt_raw) + 1023) & ~uintptr_t(1023));
    uint8_t* xs = smem;                                              // [2][BR][Wc][CBB] + slack
    uint8_t* ab = smem + 2 * a.xs_bytes;                             // [2][A hi | A lo | B hi | B lo]
    float* wdw = reinterpret_cast<float*>(ab + 2 * a.ab_bytes + (a.MR == 64 ? 8192 : 0));   // [11][C]
    uint64_t* bars = reinterpret_cast<uint64_t*>(wdw + 11 * a.C);
    uint64_t* x_full = bars;          // [2] TMA -> producers
    uint64_t* full = bars + 2;        // [2] producers -> MMA
    uint64_t* empty = bars + 4;       // [2] MMA -> producers
    uint64_t* tmem_full = bars + 6;   // MMA -> epilogue
    uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 7);

    const int tid = threadIdx.x;
    const int warp = tid >> 5, lane = tid & 31;
    const int n = blockIdx.x / a.Ho, ho = blockIdx.x - n * a.Ho;
    const int C = a.C;
    const int nchunks = (C + RT_KC - 1) / RT_KC;
    const uint32_t box_bytes = (uint32_t)(a.BR * a.Wc * CBB);
    const int tcols = a.OCN <= 32 ? 32 : a.OCN <= 64 ? 64 : a.OCN <= 128 ? 128 : 256;

    if (tid == 0) {
        for (int s = 0; s < 2; ++s) {
            mbar_init(&x_full[s], 1);
            mbar_init(&full[s], RT_NPROD);
            mbar_init(&empty[s], 1);
        }
        mbar_init(tmem_full, 1);
        fence_barrier_init();
        tma_prefetch_desc(&xmap);
    }
    if (warp == RT_NPROD) {
        switch (tcols) {
            case 32: tmem_alloc<32>(tmem_slot); break;
            case 64: tmem_alloc<64>(tmem_slot); break;
            case 128: tmem_alloc<128>(tmem_slot); break;
            default: tmem_alloc<256>(tmem_slot); break;
        }
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = *tmem_slot;
    griddep_wait();                              // PDL: x from the previous kernel is visible

    auto stage_x = [&](int ch) {                 // one thread: the whole (rows x cols x chunk) box
        const int b = ch & 1;
        mbar_arrive_expect_tx(&x_full[b], box_bytes);
        tma_load_4d(xs + b * a.xs_bytes, &xmap, &x_full[b], ch * RT_KC, -a.pw, ho * a.sh - a.ph, n);
    };

    if (warp < RT_NPROD) {
        // ======================= producers: dw + BN + ReLU -> tf32 hi/lo operand planes
        if (tid == 0) {
            stage_x(0);
            if (nchunks > 1) stage_x(1);
        }
        // dw weights [C][9] -> [9][C] plus scale / shift rows, so a vector's 8 weights of a tap
        // are one contiguous 32-byte smem read
        for (int c = tid; c < C; c += RT_NPROD * 32) {
            float w9[9];
#pragma unroll
            for (int k = 0; k < 9; ++k) w9[k] = __ldg(a.dw_w + (size_t)c * 9 + k);
            const float s0 = __ldg(a.dw_scale + c), s1 = __ldg(a.dw_shift + c);
#pragma unroll
            for (int k = 0; k < 9; ++k) wdw[k * C + c] = w9[k];
            wdw[9 * C + c] = s0;
            wdw[10 * C + c] = s1;
        }
        named_bar_sync(1, RT_NPROD * 32);
        const int v = tid % NVC, run = tid / NVC;
        const int wo0 = run * R;
        const bool active = wo0 < a.Wo;
        const int rowp = a.Wc * CBB;              // staged row pitch
        const int tap0 = wo0 * a.sw * CBB + v * 16;
        const uint32_t ab0 = smem_u32(ab);
#pragma unroll 1
        for (int ch = 0; ch < nchunks; ++ch) {
            const int s = ch & 1;
            const uint32_t par = (uint32_t)(ch >> 1) & 1u;
            const int c = ch * RT_KC + v * VC;    // first channel of this thread's vector
            const bool work = active && c < C;
            float r[R][VC];
            // W2 chunk (rows o < OCN, zero beyond OC / C): one 16-byte piece per thread-iteration
            float4 w2v[2];
#pragma unroll
            for (int i = 0; i < 2; ++i) {
                const int e = tid + i * RT_NPROD * 32;
                const int o = e >> 3, cc = ch * RT_KC + (e & 7) * 4;
                w2v[i] = make_float4(0.f, 0.f, 0.f, 0.f);
                if (e < a.OCN * 8 && o < a.OC && cc < C)
                    w2v[i] = __ldg(reinterpret_cast<const float4*>(a.pw_w + (size_t)o * C + cc));
            }
            mbar_wait(&x_full[s], par);
            if (work) {
                uint64_t acc[R][VP];
#pragma unroll
                for (int u = 0; u < R; ++u)
#pragma unroll
                    for (int p = 0; p < VP; ++p) acc[u][p] = 0ull;
                const uint8_t* xb = xs + s * a.xs_bytes + tap0;
                auto wtap = [&](int k, uint64_t (&w)[VP]) {     // tap k of the vector, as pairs
#pragma unroll
                    for (int q = 0; q < VC / 4; ++q) {
                        const float4 f = *reinterpret_cast<const float4*>(wdw + k * C + c + 4 * q);
                        w[2 * q] = f32x2_pack(f.x, f.y);
                        w[2 * q + 1] = f32x2_pack(f.z, f.w);
                    }
                };
                if constexpr (S1) {
                    // staged column wo0 + cc feeds output u through tap column j = cc - u
#pragma unroll
                    for (int i = 0; i < 3; ++i) {
                        uint64_t wk[3][VP];
#pragma unroll
                        for (int j = 0; j < 3; ++j) wtap(i * 3 + j, wk[j]);
                        const uint8_t* rp = xb + i * a.dh * rowp;
#pragma unroll
                        for (int cc = 0; cc < R + 2; ++cc) {
                            const uint4 raw = *reinterpret_cast<const uint4*>(rp + cc * CBB);
                            uint64_t xv[VP];
                            unpack16<BF16>(raw, xv);
#pragma unroll
                            for (int u = 0; u < R; ++u) {
                                const int j = cc - u;
                                if (j < 0 || j > 2) continue;
#pragma unroll
                                for (int p = 0; p < VP; ++p) acc[u][p] = f32x2_fma(wk[j][p], xv[p], acc[u][p]);
                            }
                        }
                    }
                } else {
#pragma unroll
                    for (int k = 0; k < 9; ++k) {
                        uint64_t wk[VP];
                        wtap(k, wk);
#pragma unroll
                        for (int u = 0; u < R; ++u) {
                            const int off = (k / 3) * a.dh * rowp + (u * a.sw + (k % 3) * a.dw) * CBB;
                            const uint4 raw = *reinterpret_cast<const uint4*>(xb + off);
                            uint64_t xv[VP];
                            unpack16<BF16>(raw, xv);
#pragma unroll
                            for (int p = 0; p < VP; ++p) acc[u][p] = f32x2_fma(wk[p], xv[p], acc[u][p]);
                        }
                    }
                }
                float sc[VC], sf[VC];
#pragma unroll
                for (int q = 0; q < VC / 4; ++q) {
                    const float4 s4 = *reinterpret_cast<const float4*>(wdw + 9 * C + c + 4 * q);
                    const float4 f4 = *reinterpret_cast<const float4*>(wdw + 10 * C + c + 4 * q);
                    sc[4 * q] = s4.x; sc[4 * q + 1] = s4.y; sc[4 * q + 2] = s4.z; sc[4 * q + 3] = s4.w;
                    sf[4 * q] = f4.x; sf[4 * q + 1] = f4.y; sf[4 * q + 2] = f4.z; sf[4 * q + 3] = f4.w;
                }
#pragma unroll
                for (int u = 0; u < R; ++u)
#pragma unroll
                    for (int p = 0; p < VP; ++p) {
                        r[u][2 * p] = fmaxf(fmaf(sc[2 * p], __uint_as_float((uint32_t)acc[u][p]), sf[2 * p]), 0.f);
                        r[u][2 * p + 1] =
                            fmaxf(fmaf(sc[2 * p + 1], __uint_as_float((uint32_t)(acc[u][p] >> 32)), sf[2 * p + 1]), 0.f);
                    }
            } else {
#pragma unroll
                for (int u = 0; u < R; ++u)
#pragma unroll
                    for (int e = 0; e < VC; ++e) r[u][e] = 0.f;
            }
            named_bar_sync(1, RT_NPROD * 32);    // every producer is done reading x buffer s
            if (tid == 0 && ch + 2 < nchunks) stage_x(ch + 2);
            mbar_wait(&empty[s], par ^ 1u);      // the MMAs of chunk ch - 2 are done
            const uint32_t sAh = ab0 + s * a.ab_bytes;
            const uint32_t sAl = sAh + a.MR * 128;
            const uint32_t sBh = sAl + a.MR * 128;
            const uint32_t sBl = sBh + a.OCN * 128;
            if (active) {
#pragma unroll
                for (int u = 0; u < R; ++u) {
                    const int row = wo0 + u;
                    if (row >= a.Wo) break;
#pragma unroll
                    for (int q = 0; q < VC / 4; ++q) {   // 16-byte piece j of the 128-byte row
                        const int j = v * (VC / 4) + q;
                        const uint32_t off = row * 128 + ((j ^ (row & 7)) << 4);
                        store_split4(sAh + off, sAl + off, r[u][4 * q], r[u][4 * q + 1], r[u][4 * q + 2],
                                     r[u][4 * q + 3]);
                    }
                }
            }
#pragma unroll
            for (int i = 0; i < 2; ++i) {
                const int e = tid + i * RT_NPROD * 32;
                if (e < a.OCN * 8) {
                    const int o = e >> 3, j = e & 7;
                    const uint32_t off = o * 128 + ((j ^ (o & 7)) << 4);
                    store_split4(sBh + off, sBl + off, w2v[i].x, w2v[i].y, w2v[i].z, w2v[i].w);
                }
            }
            for (int e = tid + 2 * RT_NPROD * 32; e < a.OCN * 8; e += RT_NPROD * 32) {   // OCN > 64
                const int o = e >> 3, j = e & 7;
                const int cc = ch * RT_KC + j * 4;
                float4 wv = make_float4(0.f, 0.f, 0.f, 0.f);
                if (o < a.OC && cc < C) wv = __ldg(reinterpret_cast<const float4*>(a.pw_w + (size_t)o * C + cc));
                const uint32_t off = o * 128 + ((j ^ (o & 7)) << 4);
                store_split4(sBh + off, sBl + off, wv.x, wv.y, wv.z, wv.w);
            }
            fence_proxy_async_smem();
            __syncwarp();
            if (lane == 0) mbar_arrive(&full[s]);
        }
        // ======================= epilogue: TMEM lane = pixel of the row
        if (warp < 4) {
            mbar_wait(tmem_full, 0);
            tc_fence_after();
            const int row = warp * 32 + lane;
            const size_t m = ((size_t)n * a.Ho + ho) * a.Wo + row;
#pragma unroll 1
            for (int c0 = 0; c0 < a.OCN; c0 += 32) {
                uint32_t vv[32];
                tmem_ld_32x32b_x32(tmem + ((uint32_t)(warp * 32) << 16) + c0, vv);
                tmem_ld_wait();
                if (row < a.Wo) {
#pragma unroll
                    for (int u = 0; u < 32; ++u) {
                        const int o = c0 + u;
                        if (o >= a.OC) break;
                        const float val = __uint_as_float(vv[u]) + (a.pw_b ? __ldg(a.pw_b + o) : 0.f);
                        if (o < a.n_off)
                            a.offset[m * a.n_off + o] = val;
                        else
                            a.mask[m * a.n_msk + (o - a.n_off)] = 1.f / (1.f + __expf(-val));
                    }
                }
            }
        }
    } else if (lane == 0) {
        // ======================= MMA issuer: 3xTF32 per 8-channel k-step
        const uint32_t idesc = make_idesc(2u /*TF32*/, 128, (uint32_t)a.OCN);
        const uint32_t ab0 = smem_u32(ab);
#pragma unroll 1
        for (int ch = 0; ch < nchunks; ++ch) {
            const int s = ch & 1;
            mbar_wait(&full[s], (uint32_t)(ch >> 1) & 1u);
            tc_fence_after();
            const uint32_t sAh = ab0 + s * a.ab_bytes;
            const uint32_t sAl = sAh + a.MR * 128;
            const uint32_t sBh = sAl + a.MR * 128;
            const uint32_t sBl = sBh + a.OCN * 128;
#pragma unroll
            for (int kk = 0; kk < RT_KC / 8; ++kk) {         // K = 8 tf32 = 32 bytes per step
                const uint64_t ah = make_sw128_desc(sAh + kk * 32), al = make_sw128_desc(sAl + kk * 32);
                const uint64_t bh = make_sw128_desc(sBh + kk * 32), bl = make_sw128_desc(sBl + kk * 32);
                mma_tf32_ss(tmem, al, bh, idesc, (ch | kk) != 0 ? 1u : 0u);
                mma_tf32_ss(tmem, ah, bl, idesc, 1u);
                mma_tf32_ss(tmem, ah, bh, idesc, 1u);
            }
            mma_commit(&empty[s]);
        }
        mma_commit(tmem_full);
    }
    tc_fence_before();
    __syncthreads();
    if (warp == RT_NPROD) {
        tc_fence_after();
        switch (tcols) {
            case 32: tmem_dealloc<32>(tmem); break;
            case 64: tmem_dealloc<64>(tmem); break;
            case 128: tmem_dealloc<128>(tmem); break;
            default: tmem_dealloc<256>(tmem); break;
        }
    }
}

template <bool BF16, bool S1>
cudaError_t launch_rt(const CUtensorMap& xmap, const RtArgs& a, int grid, int R, size_t smem,
                      cudaStream_t stream) {
    void (*kern)(CUtensorMap, RtArgs) = nullptr;
    switch (R) {
        case 1: kern = offset_branch_row_tc_kernel<BF16, S1, 1>; break;
        case 2: kern = offset_branch_row_tc_kernel<BF16, S1, 2>; break;
        case 3: kern = offset_branch_row_tc_kernel<BF16, S1, 3>; break;
        default: kern = offset_branch_row_tc_kernel<BF16, S1, 4>; break;
    }
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e == cudaSuccess)
        e = cudaFuncSetAttribute(kern, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
    if (e != cudaSuccess) return e;
    return launch_pdl(kern, dim3(grid), dim3(RT_THREADS), smem, stream, xmap, a);
}

}  // namespace

bool offset_branch_fused_supported(int C, int OC, int Wo, int sw, int dw, int dh, bool x_bf16) {
    RtPlan p;
    return get_encode_tiled() != nullptr && rt_plan(C, OC, Wo, sw, dw, dh, x_bf16 ? 2 : 4, &p);
}

cudaError_t launch_offset_branch_fused(const void* x, bool x_bf16, int N, int H, int W, int C,
                                       const float* dw_w, const float* dw_scale, const float* dw_shift,
                                       const float* pw_w, const float* pw_b, int n_off, int n_msk,
                                       int s_h, int s_w, int p_h, int p_w, int d_h, int d_w, int Ho,
                                       int Wo, float* offset, float* mask, cudaStream_t stream) {
    RtPlan p;
    const int ES = x_bf16 ? 2 : 4;
    const int OC = n_off + n_msk;
    if (!rt_plan(C, OC, Wo, s_w, d_w, d_h, ES, &p)) return cudaErrorInvalidValue;
    PFN_encodeTiled encode = get_encode_tiled();
    if (!encode) return cudaErrorNotSupported;
    // x as a 4-D tensor (C, W, H, N); box = (32 channels, Wc columns, BR rows, 1 image)
    CUtensorMap xmap;
    cuuint64_t dims[4] = {(cuuint64_t)C, (cuuint64_t)W, (cuuint64_t)H, (cuuint64_t)N};
    cuuint64_t strides[3] = {(cuuint64_t)C * ES, (cuuint64_t)W * C * ES, (cuuint64_t)H * W * C * ES};
    cuuint32_t box[4] = {(cuuint32_t)RT_KC, (cuuint32_t)p.Wc, (cuuint32_t)p.BR, 1u};
    cuuint32_t estr[4] = {1, 1, 1, 1};
    CUresult cr = encode(&xmap, x_bf16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4,
                         const_cast<void*>(x), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                         CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
                         CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (cr != CUDA_SUCCESS) return cudaErrorInvalidValue;
    RtArgs a;
    a.dw_w = dw_w; a.dw_scale = dw_scale; a.dw_shift = dw_shift;
    a.pw_w = pw_w; a.pw_b = pw_b; a.offset = offset; a.mask = mask;
    a.H = H; a.W = W; a.C = C; a.Ho = Ho; a.Wo = Wo;
    a.sh = s_h; a.sw = s_w; a.ph = p_h; a.pw = p_w; a.dh = d_h; a.dw = d_w;
    a.n_off = n_off; a.n_msk = n_msk; a.OC = OC; a.OCN = p.OCN;
    a.Wc = p.Wc; a.BR = p.BR; a.xs_bytes = p.xs_bytes; a.MR = p.MR; a.ab_bytes = p.ab_bytes;
    const bool s1 = s_w == 1 && d_w == 1;
    const int grid = N * Ho;
    if (x_bf16)
        return s1 ? launch_rt<true, true>(xmap, a, grid, p.R, p.smem, stream)
                  : launch_rt<true, false>(xmap, a, grid, p.R, p.smem, stream);
    return s1 ? launch_rt<false, true>(xmap, a, grid, p.R, p.smem, stream)
              : launch_rt<false, false>(xmap, a, grid, p.R, p.smem, stream);
}

}  // namespace defcon
