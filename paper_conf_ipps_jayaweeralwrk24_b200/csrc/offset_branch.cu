// offset_branch.cu -- the paper's lightweight offset branch:
//   t[c] = ReLU(scale[c] * sum_{3x3} W1[c] * x + shift[c])    depthwise 3x3 + folded BN
//   u[o] = b2[o] + sum_c W2[o][c] * t[c]                      1x1 to OC = G*K*K*(2|3)
//   offset = u[0 : 2GK^2] ([G][K*K][2] = (dy, dx), R4),  mask = sigmoid(u[2GK^2 :]) (R6)
//
// Two launches, both sized for latency hiding rather than fused into one block-local
// pass (which left one 170-register block per SM and three serialized waves):
//   dw_bn_relu_kernel  thread = (8 channels, 4 pixels), taps outer so each tap's weights
//                      are read once from shared memory for 4 pixels; 16-byte loads of x
//                      (lanes along channels, coalesced), fp32 FMA, BN + ReLU, t ->
//                      workspace ([M][C], L2-resident between the two launches): one fp32
//                      plane, or tf32 hi / lo planes (and W2 split likewise) for pw_tc_kernel.
//   pw_tc_kernel       the 1x1 projection [M x C] x [C x OC] on tcgen05 (3xTF32 from the
//                      TMA-loaded planes, TMEM accumulators) -- chosen when its tiles fill
//                      whole rounds of CTAs;
//   pw_sigmoid_kernel  otherwise the same projection with mma.sync m16n8k8 TF32 (3xTF32);
//                      both then write the offsets and sigmoid(mask logits).
// bf16 x is widened exactly; all sums are fp32.
#include <algorithm>
#include <cstdlib>
#include <cstring>

#include "common.cuh"
#include "kernels.h"

namespace defcon {
namespace {

struct BranchArgs {
    const void* x;
    const float* dw_w;
    const float* dw_scale;
    const float* dw_shift;
    const float* pw_w;
    const float* pw_b;
    float* t;          // workspace [M][C] (t, or its tf32-hi plane when t_lo is set)
    float* t_lo;       // [M][C] tf32-lo plane (t - hi) for the tcgen05 1x1, or null
    float* w_hi;       // [OCN][C] W2 tf32-hi plane (rows >= OC zero), written by the dw kernel
    float* w_lo;       // [OCN][C] W2 tf32-lo plane
    int OCN;           // OC rounded up to the 1x1's MMA N
    float* offset;
    float* mask;
    int N, H, W, C, Ho, Wo, M;
    int sh, sw, ph, pw, dh, dw;
    int n_off, n_msk, OC;
    int out_f16;       // offsets / mask written as binary16 (tex2D++, R13)
};

// ------------------------------------------------------------------ depthwise 3x3
// Thread = (8 channels, 4 pixels).  Taps are the outer loop: the 8 weights of a tap are
// read once from shared memory (layout [tap][half][vector][4], conflict-free) and used
// for all 4 pixels, so registers stay low and occupancy high.
constexpr int DW_CH = 64;                  // channels per block (8 vectors of 8)
constexpr int DW_LANES = 32;               // pixel lanes per block
#ifndef DEFCON_DW_PPT
#define DEFCON_DW_PPT 4
#endif
constexpr int DW_PPT = DEFCON_DW_PPT;      // pixels per thread
constexpr int DW_THREADS = DW_LANES * DW_CH / 8;
constexpr int DW_PIX = DW_LANES * DW_PPT;  // pixels per block

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

// 32 zero bytes: the load target of taps that fall into the zero padding, so the tap
// loop needs no branches.
__device__ __align__(32) const uint32_t g_zero32[8] = {0, 0, 0, 0, 0, 0, 0, 0};

#ifndef DEFCON_DW_MINBLOCKS
#define DEFCON_DW_MINBLOCKS 3   // <= 85 registers: 3 blocks per SM, C4 grid of 616 blocks in 2 rounds, not 3
#endif
template <bool BF16>
__global__ void __launch_bounds__(DW_THREADS, DEFCON_DW_MINBLOCKS) dw_bn_relu_kernel(const BranchArgs a) {
    __shared__ __align__(16) float w_s[9 * DW_CH];     // [tap][half][vector][4]
    __shared__ __align__(16) float sc_s[DW_CH], sf_s[DW_CH];
    griddep_wait();                        // PDL: the previous kernel's writes are visible
    griddep_launch_dependents();
    const int tid = threadIdx.x;
    const int c0 = blockIdx.y * DW_CH;
    const int cn = min(DW_CH, a.C - c0);                // multiple of 8
    for (int e = tid; e < cn * 9; e += DW_THREADS) {    // coalesced along dw_w ([C][9])
        const int c = e / 9, k = e - c * 9;
        const int vv = c >> 3, u = c & 7;
        w_s[((k * 2 + (u >> 2)) * 8 + vv) * 4 + (u & 3)] = __ldg(a.dw_w + (long)c0 * 9 + e);
    }
    for (int e = tid; e < cn; e += DW_THREADS) {
        sc_s[e] = __ldg(a.dw_scale + c0 + e);
        sf_s[e] = __ldg(a.dw_shift + c0 + e);
    }
    __syncthreads();
    if (a.w_hi) {   // split W2 into tf32 hi / lo planes for the tcgen05 1x1 (grid-stride, tiny)
        const long nw = (long)a.OCN * a.C;
        const long nthr = (long)gridDim.x * gridDim.y * DW_THREADS;
        for (long e = ((long)blockIdx.y * gridDim.x + blockIdx.x) * DW_THREADS + tid; e < nw; e += nthr) {
            const int o = (int)(e / a.C);
            const float wv = o < a.OC ? __ldg(a.pw_w + e) : 0.f;
            const float h = __uint_as_float(__float_as_uint(wv) & 0xFFFFE000u);
            a.w_hi[e] = h;
            a.w_lo[e] = wv - h;
        }
    }
    const int v = tid & 7;                 // 8-channel vector within the 64-channel slice
    const int lane_p = tid >> 3;           // pixel lane
    if (v * 8 >= cn) return;
    constexpr int ES = BF16 ? 2 : 4;       // bytes per element of x
    const int hw = a.Ho * a.Wo;
    const long pix_bytes = (long)a.C * ES;
    // per pixel: byte pointer of tap (0,0) and a 9-bit mask of taps inside the image
    const uint8_t* base[DW_PPT];
    uint32_t valid[DW_PPT];
#pragma unroll
    for (int pp = 0; pp < DW_PPT; ++pp) {
        const int m = blockIdx.x * DW_PIX + pp * DW_LANES + lane_p;
        valid[pp] = 0u;
        base[pp] = reinterpret_cast<const uint8_t*>(a.x);
        if (m < a.M) {
            const int n = m / hw;
            const int rem = m - n * hw;
            const int ho = rem / a.Wo;
            const int y0 = ho * a.sh - a.ph, x0 = (rem - ho * a.Wo) * a.sw - a.pw;
#pragma unroll
            for (int k = 0; k < 9; ++k) {
                const int yy = y0 + (k / 3) * a.dh, xx = x0 + (k % 3) * a.dw;
                if (yy >= 0 && yy < a.H && xx >= 0 && xx < a.W) valid[pp] |= 1u << k;
            }
            // may point outside x for padded taps; only dereferenced for valid taps
            base[pp] = reinterpret_cast<const uint8_t*>(a.x) +
                       (((long)n * a.H + y0) * a.W + x0) * pix_bytes + (long)(c0 + v * 8) * ES;
        }
    }
    uint64_t s[DW_PPT][4];                 // 8 channels as fp32 pairs (FFMA2)
#pragma unroll
    for (int pp = 0; pp < DW_PPT; ++pp)
#pragma unroll
        for (int u = 0; u < 4; ++u) s[pp][u] = 0ull;
#pragma unroll
    for (int k = 0; k < 9; ++k) {
        const long tap_off = ((long)(k / 3) * a.dh * a.W + (k % 3) * a.dw) * pix_bytes;
        const float4 w0 = *reinterpret_cast<const float4*>(w_s + ((k * 2 + 0) * 8 + v) * 4);
        const float4 w1 = *reinterpret_cast<const float4*>(w_s + ((k * 2 + 1) * 8 + v) * 4);
        const uint64_t wp[4] = {f32x2_pack(w0.x, w0.y), f32x2_pack(w0.z, w0.w), f32x2_pack(w1.x, w1.y),
                                f32x2_pack(w1.z, w1.w)};
#pragma unroll
        for (int pp = 0; pp < DW_PPT; ++pp) {
            const void* src = (valid[pp] >> k) & 1u ? static_cast<const void*>(base[pp] + tap_off)
                                                   : static_cast<const void*>(g_zero32);
            uint64_t xp[4];
            if (BF16) {
                const uint4 u4 = __ldg(static_cast<const uint4*>(src));
                xp[0] = bf16x2_to_f32x2(u4.x); xp[1] = bf16x2_to_f32x2(u4.y);
                xp[2] = bf16x2_to_f32x2(u4.z); xp[3] = bf16x2_to_f32x2(u4.w);
            } else {
                const float4 f0 = __ldg(static_cast<const float4*>(src));
                const float4 f1 = __ldg(static_cast<const float4*>(src) + 1);
                xp[0] = f32x2_pack(f0.x, f0.y); xp[1] = f32x2_pack(f0.z, f0.w);
                xp[2] = f32x2_pack(f1.x, f1.y); xp[3] = f32x2_pack(f1.z, f1.w);
            }
#pragma unroll
            for (int u = 0; u < 4; ++u) s[pp][u] = f32x2_fma(wp[u], xp[u], s[pp][u]);
        }
    }
#pragma unroll
    for (int pp = 0; pp < DW_PPT; ++pp) {
        const int m = blockIdx.x * DW_PIX + pp * DW_LANES + lane_p;
        if (m >= a.M) continue;
        float r[8];
#pragma unroll
        for (int u = 0; u < 4; ++u) {
            r[2 * u] = __uint_as_float((uint32_t)(s[pp][u] & 0xFFFFFFFFull));
            r[2 * u + 1] = __uint_as_float((uint32_t)(s[pp][u] >> 32));
        }
#pragma unroll
        for (int u = 0; u < 8; ++u) r[u] = fmaxf(fmaf(sc_s[v * 8 + u], r[u], sf_s[v * 8 + u]), 0.f);
        float4* dst = reinterpret_cast<float4*>(a.t + (long)m * a.C + c0 + v * 8);
        if (a.t_lo) {   // t = hi + lo exactly: hi = t with the low 13 mantissa bits cleared (tf32)
            float h[8], l[8];
#pragma unroll
            for (int u = 0; u < 8; ++u) {
                h[u] = __uint_as_float(__float_as_uint(r[u]) & 0xFFFFE000u);
                l[u] = r[u] - h[u];
            }
            float4* dlo = reinterpret_cast<float4*>(a.t_lo + (long)m * a.C + c0 + v * 8);
            dst[0] = make_float4(h[0], h[1], h[2], h[3]);
            dst[1] = make_float4(h[4], h[5], h[6], h[7]);
            dlo[0] = make_float4(l[0], l[1], l[2], l[3]);
            dlo[1] = make_float4(l[4], l[5], l[6], l[7]);
        } else {
            dst[0] = make_float4(r[0], r[1], r[2], r[3]);
            dst[1] = make_float4(r[4], r[5], r[6], r[7]);
        }
    }
}

// ------------------------------------------------------------------ 1x1 + sigmoid
// [M x C] x [C x OC] on the tensor cores with mma.sync m16n8k8 TF32 and the 3xTF32 split
// (a = a_hi + a_lo, hi = a truncated to tf32; a*b ~ a_hi*b_hi + a_hi*b_lo + a_lo*b_hi),
// i.e. fp32-level accuracy.  Block = 8 warps over a 64-pixel tile: warp w owns m-tile
// (w % 4) and every other 8-channel k-step of each chunk (w / 4); the two K halves are
// added in shared memory at the end.  64-channel chunks of t and W2 are staged with
// cp.async, double-buffered.
constexpr int PW_WARPS = 8;
constexpr int PW_PIX = 64;                 // pixels per block
constexpr int PW_KC = 64;                  // channels per K chunk
constexpr int PW_S = PW_KC + 4;            // smem row stride (floats): conflict-free fragments

__device__ __forceinline__ void mma_tf32(float (&d)[4], const uint32_t (&a)[4], const uint32_t (&b)[2]) {
    asm volatile(
        "mma.sync.aligned.m16n8k8.row.col.f32.tf32.tf32.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
        "{%0,%1,%2,%3};"
        : "+f"(d[0]), "+f"(d[1]), "+f"(d[2]), "+f"(d[3])
        : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b[0]), "r"(b[1]));
}

__device__ __forceinline__ void split_tf32(float f, uint32_t& hi, uint32_t& lo) {
    hi = __float_as_uint(f) & 0xFFFFE000u;
    lo = __float_as_uint(f - __uint_as_float(hi)) & 0xFFFFE000u;
}

__device__ __forceinline__ void cp_async16(void* smem, const void* gmem, bool valid) {
    const uint32_t s = smem_u32(smem);
    const int n = valid ? 16 : 0;   // zero-fill when invalid
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(s), "l"(gmem), "r"(n) : "memory");
}

template <int NT>
__global__ void __launch_bounds__(PW_WARPS * 32) pw_sigmoid_kernel(const BranchArgs a) {
    constexpr int OCP = 8 * NT;
    constexpr int STAGE = (PW_PIX + OCP) * PW_S;           // floats per stage
    extern __shared__ __align__(16) float sm[];
    griddep_wait();                        // PDL: t from dw_bn_relu_kernel is complete
    griddep_launch_dependents();
    const int tid = threadIdx.x;
    const int warp = tid >> 5, lane = tid & 31;
    const int g = lane >> 2, tq = lane & 3;
    const int mt = warp & 3, kh = warp >> 2;
    const int m0 = blockIdx.x * PW_PIX;
    const int nchunks = (a.C + PW_KC - 1) / PW_KC;

    auto stage_chunk = [&](int ch, int buf) {
        float* ts = sm + buf * STAGE;
        float* ws = ts + PW_PIX * PW_S;
        const int c0 = ch * PW_KC;
        for (int e = tid; e < (PW_PIX + OCP) * (PW_KC / 4); e += PW_WARPS * 32) {
            const int r = e / (PW_KC / 4), q = e - r * (PW_KC / 4);
            const int c = c0 + q * 4;
            if (r < PW_PIX) {
                const int m = m0 + r;
                const bool ok = m < a.M && c < a.C;
                cp_async16(ts + r * PW_S + q * 4, ok ? a.t + (long)m * a.C + c : a.t, ok);
            } else {
                const int o = r - PW_PIX;
                const bool ok = o < a.OC && c < a.C;
                cp_async16(ws + o * PW_S + q * 4, ok ? a.pw_w + (long)o * a.C + c : a.pw_w, ok);
            }
        }
        asm volatile("cp.async.commit_group;" ::: "memory");
    };

    float acc[NT][4];
#pragma unroll
    for (int nt = 0; nt < NT; ++nt)
#pragma unroll
        for (int u = 0; u < 4; ++u) acc[nt][u] = 0.f;

    stage_chunk(0, 0);
    for (int ch = 0; ch < nchunks; ++ch) {
        if (ch + 1 < nchunks) {
            stage_chunk(ch + 1, (ch + 1) & 1);
            asm volatile("cp.async.wait_group 1;" ::: "memory");
        } else {
            asm volatile("cp.async.wait_group 0;" ::: "memory");
        }
        __syncthreads();
        const float* ts = sm + (ch & 1) * STAGE + (mt * 16) * PW_S;
        const float* ws = sm + (ch & 1) * STAGE + PW_PIX * PW_S;
#pragma unroll
        for (int k0 = kh * 8; k0 < PW_KC; k0 += 16) {
            uint32_t ahi[4], alo[4];
            split_tf32(ts[g * PW_S + k0 + tq], ahi[0], alo[0]);
            split_tf32(ts[(g + 8) * PW_S + k0 + tq], ahi[1], alo[1]);
            split_tf32(ts[g * PW_S + k0 + tq + 4], ahi[2], alo[2]);
            split_tf32(ts[(g + 8) * PW_S + k0 + tq + 4], ahi[3], alo[3]);
#pragma unroll
            for (int nt = 0; nt < NT; ++nt) {
                uint32_t bhi[2], blo[2];
                split_tf32(ws[(nt * 8 + g) * PW_S + k0 + tq], bhi[0], blo[0]);
                split_tf32(ws[(nt * 8 + g) * PW_S + k0 + tq + 4], bhi[1], blo[1]);
                mma_tf32(acc[nt], alo, bhi);
                mma_tf32(acc[nt], ahi, blo);
                mma_tf32(acc[nt], ahi, bhi);
            }
        }
        __syncthreads();   // buffer (ch & 1) is refilled two iterations later
    }
    // reduce the two K halves: warps 4..7 hand their accumulators to warps 0..3
    float* red = sm;   // reuse stage memory: [4 warps][NT][4][32]
    if (kh == 1) {
#pragma unroll
        for (int nt = 0; nt < NT; ++nt)
#pragma unroll
            for (int u = 0; u < 4; ++u) red[((mt * NT + nt) * 4 + u) * 32 + lane] = acc[nt][u];
    }
    __syncthreads();
    if (kh == 1) return;
#pragma unroll
    for (int nt = 0; nt < NT; ++nt)
#pragma unroll
        for (int u = 0; u < 4; ++u) acc[nt][u] += red[((mt * NT + nt) * 4 + u) * 32 + lane];
    // D fragment: rows g and g+8, columns 2tq and 2tq+1 of each n-tile
#pragma unroll
    for (int h = 0; h < 2; ++h) {
        const int m = m0 + mt * 16 + g + h * 8;
        if (m >= a.M) continue;
#pragma unroll
        for (int nt = 0; nt < NT; ++nt)
#pragma unroll
            for (int u = 0; u < 2; ++u) {
                const int o = nt * 8 + 2 * tq + u;
                if (o >= a.OC) continue;
                const float val = acc[nt][h * 2 + u] + (a.pw_b ? __ldg(a.pw_b + o) : 0.f);
                if (o < a.n_off)
                    st_offset1(a.offset, (long)m * a.n_off + o, val, a.out_f16);
                else
                    st_offset1(a.mask, (long)m * a.n_msk + (o - a.n_off), 1.f / (1.f + __expf(-val)), a.out_f16);
            }
    }
}

template <int NT>
cudaError_t launch_pw(const BranchArgs& a, cudaStream_t stream) {
    constexpr int OCP = 8 * NT;
    size_t smem = sizeof(float) * 2 * (PW_PIX + OCP) * PW_S;
    const size_t red = sizeof(float) * 4 * NT * 4 * 32;
    if (red > smem) smem = red;
    auto kern = pw_sigmoid_kernel<NT>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    return launch_pdl(kern, dim3((a.M + PW_PIX - 1) / PW_PIX), dim3(PW_WARPS * 32), smem, stream, a);
}


// ------------------------------------------------------------------ 1x1 + sigmoid on tcgen05
// [M x C] x [C x OC] with t already split into tf32 hi / lo planes by the dw kernel, so the
// operand tiles come straight from L2 by TMA in the canonical K-major SWIZZLE_128B layout (no
// producer arithmetic): CTA = 128 pixels (the UMMA M), 32-channel chunks (one 128-byte row),
// 3 MMAs per 8-channel k-step (lo*hi + hi*lo + hi*hi, kind::tf32, fp32-level accuracy), fp32
// accumulators in TMEM.  Legacy mma.sync TF32 issues at about FFMA rate on sm_100a; tcgen05
// does not.  Warps 0-3: W2 chunk split + staging, then the epilogue (TMEM lane quarters);
// warp 4: TMA; warp 5: TMEM allocation + MMA issue.
constexpr int PT_THREADS = 6 * 32;
constexpr int PT_KC = 32;

template <int OCN, int STAGES>
__global__ void __launch_bounds__(PT_THREADS, 2)
    pw_tc_kernel(const __grid_constant__ CUtensorMap thi, const __grid_constant__ CUtensorMap tlo,
                 const __grid_constant__ CUtensorMap whi, const __grid_constant__ CUtensorMap wlo, const BranchArgs a) {
    constexpr int A_BYTES = 128 * 128;               // one plane: 128 rows x 128 bytes
    constexpr int B_BYTES = OCN * 128;
    constexpr int STAGE = 2 * A_BYTES + 2 * B_BYTES;
    constexpr uint32_t TCOLS = OCN <= 32 ? 32 : OCN <= 64 ? 64 : OCN <= 128 ? 128 : 256;
    extern __shared__ __align__(1024) uint8_t pt_raw[];
    uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(pt_raw) + 1023) & ~uintptr_t(1023));
    uint64_t* bars = reinterpret_cast<uint64_t*>(smem + STAGES * STAGE);
    uint64_t* full = bars;                   // [STAGES] TMA tx (t and W2 planes)
    uint64_t* empty = bars + STAGES;         // [STAGES] MMA commit
    uint64_t* tmem_full = bars + 2 * STAGES;
    uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tmem_full + 1);
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int m0 = blockIdx.x * 128;
    const int nch = (a.C + PT_KC - 1) / PT_KC;
    if (tid == 0) {
        for (int s = 0; s < STAGES; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], 1);
        }
        mbar_init(tmem_full, 1);
        fence_barrier_init();
        tma_prefetch_desc(&thi);
        tma_prefetch_desc(&tlo);
        tma_prefetch_desc(&whi);
        tma_prefetch_desc(&wlo);
    }
    if (warp == 5) tmem_alloc<TCOLS>(tmem_slot);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = *tmem_slot;
    griddep_wait();                          // PDL: t and the W2 planes from the dw kernel are complete
    const uint32_t st0 = smem_u32(smem);
    if (warp < 4) {
        // ---- epilogue: TMEM lane = pixel of the tile
        mbar_wait(tmem_full, 0);
        tc_fence_after();
        const int row = warp * 32 + lane;
        const int m = m0 + row;
#pragma unroll 1
        for (int c0 = 0; c0 < OCN; c0 += 16) {
            uint32_t vv[16];
            tmem_ld_32x32b_x16(tmem + ((uint32_t)(warp * 32) << 16) + c0, vv);
            tmem_ld_wait();
            if (m < a.M) {
#pragma unroll
                for (int u = 0; u < 16; ++u) {
                    const int o = c0 + u;
                    if (o >= a.OC) break;
                    const float val = __uint_as_float(vv[u]) + (a.pw_b ? __ldg(a.pw_b + o) : 0.f);
                    if (o < a.n_off)
                        st_offset1(a.offset, (long)m * a.n_off + o, val, a.out_f16);
                    else
                        st_offset1(a.mask, (long)m * a.n_msk + (o - a.n_off), 1.f / (1.f + __expf(-val)), a.out_f16);
                }
            }
        }
    } else if (warp == 4) {
        if (lane == 0) {                     // ---- TMA: t and W2 hi / lo chunks (rows past M zero)
            for (int ch = 0; ch < nch; ++ch) {
                const int s = ch % STAGES;
                mbar_wait(&empty[s], ((uint32_t)(ch / STAGES) & 1u) ^ 1u);
                mbar_arrive_expect_tx(&full[s], STAGE);
                uint8_t* st = smem + s * STAGE;
                tma_load_2d(st, &thi, &full[s], ch * PT_KC, m0);
                tma_load_2d(st + A_BYTES, &tlo, &full[s], ch * PT_KC, m0);
                tma_load_2d(st + 2 * A_BYTES, &whi, &full[s], ch * PT_KC, 0);
                tma_load_2d(st + 2 * A_BYTES + B_BYTES, &wlo, &full[s], ch * PT_KC, 0);
            }
        }
    } else if (lane == 0) {                  // ---- MMA issuer
        constexpr uint32_t idesc = make_idesc(2u /*TF32*/, 128, OCN);
        for (int ch = 0; ch < nch; ++ch) {
            const int s = ch % STAGES;
            mbar_wait(&full[s], (uint32_t)(ch / STAGES) & 1u);
            tc_fence_after();
            const uint32_t ah = st0 + s * STAGE, al = ah + A_BYTES, bh = al + A_BYTES, bl = bh + B_BYTES;
#pragma unroll
            for (int kk = 0; kk < PT_KC / 8; ++kk) {
                const uint64_t dah = make_sw128_desc(ah + kk * 32), dal = make_sw128_desc(al + kk * 32);
                const uint64_t dbh = make_sw128_desc(bh + kk * 32), dbl = make_sw128_desc(bl + kk * 32);
                mma_tf32_ss(tmem, dal, dbh, idesc, (ch | kk) != 0 ? 1u : 0u);
                mma_tf32_ss(tmem, dah, dbl, idesc, 1u);
                mma_tf32_ss(tmem, dah, dbh, idesc, 1u);
            }
            mma_commit(&empty[s]);
        }
        mma_commit(tmem_full);
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 5) {
        tc_fence_after();
        tmem_dealloc<TCOLS>(tmem);
    }
}

template <int OCN, int STAGES>
cudaError_t launch_pw_tc(const BranchArgs& a, cudaStream_t stream) {
    PFN_encodeTiled encode = get_encode_tiled();
    if (!encode) return cudaErrorNotSupported;
    CUtensorMap maps[4];
    for (int p = 0; p < 4; ++p) {
        const bool t = p < 2;
        cuuint64_t dims[2] = {(cuuint64_t)a.C, (cuuint64_t)(t ? a.M : OCN)};
        cuuint64_t strides[1] = {(cuuint64_t)a.C * 4};
        cuuint32_t box[2] = {(cuuint32_t)PT_KC, t ? 128u : (cuuint32_t)OCN};
        cuuint32_t estr[2] = {1, 1};
        float* base = p == 0 ? a.t : p == 1 ? a.t_lo : p == 2 ? a.w_hi : a.w_lo;
        CUresult cr = encode(&maps[p], CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, base, dims, strides, box, estr,
                             CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                             CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
        if (cr != CUDA_SUCCESS) return cudaErrorInvalidValue;
    }
    constexpr int STAGE = 2 * 128 * 128 + 2 * OCN * 128;
    const size_t smem = 1024 + (size_t)STAGES * STAGE + (2 * STAGES + 1) * 8 + 16;
    auto kern = pw_tc_kernel<OCN, STAGES>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    return launch_pdl(kern, dim3((a.M + 127) / 128), dim3(PT_THREADS), smem, stream, maps[0], maps[1], maps[2],
                      maps[3], a);
}

int pw_tc_ocn(int OC) { return OC <= 32 ? 32 : OC <= 64 ? 64 : OC <= 128 ? 128 : 256; }

cudaError_t launch_pw_tc_any(const BranchArgs& a, cudaStream_t stream) {
    // 2 stages keep two CTAs per SM for N <= 64 (the C4 grid of 154 tiles in one round)
    if (a.OCN == 32) return launch_pw_tc<32, 2>(a, stream);
    if (a.OCN == 64) return launch_pw_tc<64, 2>(a, stream);
    if (a.OCN == 128) return launch_pw_tc<128, 2>(a, stream);
    return launch_pw_tc<256, 2>(a, stream);
}

}  // namespace

// t as two fp32 planes (tf32 hi / lo) for the tcgen05 1x1 (or plain t in the first plane), then
// the W2 hi / lo planes padded to 256 rows
static size_t two_pass_workspace(int M, int C) { return (2 * (size_t)M * C + 2 * (size_t)256 * C) * sizeof(float); }

static bool use_onepass(int N, int H, int W, int C, int Ho, int Wo, int K, int G, int sh, int sw, int ph, int pw,
                        int dh, int dw, bool x_bf16) {
#ifdef DEFCON_DEV_TWO_PASS   // dev builds (tools/build_variants.py): time the two-launch path
    return false;
#endif
    return offset_branch_onepass_plan(N, H, W, C, Ho, Wo, sh, sw, ph, pw, dh, dw, 3 * G * K * K, x_bf16);
}

size_t offset_branch_workspace(int N, int H, int W, int C, int Ho, int Wo, int K, int G, int sh, int sw, int ph,
                               int pw, int dh, int dw, bool x_bf16) {
    if (use_onepass(N, H, W, C, Ho, Wo, K, G, sh, sw, ph, pw, dh, dw, x_bf16))
        return offset_branch_onepass_workspace(C, 3 * G * K * K);
    return two_pass_workspace(N * Ho * Wo, C);
}

bool offset_branch_is_onepass(int N, int H, int W, int C, int Ho, int Wo, int K, int G, int sh, int sw, int ph,
                              int pw, int dh, int dw, bool x_bf16) {
    return use_onepass(N, H, W, C, Ho, Wo, K, G, sh, sw, ph, pw, dh, dw, x_bf16);
}

cudaError_t launch_offset_branch(const void* x, bool x_bf16, int N, int H, int W, int C,
                                 const float* dw_w, const float* dw_scale, const float* dw_shift,
                                 const float* pw_w, const float* pw_b, int K, int G, bool with_mask,
                                 int s_h, int s_w, int p_h, int p_w, int d_h, int d_w, int Ho, int Wo,
                                 float* offset, float* mask, float* t_ws, cudaStream_t stream,
                                 bool out_f16, bool prepacked) {
    BranchArgs a;
    a.out_f16 = out_f16 ? 1 : 0;
    a.x = x; a.dw_w = dw_w; a.dw_scale = dw_scale; a.dw_shift = dw_shift;
    a.pw_w = pw_w; a.pw_b = pw_b; a.t = t_ws; a.t_lo = nullptr; a.w_hi = nullptr; a.w_lo = nullptr;
    a.offset = offset; a.mask = mask;
    a.N = N; a.H = H; a.W = W; a.C = C; a.Ho = Ho; a.Wo = Wo; a.M = N * Ho * Wo;
    a.sh = s_h; a.sw = s_w; a.ph = p_h; a.pw = p_w; a.dh = d_h; a.dw = d_w;
    a.n_off = 2 * G * K * K;
    a.n_msk = with_mask ? G * K * K : 0;
    a.OC = a.n_off + a.n_msk;
    if (a.OC > 256) return cudaErrorInvalidValue;   // api.cu maps this to DEFCON_ERR_LIMIT
    // One pass per pixel tile (offset_branch_onepass.cu) wherever it tiles; the two-launch path
    // (dw kernel -> t in HBM -> 1x1 kernel) covers input rows wider than its TMA box.
    if (use_onepass(N, H, W, C, Ho, Wo, K, G, s_h, s_w, p_h, p_w, d_h, d_w, x_bf16))
        return launch_offset_branch_onepass(x, x_bf16, N, H, W, C, dw_w, dw_scale, dw_shift, pw_w, pw_b,
                                            a.n_off, a.n_msk, s_h, s_w, p_h, p_w, d_h, d_w, Ho, Wo, offset,
                                            mask, t_ws, stream, out_f16, prepacked);
    if (prepacked) return cudaErrorNotSupported;   // pre-packed parameters serve the one-pass kernel only
    // 1x1 on tcgen05 from TMA-loaded hi / lo planes, or the mma.sync 3xTF32 kernel (t in one
    // plane)
    // The tcgen05 kernel runs one 128-pixel tile per CTA, two CTAs per SM, each CTA a latency
    // chain over the channel chunks: it wins when its tiles fill whole rounds of CTAs, so a grid
    // whose last round would hold a few stragglers (C3: 298 tiles for 296 slots) keeps mma.sync.
    int sms = 148;
    {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    }
    const int pw_tiles = (a.M + 127) / 128, pw_slots = 2 * sms;
    const int pw_rounds = (pw_tiles + pw_slots - 1) / pw_slots;
    const bool pw_fill = pw_rounds == 1 || pw_tiles - (pw_rounds - 1) * pw_slots >= pw_slots / 2;
    const bool pw_tc = C % 4 == 0 && get_encode_tiled() != nullptr && pw_fill;
    a.OCN = pw_tc_ocn(a.OC);
    if (pw_tc) {
        a.t_lo = t_ws + (size_t)a.M * C;
        a.w_hi = t_ws + 2 * (size_t)a.M * C;
        a.w_lo = a.w_hi + (size_t)256 * C;
    }
    dim3 g1((a.M + DW_PIX - 1) / DW_PIX, (C + DW_CH - 1) / DW_CH);
    cudaError_t e = x_bf16 ? launch_pdl(dw_bn_relu_kernel<true>, g1, dim3(DW_THREADS), 0, stream, a)
                           : launch_pdl(dw_bn_relu_kernel<false>, g1, dim3(DW_THREADS), 0, stream, a);
    if (e != cudaSuccess) return e;
    if (pw_tc) return launch_pw_tc_any(a, stream);
    if (a.OC <= 32) return launch_pw<4>(a, stream);
    if (a.OC <= 64) return launch_pw<8>(a, stream);
    if (a.OC <= 128) return launch_pw<16>(a, stream);
    return launch_pw<32>(a, stream);
}

}  // namespace defcon
