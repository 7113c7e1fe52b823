// dcn_tc_bf16.cu -- fused deformable convolution forward on the 5th-gen tensor cores.
//
// Computes Eq.2 with the bilinear kernel Eq.3, zero outside
// the image, offset groups and the DCNv2 mask (R6) as one implicit GEMM
//     Y[m, co] = bias[co] + sum_kd A[m, kd] * Wt[co, kd],   kd = tap * Cin + ci
// where A[m, kd] = m_k * X(p_o + p_k + dp_k) is produced on the fly (never in HBM).
//
// Per CTA: one 128-row (output pixel) x BLOCK_N (output channel) tile.
//   warps 0..NPW-1  A producers: bilinear gathers from NHWC bf16 x (16-byte vectors,
//                   fp32 weights and lerp, RNE to bf16) written into the canonical
//                   SWIZZLE_128B K-major smem layout; afterwards they run the epilogue
//                   (tcgen05.ld -> + bias -> bf16 -> NHWC store).
//   warp NPW        TMA producer for the weight tile (B, K-major, SWIZZLE_128B).
//   warp NPW+1      TMEM allocator and single-thread tcgen05.mma issuer (M=128, N<=256
//                   per instruction, K=16), fp32 accumulators in TMEM.
// K loop: 64-channel chunks (outer) x taps (inner) so the taps of one chunk revisit
// the same input neighbourhood while it is hot in L1.  Per-(row, tap) sampling
// metadata (4 corner offsets, 4 mask-scaled weights) is computed once per offset group
// into shared memory and reused by every chunk of that group.
#include <cstdio>

#include "common.cuh"
#include "kernels.h"

namespace defcon {
namespace {

constexpr int BM = 128;          // rows per tile (UMMA M)
constexpr int BK = 64;           // bf16 elements per K chunk (= one 128-byte swizzle row)
constexpr int A_STAGE_BYTES = BM * BK * 2;
constexpr int META_ENTRY = 32;   // int4 corner offsets + float4 weights

struct TcArgs {
    const __nv_bfloat16* x;
    const float* offset;
    const float* mask;
    const float* bias;
    __nv_bfloat16* y;
    int H, W, Cin, Cout, Kw, Ho, Wo;
    int sh, sw, ph, pw, dh, dw;
    int G, Cg, M, KK;
    int num_chunks;   // Cin / BK
    int num_iters;    // num_chunks * KK
};

template <int BLOCK_N>
struct TcCfg {
    static constexpr int UMMA_N = BLOCK_N > 256 ? 256 : BLOCK_N;
    static constexpr int N_MMA = BLOCK_N / UMMA_N;
    static constexpr int B_STAGE_BYTES = BLOCK_N * BK * 2;
    static constexpr int STAGE_BYTES = A_STAGE_BYTES + B_STAGE_BYTES;
    static constexpr int TMEM_COLS = BLOCK_N < 32 ? 32 : BLOCK_N;
    static constexpr int TMA_BOX_N = BLOCK_N > 256 ? 256 : BLOCK_N;
};

// Sampling metadata for (row, tap) of offset group g: the element index of channel 0 of
// each of the 4 bilinear corners and the 4 corner weights with the mask folded in.
// Corners outside the image get weight 0 and a harmless in-bounds index 0 (R8).
__device__ __forceinline__ void build_meta_entry(const TcArgs& a, int m0, int row, int tap, int g,
                                                 uint8_t* meta) {
    int4 off = make_int4(0, 0, 0, 0);
    float4 wt = make_float4(0.f, 0.f, 0.f, 0.f);
    const int m = m0 + row;
    if (m < a.M) {
        const int hw = a.Ho * a.Wo;
        const int n = m / hw;
        const int rem = m - n * hw;
        const int ho = rem / a.Wo;
        const int wo = rem - ho * a.Wo;
        const int i = tap / a.Kw;
        const int j = tap - i * a.Kw;
        const long pix = (long)m * a.G + g;
        const float2 d = *reinterpret_cast<const float2*>(a.offset + (pix * a.KK + tap) * 2);
        const float mk = a.mask ? a.mask[pix * a.KK + tap] : 1.0f;
        float py = (float)(ho * a.sh - a.ph + i * a.dh) + d.x;
        float px = (float)(wo * a.sw - a.pw + j * a.dw) + d.y;
        // Anything beyond one pixel outside samples only zeros; clamping keeps the
        // int conversion defined for huge / non-finite offsets.
        py = fminf(fmaxf(py, -2.0f), (float)a.H + 1.0f);
        px = fminf(fmaxf(px, -2.0f), (float)a.W + 1.0f);
        if (py == py && px == px) {
            const float fy = floorf(py), fx = floorf(px);
            const float ly = py - fy, lx = px - fx;
            const int y0 = (int)fy, x0 = (int)fx;
            const bool vy0 = (y0 >= 0) && (y0 < a.H), vy1 = (y0 + 1 >= 0) && (y0 + 1 < a.H);
            const bool vx0 = (x0 >= 0) && (x0 < a.W), vx1 = (x0 + 1 >= 0) && (x0 + 1 < a.W);
            const int base = n * a.H;
            if (vy0 && vx0) { off.x = ((base + y0) * a.W + x0) * a.Cin;         wt.x = (1.f - ly) * (1.f - lx) * mk; }
            if (vy0 && vx1) { off.y = ((base + y0) * a.W + x0 + 1) * a.Cin;     wt.y = (1.f - ly) * lx * mk; }
            if (vy1 && vx0) { off.z = ((base + y0 + 1) * a.W + x0) * a.Cin;     wt.z = ly * (1.f - lx) * mk; }
            if (vy1 && vx1) { off.w = ((base + y0 + 1) * a.W + x0 + 1) * a.Cin; wt.w = ly * lx * mk; }
        }
    }
    uint8_t* e = meta + (row * a.KK + tap) * META_ENTRY;
    *reinterpret_cast<int4*>(e) = off;
    *reinterpret_cast<float4*>(e + 16) = wt;
}

__device__ __forceinline__ void lerp_accumulate(float (&acc)[8], const uint4& v, float w) {
    acc[0] = fmaf(w, bf16lo_to_f32(v.x), acc[0]);
    acc[1] = fmaf(w, bf16hi_to_f32(v.x), acc[1]);
    acc[2] = fmaf(w, bf16lo_to_f32(v.y), acc[2]);
    acc[3] = fmaf(w, bf16hi_to_f32(v.y), acc[3]);
    acc[4] = fmaf(w, bf16lo_to_f32(v.z), acc[4]);
    acc[5] = fmaf(w, bf16hi_to_f32(v.z), acc[5]);
    acc[6] = fmaf(w, bf16lo_to_f32(v.w), acc[6]);
    acc[7] = fmaf(w, bf16hi_to_f32(v.w), acc[7]);
}

template <int BLOCK_N, int STAGES, int NPW>
__global__ void __launch_bounds__((NPW + 2) * 32, 1)
    dcn_fwd_bf16_tc_kernel(const __grid_constant__ CUtensorMap wmap, const TcArgs a) {
    using Cfg = TcCfg<BLOCK_N>;
    constexpr int NPT = NPW * 32;                 // producer threads
    constexpr int ROWS_PER_PASS = NPT / 8;        // 8 threads (16 B each) per 128-B row
    constexpr int PASSES = BM / ROWS_PER_PASS;    // rows per producer thread

    extern __shared__ __align__(1024) uint8_t smem_raw[];
    // 1024-byte alignment for the SWIZZLE_128B atoms.
    uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                               ~uintptr_t(1023));
    uint8_t* sA = smem;
    uint8_t* sB = smem + STAGES * A_STAGE_BYTES;
    uint8_t* meta = sB + STAGES * Cfg::B_STAGE_BYTES;
    uint64_t* bars = reinterpret_cast<uint64_t*>(meta + BM * a.KK * META_ENTRY);
    uint64_t* full_a = bars;
    uint64_t* full_b = bars + STAGES;
    uint64_t* empty = bars + 2 * STAGES;
    uint64_t* accum_full = bars + 3 * STAGES;
    uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 3 * STAGES + 1);

    const int warp = threadIdx.x >> 5;
    const int lane = threadIdx.x & 31;
    const int m0 = blockIdx.x * BM;
    const int n0 = blockIdx.y * BLOCK_N;

    if (warp == NPW && lane == 0) {
        for (int s = 0; s < STAGES; ++s) {
            mbar_init(&full_a[s], NPW);
            mbar_init(&full_b[s], 1);
            mbar_init(&empty[s], 1);
        }
        mbar_init(accum_full, 1);
        fence_barrier_init();
        tma_prefetch_desc(&wmap);
    }
    if (warp == NPW + 1) tmem_alloc<Cfg::TMEM_COLS>(tmem_slot);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = *tmem_slot;

    if (warp < NPW) {
        // ===================== A producers =====================
        const int t = threadIdx.x;
        const int cvec = t & 7;            // 16-byte vector within the 128-byte row
        const int rsub = t >> 3;
        int cur_group = -1;
        for (int it = 0; it < a.num_iters; ++it) {
            const int chunk = it / a.KK;
            const int tap = it - chunk * a.KK;
            const int g = (chunk * BK) / a.Cg;
            if (g != cur_group) {
                if (cur_group >= 0) named_bar_sync(1, NPT);   // old table no longer read
                for (int e = t; e < BM * a.KK; e += NPT) build_meta_entry(a, m0, e / a.KK, e % a.KK, g, meta);
                named_bar_sync(1, NPT);
                cur_group = g;
            }
            const int s = it % STAGES;
            const uint32_t ph = (uint32_t)(it / STAGES) & 1u;
            mbar_wait(&empty[s], ph ^ 1u);

            const int ch = chunk * BK + cvec * 8;
            const __nv_bfloat16* xc = a.x + ch;
            uint4 v[PASSES][4];
            float4 w[PASSES];
#pragma unroll
            for (int p = 0; p < PASSES; ++p) {
                const int row = rsub + p * ROWS_PER_PASS;
                const uint8_t* e = meta + (row * a.KK + tap) * META_ENTRY;
                const int4 o = *reinterpret_cast<const int4*>(e);
                w[p] = *reinterpret_cast<const float4*>(e + 16);
                v[p][0] = ldg_nc_v4(xc + o.x);
                v[p][1] = ldg_nc_v4(xc + o.y);
                v[p][2] = ldg_nc_v4(xc + o.z);
                v[p][3] = ldg_nc_v4(xc + o.w);
            }
            const uint32_t a_stage = smem_u32(sA + s * A_STAGE_BYTES);
#pragma unroll
            for (int p = 0; p < PASSES; ++p) {
                const int row = rsub + p * ROWS_PER_PASS;
                float acc[8];
#pragma unroll
                for (int c = 0; c < 8; ++c) acc[c] = 0.f;
                lerp_accumulate(acc, v[p][0], w[p].x);
                lerp_accumulate(acc, v[p][1], w[p].y);
                lerp_accumulate(acc, v[p][2], w[p].z);
                lerp_accumulate(acc, v[p][3], w[p].w);
                const uint32_t dst = a_stage + row * 128 + ((cvec ^ (row & 7)) << 4);
                st_shared_v4(dst, pack_bf16x2(acc[0], acc[1]), pack_bf16x2(acc[2], acc[3]),
                             pack_bf16x2(acc[4], acc[5]), pack_bf16x2(acc[6], acc[7]));
            }
            fence_proxy_async_smem();
            __syncwarp();
            if (lane == 0) mbar_arrive(&full_a[s]);
        }

        // ===================== epilogue =====================
        mbar_wait(accum_full, 0);
        tc_fence_after();
        const int q = warp & 3;                    // TMEM lane quarter of this warp
        constexpr int SLICES = NPW / 4;
        constexpr int COLS = BLOCK_N / SLICES;
        const int col0 = (warp >> 2) * COLS;
        const int row = m0 + q * 32 + lane;
        __nv_bfloat16* yrow = a.y + (size_t)row * a.Cout + n0;
#pragma unroll 1
        for (int c = col0; c < col0 + COLS; c += 16) {
            uint32_t r[16];
            tmem_ld_32x32b_x16(tmem_base + ((uint32_t)(q * 32) << 16) + (uint32_t)c, r);
            tmem_ld_wait();
            if (row < a.M && n0 + c < a.Cout) {
                uint32_t pk[8];
#pragma unroll
                for (int j = 0; j < 8; ++j) {
                    float b0 = a.bias ? __ldg(a.bias + n0 + c + 2 * j) : 0.f;
                    float b1 = a.bias ? __ldg(a.bias + n0 + c + 2 * j + 1) : 0.f;
                    pk[j] = pack_bf16x2(__uint_as_float(r[2 * j]) + b0,
                                        __uint_as_float(r[2 * j + 1]) + b1);
                }
                uint4* dst = reinterpret_cast<uint4*>(yrow + c);
                dst[0] = make_uint4(pk[0], pk[1], pk[2], pk[3]);
                dst[1] = make_uint4(pk[4], pk[5], pk[6], pk[7]);
            }
        }
    } else if (warp == NPW) {
        // ===================== TMA producer (weights) =====================
        if (lane == 0) {
            for (int it = 0; it < a.num_iters; ++it) {
                const int chunk = it / a.KK;
                const int tap = it - chunk * a.KK;
                const int s = it % STAGES;
                const uint32_t ph = (uint32_t)(it / STAGES) & 1u;
                mbar_wait(&empty[s], ph ^ 1u);
                mbar_arrive_expect_tx(&full_b[s], Cfg::B_STAGE_BYTES);
                const int kd = tap * a.Cin + chunk * BK;
#pragma unroll
                for (int h = 0; h < BLOCK_N / Cfg::TMA_BOX_N; ++h)
                    tma_load_2d(sB + s * Cfg::B_STAGE_BYTES + h * Cfg::TMA_BOX_N * 128, &wmap,
                                &full_b[s], kd, n0 + h * Cfg::TMA_BOX_N);
            }
        }
    } else {
        // ===================== MMA issuer =====================
        if (lane == 0) {
            constexpr uint32_t idesc = make_idesc(1u /*BF16*/, BM, Cfg::UMMA_N);
            for (int it = 0; it < a.num_iters; ++it) {
                const int s = it % STAGES;
                const uint32_t ph = (uint32_t)(it / STAGES) & 1u;
                mbar_wait(&full_a[s], ph);
                mbar_wait(&full_b[s], ph);
                tc_fence_after();
                const uint32_t a_addr = smem_u32(sA + s * A_STAGE_BYTES);
                const uint32_t b_addr = smem_u32(sB + s * Cfg::B_STAGE_BYTES);
#pragma unroll
                for (int kk = 0; kk < BK / 16; ++kk) {
                    const uint64_t adesc = make_sw128_desc(a_addr + kk * 32);
#pragma unroll
                    for (int h = 0; h < Cfg::N_MMA; ++h) {
                        const uint64_t bdesc =
                            make_sw128_desc(b_addr + h * Cfg::UMMA_N * 128 + kk * 32);
                        mma_bf16_ss(tmem_base + h * Cfg::UMMA_N, adesc, bdesc, idesc,
                                    (it | kk) != 0 ? 1u : 0u);
                    }
                }
                mma_commit(&empty[s]);
            }
            mma_commit(accum_full);
        }
    }

    __syncwarp();
    tc_fence_before();
    __syncthreads();
    if (warp == NPW + 1) {
        tc_fence_after();
        tmem_dealloc<Cfg::TMEM_COLS>(tmem_base);
    }
}

template <int BLOCK_N, int STAGES, int NPW>
cudaError_t launch_impl(const DcnGeom& g, const DcnPtrs& p, cudaStream_t stream,
                        const char** detail) {
    using Cfg = TcCfg<BLOCK_N>;
    PFN_encodeTiled encode = get_encode_tiled();
    if (!encode) {
        *detail = "cuTensorMapEncodeTiled entry point unavailable";
        return cudaErrorNotSupported;
    }
    const int Kd = g.KK * g.Cin;
    CUtensorMap wmap;
    cuuint64_t dims[2] = {(cuuint64_t)Kd, (cuuint64_t)g.Cout};
    cuuint64_t strides[1] = {(cuuint64_t)Kd * 2};
    cuuint32_t box[2] = {(cuuint32_t)BK, (cuuint32_t)Cfg::TMA_BOX_N};
    cuuint32_t estr[2] = {1, 1};
    CUresult cr = encode(&wmap, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(p.weight),
                         dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                         CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                         CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (cr != CUDA_SUCCESS) {
        *detail = "cuTensorMapEncodeTiled failed for the weight tensor";
        return cudaErrorInvalidValue;
    }
    TcArgs a;
    a.x = static_cast<const __nv_bfloat16*>(p.x);
    a.offset = p.offset;
    a.mask = p.mask;
    a.bias = p.bias;
    a.y = static_cast<__nv_bfloat16*>(p.y);
    a.H = g.H; a.W = g.W; a.Cin = g.Cin; a.Cout = g.Cout; a.Kw = g.Kw; a.Ho = g.Ho; a.Wo = g.Wo;
    a.sh = g.sh; a.sw = g.sw; a.ph = g.ph; a.pw = g.pw; a.dh = g.dh; a.dw = g.dw;
    a.G = g.G; a.Cg = g.Cg; a.M = g.M; a.KK = g.KK;
    a.num_chunks = g.Cin / BK;
    a.num_iters = a.num_chunks * g.KK;

    const size_t smem = 1024 + (size_t)STAGES * Cfg::STAGE_BYTES + (size_t)BM * g.KK * META_ENTRY +
                        (3 * STAGES + 1) * 8 + 16;
    auto kern = dcn_fwd_bf16_tc_kernel<BLOCK_N, STAGES, NPW>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) {
        *detail = "cudaFuncSetAttribute(MaxDynamicSharedMemorySize) failed";
        return e;
    }
    dim3 grid((g.M + BM - 1) / BM, (g.Cout + BLOCK_N - 1) / BLOCK_N);
    kern<<<grid, (NPW + 2) * 32, smem, stream>>>(wmap, a);
    e = cudaGetLastError();
    if (e != cudaSuccess) *detail = "dcn_fwd_bf16_tc_kernel launch failed";
    return e;
}

}  // namespace

// Shared-memory budget: stages + metadata for up to 5x5 taps must fit in 227 KB.
bool dcn_tc_bf16_supported(const DcnGeom& g) {
    if (g.Cin % BK != 0 || g.Cg % BK != 0) return false;
    if (g.Cout % 16 != 0) return false;
    if ((long)BM * g.KK * META_ENTRY > 48 * 1024) return false;
    return true;
}

cudaError_t launch_dcn_tc_bf16(const DcnGeom& g, const DcnPtrs& p, cudaStream_t stream,
                               const char** detail) {
    if (g.Cout <= 64) return launch_impl<64, 6, 8>(g, p, stream, detail);
    if (g.Cout <= 128) return launch_impl<128, 4, 8>(g, p, stream, detail);
    if (g.Cout <= 256) return launch_impl<256, 3, 8>(g, p, stream, detail);
    return launch_impl<512, 2, 8>(g, p, stream, detail);
}

}  // namespace defcon
