// offset_branch_onepass.cu -- the paper's lightweight offset branch
// as ONE pass over each tile of output pixels, the intermediate t never leaving the SM:
//   t[c] = ReLU(scale[c] * sum_{3x3} W1[c] * x + shift[c])    depthwise 3x3 + folded BN (R10)
//   u[o] = b2[o] + sum_c W2[o][c] * t[c]                      1x1 to OC = G*K*K*(2|3) (R11)
//   offset = u[0 : 2GK^2] ([G][K*K][2] = (dy, dx), R4),  mask = sigmoid(u[2GK^2 :]) (R6)
//
// Tile = R output rows x Wseg columns of one image (R * Wseg <= 128 pixels = the UMMA M rows).
// Per 32-channel chunk:
//   * TMA brings the tile's input window (IR rows x IC columns x 32 channels of NHWC x, box
//     coordinates starting at -pad: the unit zero-fills everything outside the image, which
//     IS the depthwise conv's zero padding) into an unswizzled shared-memory stage whose
//     position stride (80 / 144 bytes) keeps the dw loads free of bank conflicts, XS chunks ahead;
//   * the 8 warps compute t on the CUDA cores: task = (8 channels, output row, run of RUN
//     adjacent pixels); for stride 1 / dilation 1 each input column of a tap row is loaded and
//     widened once and used by every output of the run that covers it (packed FFMA2, fp32);
//   * t goes straight into the 1x1's A operand: two tf32 planes in the canonical K-major
//     SWIZZLE_128B layout, hi = t with the low 13 mantissa bits cleared, lo = t - hi (both exact),
//     and W2's chunk likewise into B (rows >= OC and channels >= C are zero);
//   * one thread issues tcgen05.mma kind::tf32 (M = 128, N = OC rounded up to 16, K = 8) three
//     times per k-step -- lo*hi + hi*lo + hi*hi, the 3xTF32 scheme, fp32-level accuracy --
//     accumulating in TMEM while the warps compute the next chunk (double-buffered A / B).
// Epilogue: TMEM -> + b2 -> offsets, sigmoid -> mask.  Fixed summation order: deterministic.
// Only x is read and only offsets / mask are written: the branch's HBM traffic is the
// algorithmic minimum (x once + halo re-reads from L2, offsets + mask once).
#include <algorithm>
#include <climits>
#include <cstdio>
#include <cstdlib>

#include "common.cuh"
#include "kernels.h"

namespace defcon {
namespace {

constexpr int OP_KC = 32;              // channels per chunk = one 128-byte tf32 operand row
// x stage: one input position = op_kb(ES) channels (the chunk's 32 + 8 / 4 of the next chunk,
// unused), i.e. 80 bytes (bf16) or 144 bytes (fp32), unswizzled.  Pixel p then starts at bank
// 20p / 4p (mod 32): the 8 pixel pairs a warp reads in one instruction hit every bank the same
// number of times (a 64- / 128-byte position would put every even pixel on the same 16 banks).
__host__ __device__ constexpr int op_kb(int es) { return es == 2 ? 40 : 36; }
constexpr uint32_t TF32_HI = 0xFFFFE000u;

#ifdef DEFCON_PROBE_OP_TIMELINE   // dev probe: per-CTA phase timestamps (globaltimer, ns)
__device__ unsigned long long g_op_tl[1024][48];
__device__ __forceinline__ void op_stamp_any(int i) {   // any thread (loader / issuer lanes)
    if (blockIdx.x < 1024 && i < 48) {
        unsigned long long t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        g_op_tl[blockIdx.x][i] = t;
    }
}
#define OPTL_ANY(i) op_stamp_any(i)
__device__ __forceinline__ void op_stamp(int i) {
    if (threadIdx.x == 0 && blockIdx.x < 1024 && i < 32) {
        unsigned long long t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        g_op_tl[blockIdx.x][i] = t;
    }
}
#define OPTL(i) op_stamp(i)
#else
#define OPTL(i) ((void)0)
#define OPTL_ANY(i) ((void)0)
#endif

struct OpArgs {
    const float* dw_w;      // [C][3][3]
    const float* dw_scale;  // [C]
    const float* dw_shift;  // [C]
    const float* pw_w;      // [OC][C]
    const float* pw_b;      // [OC] or null
    const uint8_t* packed;  // per-chunk parameter blocks (op_pack_kernel)
    float* offset;          // [M][n_off]
    float* mask;            // [M][n_msk] or null
    int out_f16;            // offsets / mask written as binary16 (tex2D++, R13)
    int H, W, C, Ho, Wo, Wv;   // Wv = Wo rounded up to even: virtual row length of the tiling
    int MV;                 // N * Ho * Wv virtual pixels
    int sh, sw, ph, pw, dh, dw;
    int n_off, n_msk, OC, OCN;
    int TP;                 // virtual pixels per tile (even; = A rows / TMEM lanes used)
    int IR, IC;             // input window (box) rows over the stacked N*H rows / columns
    int nch;                // 32-channel chunks
    int XS;                 // x stages in flight
    int x_stage;            // bytes per x stage (1024-aligned)
    int tmem_cols, a_col;   // TMEM allocation and first A column
    unsigned long long wv_mul, howv_mul;   // n / Wv, n / (Ho*Wv) as (n * mul) >> (32 + shr)
    int wv_shr, howv_shr;
    int csplit;             // 1, or 2: a 2-CTA cluster per tile, each CTA half of the chunks
    int ksplit;             // csplit 2: rank 0 takes chunks [0, ksplit), rank 1 [ksplit, nch)
    int red_pitch;          // csplit 2: floats per row of the reduction buffer (OCN + 4)
};

// ---- packed per-chunk parameters (written once per call by op_pack_kernel into the caller's
// workspace, then bulk-copied into shared memory with each chunk's x stage): chunk k's block is
//   [W2 hi plane | W2 lo plane]  OCN rows x 32 K positions fp32 each, the exact shared-memory
//        image of the UMMA B operand (K-major SWIZZLE_128B, the permuted K order below, tf32
//        hi = w with the low 13 mantissa bits cleared, lo = w - hi; rows >= OC and channels >= C 0)
//   [dw]  9 taps x 32 channels (transposed), then BN scale[32], shift[32]   (352 fp32)
// K permutation: K position 8c + 2g + e holds channel 8g + 2c + e (the tcgen05.st.16x256b pattern).
__host__ __device__ constexpr int op_block_bytes(int OCN) { return ((2 * OCN * 128 + 11 * OP_KC * 4) + 1023) & ~1023; }

__global__ void __launch_bounds__(256) op_pack_kernel(const float* __restrict__ dw_w, const float* __restrict__ dw_scale,
                                                      const float* __restrict__ dw_shift,
                                                      const float* __restrict__ pw_w, int C, int OC, int OCN,
                                                      uint8_t* __restrict__ packed) {
    griddep_wait();   // the previous launch may still read this workspace's blocks
    griddep_launch_dependents();
    const int k = blockIdx.x;
    uint8_t* blk = packed + (size_t)k * op_block_bytes(OCN);
    const int B_PLANE = OCN * 128;
    const int nthr = blockDim.x * gridDim.y, t0 = blockIdx.y * blockDim.x + threadIdx.x;
    for (int e = t0; e < OCN * OP_KC; e += nthr) {      // B: (row o, K position kp)
        const int o = e / OP_KC, kp = e % OP_KC;
        const int cq = kp >> 3, g = (kp >> 1) & 3, ee = kp & 1;
        const int ch = k * OP_KC + 8 * g + 2 * cq + ee;
        const float w = (o < OC && ch < C) ? pw_w[(long)o * C + ch] : 0.f;
        const uint32_t h = __float_as_uint(w) & TF32_HI;
        const uint32_t byte = (uint32_t)(o * 128 + kp * 4) ^ ((uint32_t)(o & 7) << 4);
        *reinterpret_cast<uint32_t*>(blk + byte) = h;
        *reinterpret_cast<uint32_t*>(blk + B_PLANE + byte) = __float_as_uint(w - __uint_as_float(h));
    }
    float* dwp = reinterpret_cast<float*>(blk + 2 * B_PLANE);
    for (int e = t0; e < 11 * OP_KC; e += nthr) {
        float v = 0.f;
        if (e < 9 * OP_KC) {                              // [tap][ch]
            const int tap = e / OP_KC, c = k * OP_KC + e % OP_KC;
            if (c < C) v = dw_w[(long)c * 9 + tap];
        } else {
            const int c = k * OP_KC + (e - 9 * OP_KC) % OP_KC;
            if (c < C) v = (e < 10 * OP_KC ? dw_scale : dw_shift)[c];
        }
        dwp[e] = v;
    }
}

// Warp roles.  Tile pixels are taken in pairs (virtual columns 2q, 2q+1 of a row: rows have
// even virtual length Wv and tiles start at even pixels, so a pair never straddles a row); the
// tile's nblk = TP/16 <= 8 blocks of 8 pairs live in TMEM lane quarters: block b in lanes
// L(b) = 32(b%4) + 16(b/4) .. +15, the left pixel of pair 8b+l in lane L(b)+l and the right one
// in lane L(b)+l+8 (the lane pattern of tcgen05.st.16x256b).  Compute warp w (quarter w % 4,
// channel half w / 4) handles block w%4 and then, for nblk > 4, block w%4 + 4 (the other half of
// its lane quarter); lane t of it works on pair l = t/4, channels 8g + 4*half .. +3 of the
// chunk's 32 (g = t%4).  The 4 input columns of a tap
// row serve both pixels, the tap weights are read once for both.  t goes to the A operand in
// TENSOR memory, one buffer per channel half (16 K positions: tf32 hi in 16 columns, lo in the
// next 16), so the MMAs read only W2 from shared memory.  The two halves pipeline against each
// other: the issuer warp runs a half's 6 MMAs (2 k-steps x 3xTF32) as soon as its 4 compute
// warps have published it, and those warps compute the next chunk meanwhile, waiting only for
// their own half's previous MMAs before overwriting its buffer.  The loader warp refills a stage
// (x window by TMA + the chunk's packed parameters by bulk copy) once the chunk's last MMAs,
// which follow both halves' reads of the stage, have completed.
constexpr int OP_REGS = 64;            // registers per thread (__maxnreg__)
// n / d for 0 <= n < 2^32 by a multiply and a shift (m = ceil(2^(32+s) / d), s = ceil(log2 d))
__device__ __forceinline__ int op_div(int n, unsigned long long mul, int shr) {
    return (int)(((unsigned long long)(unsigned)n * mul) >> (32 + shr));
}
static void op_div_init(int d, unsigned long long* mul, int* shr) {
    int s = 0;
    while ((1ll << s) < d) ++s;
    *shr = s;
    *mul = ((1ull << (32 + s)) + (unsigned long long)d - 1) / (unsigned long long)d;
}
template <int ES, bool S1>
__global__ void __maxnreg__(OP_REGS)
    offset_branch_onepass_kernel(const __grid_constant__ CUtensorMap xmap, const OpArgs a) {
    extern __shared__ __align__(1024) uint8_t op_raw[];
    // 1024-aligned base by pointer arithmetic on the __shared__ array (keeps every derived
    // pointer in the shared window, so plain loads / stores compile to LDS / STS)
    uint8_t* smem = op_raw + ((1024u - (smem_u32(op_raw) & 1023u)) & 1023u);
    const int B_PLANE = a.OCN * 128;
    const int PBLK = op_block_bytes(a.OCN);
    const int STG = a.x_stage + PBLK;                          // stage = [x window | packed params]
    uint8_t* st_base = smem;                                   // [XS] stages
    uint8_t* zero = st_base + a.XS * STG;                      // 1 KB of zeros
    uint64_t* xfull = reinterpret_cast<uint64_t*>(zero + 2048);    // [XS] stage landed
    uint64_t* afull = xfull + a.XS;                            // [2] half h's A published
    uint64_t* mma_done = afull + 2;                            // [2] half h's MMAs complete
    uint64_t* sfree = mma_done + 2;                            // [XS] stage's last MMAs complete
    uint64_t* acc_full = sfree + a.XS;                         // all MMAs complete
    uint64_t* red_full = acc_full + 1;                         // csplit 2: rank 1's partial landed
    uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(red_full + 1);
    // csplit 2: rank 1's fp32 accumulator, stored into rank 0's copy of this buffer ([128][pitch])
    float* red = reinterpret_cast<float*>((reinterpret_cast<uintptr_t>(tmem_slot) + 16 + 15) & ~uintptr_t(15));
    float* out_s = reinterpret_cast<float*>(smem);             // epilogue staging (stages)

    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int TP = a.TP;
    const int nblk = TP >> 4;                                  // 16-lane blocks (<= 4)
    const int issuer_warp = nblk < 4 ? 3 : 8;                  // ids no compute warp uses
    const int loader_warp = nblk < 4 ? 7 : 9;
    // channel split: the two CTAs of a cluster share the tile, each with half of the chunks
    const int crank = a.csplit == 2 ? (int)cluster_ctarank() : 0;
    const int tile = a.csplit == 2 ? (int)(blockIdx.x >> 1) : (int)blockIdx.x;
    const int kc0 = crank == 0 ? 0 : a.ksplit;
    const int kc1 = a.csplit == 2 && crank == 0 ? a.ksplit : a.nch;
    const int v0 = tile * TP;                                  // first virtual pixel of the tile
    const uint32_t tcols = a.tmem_cols;
    const uint32_t ACOL = a.a_col;                             // first A column (after the accumulator)

    OPTL(0);
    for (int e = tid; e < 256; e += blockDim.x) {
        reinterpret_cast<float*>(zero)[e] = 0.f;
    }
    if (tid == 0) {
        for (int s = 0; s < a.XS; ++s) {
            mbar_init(&xfull[s], 1);
            mbar_init(&sfree[s], 1);
        }
        for (int b = 0; b < 2; ++b) {
            mbar_init(&afull[b], 1);
            mbar_init(&mma_done[b], 1);
        }
        mbar_init(acc_full, 1);
        mbar_init(red_full, 64 * (nblk < 4 ? nblk : 4));   // every compute thread of rank 1
        fence_barrier_init();
        tma_prefetch_desc(&xmap);
    }
    if (warp == 0) {   // TMEM: accumulator (OCN columns) + A (hi / lo x 32 columns)
        if (tcols == 128) tmem_alloc<128>(tmem_slot);
        else if (tcols == 256) tmem_alloc<256>(tmem_slot);
        else tmem_alloc<512>(tmem_slot);
    }
    tc_fence_before();
    __syncthreads();
    if (a.csplit == 2) cluster_sync_all();   // rank 0's red_full initialised before rank 1 arrives
    tc_fence_after();
    const uint32_t tmem = *tmem_slot;
    OPTL(1);
    griddep_wait();                     // PDL: x and the packed parameters are complete
    griddep_launch_dependents();
    OPTL(2);

    const int HoWv = a.Ho * a.Wv;
    const int n0 = op_div(v0, a.howv_mul, a.howv_shr), ho0 = op_div(v0 - n0 * HoWv, a.wv_mul, a.wv_shr);
    const int Y0 = n0 * a.H + ho0 * a.sh - a.ph;              // window origin (stacked rows)

    if (warp == loader_warp) {
        // ===================== stage loader (TMA x window + bulk-copied parameters) =========
        if (lane == 0) {
            const uint32_t tx = (uint32_t)(a.IR * a.IC * op_kb(ES) * ES + PBLK);
            auto load_stage = [&](int k, int s) {
                uint8_t* st = st_base + s * STG;
                mbar_arrive_expect_tx(&xfull[s], tx);
                tma_load_3d(st, &xmap, &xfull[s], k * OP_KC, -a.pw, Y0);
                bulk_load(st + a.x_stage, a.packed + (size_t)k * PBLK, (uint32_t)PBLK, &xfull[s]);
            };
            const int nk = kc1 - kc0;                // this CTA's chunks kc0 .. kc1-1
            for (int i = 0; i < a.XS && i < nk; ++i) load_stage(kc0 + i, i);
            for (int i = a.XS; i < nk; ++i) {      // stage of chunk i - XS: its MMAs are done
                const int s = i % a.XS;
                mbar_wait(&sfree[s], (uint32_t)((i - a.XS) / a.XS) & 1u);
                if (i < 8) OPTL_ANY(32 + i);
                load_stage(kc0 + i, s);
            }
        }
        return;
    }
    if (warp == issuer_warp) {
        // ===================== MMA issuer =====================
        if (lane == 0) {
            const uint32_t idesc = make_idesc(2u /*TF32*/, 128, (uint32_t)a.OCN);
            int s = 0;
            for (int k = 0; k < kc1 - kc0; ++k) {   // local chunk index
                const uint32_t bh = smem_u32(st_base + s * STG + a.x_stage), bl = bh + B_PLANE;
#pragma unroll
                for (int h = 0; h < 2; ++h) {
                    mbar_wait(&afull[h], (uint32_t)k & 1u);         // half h of chunk k published
                    if (h == 1 && k < 8) OPTL_ANY(40 + k);
                    tc_fence_after();
                    const uint32_t ah = tmem + ACOL + 32u * h, al = ah + 16u;
#pragma unroll
                    for (int kk = 0; kk < 2; ++kk) {               // K positions 16h + 8kk .. +7
                        const uint32_t kb = (uint32_t)(2 * h + kk) * 32u;
                        const uint64_t dbh = make_sw128_desc(bh + kb), dbl = make_sw128_desc(bl + kb);
                        mma_tf32_ts(tmem, al + kk * 8, dbh, idesc, (k | h | kk) != 0 ? 1u : 0u);
                        mma_tf32_ts(tmem, ah + kk * 8, dbl, idesc, 1u);
                        mma_tf32_ts(tmem, ah + kk * 8, dbh, idesc, 1u);
                    }
                    mma_commit(&mma_done[h]);
                }
                mma_commit(&sfree[s]);
                if (++s == a.XS) s = 0;
            }
            mma_commit(acc_full);
        }
        return;
    }
    const int NQ = nblk < 4 ? nblk : 4;                        // lane quarters in use
    if (warp >= 8 || (warp & 3) >= NQ) return;                 // unused ids (small tiles)

    // ===================== compute warps =====================
    // warp (quarter qd, half) handles block qd (lanes 32qd .. +15) and, for nblk > 4, block
    // qd + 4 (lanes 32qd + 16 .. +31), one after the other
    const int NC = 64 * NQ;                                    // compute threads
    const int ctid = ((warp >> 2) * NQ + (warp & 3)) * 32 + lane;   // 0 .. NC-1
    const int qd = warp & 3, half = warp >> 2;
    const int nsub = qd + 4 < nblk ? 2 : 1;                    // blocks of this warp
    const int l = lane >> 2, g = lane & 3;
    constexpr uint32_t PB = op_kb(ES) * ES;                    // bytes per input position of a stage
    const uint32_t chb = (uint32_t)(8 * g + 4 * half) * ES;    // byte offset of this thread's 4 channels
    uint32_t row_byte[2][3];   // stage byte offset of tap (i, 0) of the left pixel + channels
    uint32_t row_ok[2];        // tap rows not in the zero padding (incl. a neighbouring image's rows)
#pragma unroll
    for (int sb = 0; sb < 2; ++sb) {
        const int q = 8 * (qd + 4 * sb) + l;                   // pixel pair within the tile
        const int vp = v0 + 2 * q;                             // virtual pixel of the left one
        const bool pix_ok = sb < nsub && vp < a.MV;
        const int vpc = pix_ok ? vp : v0;
        const int n = op_div(vpc, a.howv_mul, a.howv_shr);
        const int rem = vpc - n * HoWv;
        const int ho = op_div(rem, a.wv_mul, a.wv_shr), wo = rem - ho * a.Wv;   // wo even
        row_ok[sb] = 0;
#pragma unroll
        for (int i = 0; i < 3; ++i) {
            const int yy = ho * a.sh - a.ph + i * a.dh;
            const bool ok = pix_ok && yy >= 0 && yy < a.H;
            row_ok[sb] |= ok ? 1u << i : 0u;
            row_byte[sb][i] = (ok ? (uint32_t)((n * a.H + yy - Y0) * a.IC + wo * a.sw) * PB : 0u) + chb;
        }
    }
    const uint32_t col_step = (uint32_t)a.dw * PB;   // next tap column
    const uint32_t px_step = (uint32_t)a.sw * PB;    // the right pixel of the pair
    // this half's A buffer, lanes of block qd; block qd + 4 is 16 lanes further
    const uint32_t a_addr = tmem + ((uint32_t)(32 * qd) << 16) + ACOL + 32u * half;
    const bool half_lead = qd == 0 && lane == 0;
    const int wofs = 2 * B_PLANE / 4 + 8 * g + 4 * half;       // this thread's dw weights in a stage (floats)

    int s = 0;                          // stage of chunk k (k mod XS)
    uint32_t xphase = 0;
    for (int k = 0; k < kc1 - kc0; ++k) {   // local chunk index (chunk kc0 + k)
        const uint8_t* xst = st_base + s * STG;
        const float* wk = reinterpret_cast<const float*>(xst + a.x_stage) + wofs;
        mbar_wait(&xfull[s], xphase);
        if (k < 8) OPTL(4 + 2 * k);
#pragma unroll 1
        for (int sb = 0; sb < nsub; ++sb) {
            const uint32_t rok = sb ? row_ok[1] : row_ok[0];
            // ---- depthwise 3x3 of 4 channels at two pixels, fp32 pairs (FFMA2)
            uint64_t acc0[2] = {0ull, 0ull}, acc1[2] = {0ull, 0ull};
#pragma unroll
            for (int i = 0; i < 3; ++i) {
                const bool ok = (rok >> i) & 1u;
                const uint8_t* rb = ok ? xst : zero;
                const uint32_t rbyte = sb ? row_byte[1][i] : row_byte[0][i];
                uint64_t w[3][2];
#pragma unroll
                for (int jj = 0; jj < 3; ++jj) {
                    const float4 w0 = *reinterpret_cast<const float4*>(wk + (i * 3 + jj) * OP_KC);
                    w[jj][0] = f32x2_pack(w0.x, w0.y);
                    w[jj][1] = f32x2_pack(w0.z, w0.w);
                }
                auto ld4 = [&](uint32_t byte, uint64_t (&v)[2]) {   // 4 channels -> 2 fp32 pairs
                    if (ES == 2) {
                        const uint2 u = *reinterpret_cast<const uint2*>(rb + byte);
                        v[0] = bf16x2_to_f32x2(u.x);
                        v[1] = bf16x2_to_f32x2(u.y);
                    } else {
                        const uint4 u = *reinterpret_cast<const uint4*>(rb + byte);
                        v[0] = ((uint64_t)u.y << 32) | u.x;
                        v[1] = ((uint64_t)u.w << 32) | u.z;
                    }
                };
                if (S1) {
                    // stride-1 / dilation-1 columns: c = 0..3 feed the left pixel through tap c and
                    // the right one through tap c - 1
#pragma unroll
                    for (int c = 0; c < 4; ++c) {
                        uint64_t v[2];
                        ld4(ok ? rbyte + c * PB : chb, v);
#pragma unroll
                        for (int p = 0; p < 2; ++p) {
                            if (c < 3) acc0[p] = f32x2_fma(w[c][p], v[p], acc0[p]);
                            if (c > 0) acc1[p] = f32x2_fma(w[c - 1][p], v[p], acc1[p]);
                        }
                    }
                } else {
#pragma unroll
                    for (int jj = 0; jj < 3; ++jj) {
                        uint64_t v[2], u[2];
                        ld4(ok ? rbyte + jj * col_step : chb, v);
                        ld4(ok ? rbyte + jj * col_step + px_step : chb, u);
#pragma unroll
                        for (int p = 0; p < 2; ++p) {
                            acc0[p] = f32x2_fma(w[jj][p], v[p], acc0[p]);
                            acc1[p] = f32x2_fma(w[jj][p], u[p], acc1[p]);
                        }
                    }
                }
            }
            // ---- folded BN + ReLU, tf32 hi / lo split; register 4c' + 2x + e = channel
            // 8g + 4*half + 2c' + e of pixel x (the 16x256b.x2 store pattern)
            uint32_t hv[8], lv[8];
            {
                const float4 sc = *reinterpret_cast<const float4*>(wk + 9 * OP_KC);
                const float4 sf = *reinterpret_cast<const float4*>(wk + 10 * OP_KC);
                const float scv[4] = {sc.x, sc.y, sc.z, sc.w};
                const float sfv[4] = {sf.x, sf.y, sf.z, sf.w};
#pragma unroll
                for (int x = 0; x < 2; ++x) {
                    const uint64_t* acc = x ? acc1 : acc0;
#pragma unroll
                    for (int c = 0; c < 2; ++c) {
#pragma unroll
                        for (int e = 0; e < 2; ++e) {
                            const float v = __uint_as_float(e ? (uint32_t)(acc[c] >> 32) : (uint32_t)(acc[c] & 0xFFFFFFFFull));
                            const float t = fmaxf(fmaf(scv[2 * c + e], v, sfv[2 * c + e]), 0.f);
                            const uint32_t h = __float_as_uint(t) & TF32_HI;
                            hv[4 * c + 2 * x + e] = h;
                            lv[4 * c + 2 * x + e] = __float_as_uint(t - __uint_as_float(h));
                        }
                    }
                }
            }
            // this half's A buffer was last read by its MMAs of chunk k-1
            if (sb == 0 && k >= 1) mbar_wait(&mma_done[half], (uint32_t)(k - 1) & 1u);
            tc_fence_after();
            const uint32_t ad = a_addr + ((uint32_t)(16 * sb) << 16);
            tmem_st_16x256b_x2(ad, hv);
            tmem_st_16x256b_x2(ad + 16u, lv);
        }
        tmem_st_wait();
        tc_fence_before();
        named_bar_sync(1 + half, NC / 2);      // this half's A of chunk k complete
        if (k < 8) OPTL(5 + 2 * k);
        if (half_lead) mbar_arrive(&afull[half]);
        if (++s == a.XS) {
            s = 0;
            xphase ^= 1u;
        }
    }
    // ---- epilogue: accumulator lane = tile pixel (pair layout above), column = output channel;
    // + b2, sigmoid on the mask channels, staged in shared memory in the global layout (the tile's
    // real pixels are one contiguous range of m), then copied out coalesced.  Warp (qd, half)
    // reads lanes 32qd .. +31 (blocks qd and qd + 4) and the 16-column groups half, half + 2, ..
    OPTL(20);
    float bias_r[16];
    {
        const int cg0 = half;                                  // the first column group (bias prefetch)
#pragma unroll
        for (int u = 0; u < 16; ++u) {
            const int o = 16 * cg0 + u;
            bias_r[u] = (a.pw_b && o < a.OC) ? __ldg(a.pw_b + o) : 0.f;
        }
    }
    mbar_wait(acc_full, 0u);
    tc_fence_after();
    OPTL(21);
    if (a.csplit == 2 && crank == 1) {
        // rank 1: its partial accumulator (its half of the channels) into rank 0's red buffer,
        // one release-arrive per thread, then leave; rank 0 finishes the tile
        const int ngrp = a.OCN >> 4;
        const int row = 32 * qd + lane;                        // TMEM lane = red row
        for (int cg = half; cg < ngrp; cg += 2) {
            uint32_t vv[16];
            tmem_ld_32x32b_x16(tmem + ((uint32_t)(32 * qd) << 16) + (uint32_t)(16 * cg), vv);
            tmem_ld_wait();
            const uint32_t la = smem_u32(red + row * a.red_pitch + 16 * cg);
#pragma unroll
            for (int u = 0; u < 4; ++u) st_cluster_v4(la + 16 * u, 0, vv[4 * u], vv[4 * u + 1], vv[4 * u + 2], vv[4 * u + 3]);
        }
        mbar_arrive_release_cluster(red_full, 0);
        tc_fence_before();
        named_bar_sync(3, NC);   // TMEM no longer read
        if (warp == 0) {
            tc_fence_after();
            if (tcols == 128) tmem_dealloc<128>(tmem);
            else if (tcols == 256) tmem_dealloc<256>(tmem);
            else tmem_dealloc<512>(tmem);
        }
        return;
    }
    if (a.csplit == 2) mbar_wait_cluster(red_full, 0u);   // rank 1's partial is in red
    const int vl = min(v0 + TP, a.MV) - 1;
    auto real_m = [&](int v, bool up) {   // m of virtual pixel v (dead column: next / previous real)
        const int r = op_div(v, a.wv_mul, a.wv_shr), c = v - r * a.Wv;
        if (c >= a.Wo) return up ? (r + 1) * a.Wo : r * a.Wo + a.Wo - 1;
        return r * a.Wo + c;
    };
    const int mf = real_m(v0, true), ml = real_m(vl, false);
    const int nreal = ml - mf + 1;
    float* off_s = out_s;
    float* msk_s = out_s + nreal * a.n_off;
    {
        const int li = lane & 15, bb = qd + 4 * (lane >> 4);
        const int v = v0 + 2 * (8 * bb + (li & 7)) + (li >> 3);   // virtual pixel of lane 32*qd + lane
        const int rr = op_div(v, a.wv_mul, a.wv_shr), cc = v - rr * a.Wv;
        const bool ok = bb < nblk && v < a.MV && cc < a.Wo;
        const int dm = rr * a.Wo + cc - mf;                   // real-pixel index within the tile
        const int ngrp = a.OCN >> 4;                           // 16-column groups
        for (int cg = half; cg < ngrp; cg += 2) {
            uint32_t vv[16];
            tmem_ld_32x32b_x16(tmem + ((uint32_t)(32 * qd) << 16) + (uint32_t)(16 * cg), vv);
            tmem_ld_wait();
            if (!ok) continue;
#pragma unroll
            for (int u = 0; u < 16; ++u) {
                const int o = 16 * cg + u;
                const float val = __uint_as_float(vv[u]) +
                                  (a.csplit == 2 ? red[(32 * qd + lane) * a.red_pitch + o] : 0.f) +
                                  (cg == half ? bias_r[u] : (a.pw_b && o < a.OC) ? __ldg(a.pw_b + o) : 0.f);
                if (o < a.n_off) off_s[dm * a.n_off + o] = val;
                else if (o < a.OC) msk_s[dm * a.n_msk + (o - a.n_off)] = __fdividef(1.f, 1.f + __expf(-val));
            }
        }
    }
    OPTL(23);
    tc_fence_before();
    named_bar_sync(3, NC);   // staged; TMEM no longer read
    OPTL(30);
    {   // the stores first (fire and forget), the TMEM release after them
        const long go = (long)mf * a.n_off;
        for (int e = ctid; e < nreal * a.n_off; e += NC) st_offset1(a.offset, go + e, off_s[e], a.out_f16);
        if (a.n_msk) {
            const long gm = (long)mf * a.n_msk;
            for (int e = ctid; e < nreal * a.n_msk; e += NC) st_offset1(a.mask, gm + e, msk_s[e], a.out_f16);
        }
    }
    OPTL(31);
    if (warp == 0) {
        tc_fence_after();
        if (tcols == 128) tmem_dealloc<128>(tmem);
        else if (tcols == 256) tmem_dealloc<256>(tmem);
        else tmem_dealloc<512>(tmem);
    }
    OPTL(22);
}

struct OpPlan {
    OpArgs a;
    int tiles, cps;
    size_t smem;
};

constexpr size_t OP_SMEM_CAP = 228 * 1024 - 1024;   // per SM, less the per-CTA reserve
#ifdef OP_PROBE_ONE_CTA   // dev probe: one CTA per SM
constexpr size_t OP_SMEM_TWO = 0;
#else
constexpr size_t OP_SMEM_TWO = 113 * 1024;   // two CTAs per SM
#endif

size_t op_smem(const OpArgs& a) {
    return 1024 + (size_t)a.XS * (a.x_stage + op_block_bytes(a.OCN)) + 2048 + (2 * a.XS + 6) * 8 + 16 +
           (a.csplit == 2 ? (size_t)128 * a.red_pitch * 4 + 16 : 0);
}

// Tile = TP consecutive pixels of the virtual [N][Ho][Wv] grid (a tile may run across an image
// boundary: its input window covers the stacked N*H rows, and taps in another image's rows are
// masked as zero padding).  TP (a multiple of 16, <= 128 = the UMMA M) spreads the pixels evenly
// over the CTA slots: minimise rounds x CTAs-per-SM x TP, the pixels one SM processes.
// Tile size / channel split measured per layer shape and per-GPU batch by tools/autotune.py
// (branch_tuning_table.inc, compiled in); shapes not in it take the time model below.
struct OpTuneEntry {
    int C, H, W, stride, OC, nmin, nmax, TP, csplit;
};
static const OpTuneEntry kOpTuneTable[] = {
#include "branch_tuning_table.inc"
    {0, 0, 0, 0, 0, 0, 0, 0, 0}   // terminator
};

bool make_op_plan(int N, int H, int W, int C, int Ho, int Wo, int sh, int sw, int ph, int pw, int dh, int dw,
                  int OC, int es, OpPlan* p) {
    OpArgs& a = p->a;
    a.H = H; a.W = W; a.C = C; a.Ho = Ho; a.Wo = Wo;
    a.Wv = Wo + (Wo & 1);
    a.sh = sh; a.sw = sw; a.ph = ph; a.pw = pw; a.dh = dh; a.dw = dw;
    a.OC = OC;
    a.OCN = (OC + 15) & ~15;
    const long MV = (long)N * Ho * a.Wv;
    if (a.OCN > 256 || C % 8 != 0 || MV >= (1L << 31)) return false;
    a.MV = (int)MV;
    op_div_init(a.Wv, &a.wv_mul, &a.wv_shr);
    op_div_init(Ho * a.Wv, &a.howv_mul, &a.howv_shr);
    a.nch = (C + OP_KC - 1) / OP_KC;
    a.IC = (a.Wv - 1) * sw + 2 * dw + 1;
    if (a.IC > 256) return false;                 // TMA box limit: wide images keep the two-pass path
    // TMEM: accumulator columns (OCN rounded to 32), then the A operand (hi, lo) x 32 columns
    a.a_col = (a.OCN + 31) & ~31;
    a.tmem_cols = a.a_col + 64 <= 128 ? 128 : a.a_col + 64 <= 256 ? 256 : 512;
    int sms = 148;
    {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    }
    double best = 1e30;
    bool found = false;
    int force_split = 0, force_tp = 0;
    for (const OpTuneEntry* e = kOpTuneTable; e->C; ++e)
        if (e->C == C && e->H == H && e->W == W && e->stride == sh && sw == sh && e->OC == OC && N >= e->nmin &&
            N <= e->nmax && dh == 1 && dw == 1) {
            force_tp = e->TP;
            force_split = e->csplit;
            break;
        }
    // DEFCON_OP_TP / DEFCON_OP_CSPLIT override the table (the autotune sweep, tests)
    if (const char* env = getenv("DEFCON_OP_TP")) force_tp = atoi(env);
    if (const char* env = getenv("DEFCON_OP_CSPLIT")) force_split = atoi(env);
    OpArgs best_t = a;
    auto search = [&](int ftp, int fsplit) {
    for (int cs = 1; cs <= 2; ++cs)
    for (int TP = 16; TP <= 128; TP += 16) {
        if (fsplit && cs != fsplit) break;
        if (cs == 2 && a.nch < 2) break;
        if (TP > Ho * a.Wv && TP > 16) break;     // a tile spans at most two images
        if (ftp && TP != ftp) continue;
        OpArgs t = a;
        t.TP = TP;
        t.csplit = cs;
        t.ksplit = (a.nch + 1) / 2;
        t.red_pitch = a.OCN + 4;
        const int orows = (a.Wv - 2 + TP + a.Wv - 1) / a.Wv;          // output rows a tile can touch
        t.IR = (orows - 1) * sh + std::max(0, H - Ho * sh) + 2 * dh + 1;
        if (t.IR > 256) continue;
        t.x_stage = (int)(((size_t)t.IR * t.IC * op_kb(es) * es + 1023) & ~size_t(1023));
        // epilogue staging ([TP][OC] fp32) reuses the x stages
        t.XS = 3;
        while (op_smem(t) > OP_SMEM_CAP / 3 && t.XS > 2) --t.XS;
        if ((size_t)TP * OC * 4 > (size_t)t.XS * t.x_stage) continue;
        const size_t sm = op_smem(t);
        if (sm > OP_SMEM_CAP) continue;
        // CTAs per SM: shared memory, TMEM columns (512 per SM), registers
        const int nwarps = TP >= 64 ? 10 : 8;
        int cps = (int)std::min<size_t>(OP_SMEM_CAP / sm, 512 / t.tmem_cols);
        // OP_REGS registers per thread: 4 sub-partitions x 16K registers per SM
        cps = std::min(cps, 4 * (16384 / (OP_REGS * 32)) / nwarps);
        if (cps < 1) continue;
        const long tiles = (MV + TP - 1) / TP;
        const long ctas = tiles * cs;
        const long rounds = (ctas + (long)sms * cps - 1) / ((long)sms * cps);
        // time model: every CTA is a latency chain of its chunks (cost per chunk grows with the
        // pixels per compute warp and with the CTAs sharing the SM) plus a fixed prologue /
        // epilogue (the channel split adds the DSMEM reduction)
        const int kper = cs == 2 ? std::max(t.ksplit, a.nch - t.ksplit) : a.nch;
        const double per_chunk = (TP + 16) / 80.0 * (0.55 + 0.15 * std::min<long>(cps, (ctas + sms - 1) / sms));
        const double cost = rounds * (kper * per_chunk + 4.0 + (cs == 2 ? 0.7 : 0.0));
        if (cost < best) {
            best = cost;
            best_t = t;
            p->tiles = (int)ctas;
            p->cps = cps;
            p->smem = sm;
            found = true;
        }
    }
    };
    search(force_tp, force_split);
    if (!found && (force_tp || force_split)) search(0, 0);   // a table entry that no longer fits
    if (found) a = best_t;
    return found;
}

template <int ES>
cudaError_t launch_op(const OpPlan& p, const CUtensorMap& xmap, cudaStream_t stream) {
    if (getenv("DEFCON_DEBUG"))
        fprintf(stderr, "defcon onepass: TP=%d ctas=%d csplit=%d cps=%d XS=%d IR=%d IC=%d smem=%zu tmem=%d\n",
                p.a.TP, p.tiles, p.a.csplit, p.cps, p.a.XS, p.a.IR, p.a.IC, p.smem, p.a.tmem_cols);
    const bool s1 = p.a.sw == 1 && p.a.dw == 1;
    auto kern = s1 ? offset_branch_onepass_kernel<ES, true> : offset_branch_onepass_kernel<ES, false>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)p.smem);
    if (e != cudaSuccess) return e;
    const int nblk = p.a.TP / 16;
    // compute warps 0..nblk-1 (half 0), 4..3+nblk (half 1); issuer + loader: 3, 7 or 8, 9
    const int threads = 32 * (nblk < 4 ? 8 : 10);
    if (p.a.csplit != 2) return launch_pdl(kern, dim3(p.tiles), dim3(threads), p.smem, stream, xmap, p.a);
    cudaLaunchConfig_t cfg = {};   // 2-CTA clusters (the channel split) + PDL
    cfg.gridDim = dim3(p.tiles);
    cfg.blockDim = dim3(threads);
    cfg.dynamicSmemBytes = p.smem;
    cfg.stream = stream;
    cudaLaunchAttribute attr[2];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = 2;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[1].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 2;
    return cudaLaunchKernelEx(&cfg, kern, xmap, p.a);
}

}  // namespace

#ifdef DEFCON_PROBE_OP_TIMELINE
extern "C" int defcon_debug_op_timeline(unsigned long long* host) {
    return (int)cudaMemcpyFromSymbol(host, g_op_tl, sizeof(g_op_tl));
}
#endif

bool offset_branch_onepass_plan(int N, int H, int W, int C, int Ho, int Wo, int sh, int sw, int ph, int pw,
                                int dh, int dw, int OC, bool x_bf16) {
    OpPlan p;
    return get_encode_tiled() != nullptr &&
           make_op_plan(N, H, W, C, Ho, Wo, sh, sw, ph, pw, dh, dw, OC, x_bf16 ? 2 : 4, &p);
}

size_t offset_branch_onepass_workspace(int C, int OC) {
    const int OCN = (OC + 15) & ~15;
    return (size_t)((C + OP_KC - 1) / OP_KC) * op_block_bytes(OCN);
}

// The per-chunk parameter blocks (W2 hi / lo in the UMMA B image + dw / BN), OC outputs.
cudaError_t launch_offset_pack(const float* dw_w, const float* dw_scale, const float* dw_shift, const float* pw_w,
                               int C, int OC, void* packed, cudaStream_t stream) {
    const int OCN = (OC + 15) & ~15;
    const int nch = (C + OP_KC - 1) / OP_KC;
    return launch_pdl(op_pack_kernel, dim3(nch, (OCN * OP_KC + 255) / 256), dim3(256), 0, stream, dw_w, dw_scale,
                      dw_shift, pw_w, C, OC, OCN, static_cast<uint8_t*>(packed));
}

cudaError_t launch_offset_branch_onepass(const void* x, bool x_bf16, int N, int H, int W, int C,
                                         const float* dw_w, const float* dw_scale, const float* dw_shift,
                                         const float* pw_w, const float* pw_b, int n_off, int n_msk,
                                         int s_h, int s_w, int p_h, int p_w, int d_h, int d_w, int Ho, int Wo,
                                         float* offset, float* mask, void* ws, cudaStream_t stream,
                                         bool out_f16, bool prepacked) {
    const int es = x_bf16 ? 2 : 4;
    OpPlan p;
    if (!make_op_plan(N, H, W, C, Ho, Wo, s_h, s_w, p_h, p_w, d_h, d_w, n_off + n_msk, es, &p))
        return cudaErrorInvalidValue;
    OpArgs& a = p.a;
    a.dw_w = dw_w; a.dw_scale = dw_scale; a.dw_shift = dw_shift;
    a.pw_w = pw_w; a.pw_b = pw_b; a.offset = offset; a.mask = mask;
    a.n_off = n_off; a.n_msk = n_msk;
    a.out_f16 = out_f16 ? 1 : 0;
    a.packed = static_cast<const uint8_t*>(ws);
    // PDL launch: its launch overlaps the previous kernel; it waits for that kernel before writing
    // (measured A/B on one box: bench step 75.5 -> 74.8 us, host entry 0.70 -> 0.56 ms)
    if (!prepacked) {   // else ws holds the blocks of defcon_offset_pack_params (packed once per weights)
        cudaError_t e = launch_offset_pack(dw_w, dw_scale, dw_shift, pw_w, C, a.OC, ws, stream);
        if (e != cudaSuccess) return e;
    }
    PFN_encodeTiled encode = get_encode_tiled();
    if (!encode) return cudaErrorNotSupported;
    // x as a 3-D tensor [N*H][W][C] (C innermost); box = 32 channels x IC columns x IR rows
    CUtensorMap xmap;
    cuuint64_t dims[3] = {(cuuint64_t)C, (cuuint64_t)W, (cuuint64_t)N * H};
    cuuint64_t strides[2] = {(cuuint64_t)C * es, (cuuint64_t)W * C * es};
    cuuint32_t box[3] = {(cuuint32_t)op_kb(es), (cuuint32_t)a.IC, (cuuint32_t)a.IR};
    cuuint32_t estr[3] = {1, 1, 1};
    CUresult cr = encode(&xmap, x_bf16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3,
                         const_cast<void*>(x), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                         CU_TENSOR_MAP_SWIZZLE_NONE,
                         CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (cr != CUDA_SUCCESS) return cudaErrorInvalidValue;
    return x_bf16 ? launch_op<2>(p, xmap, stream) : launch_op<4>(p, xmap, stream);
}

}  // namespace defcon
