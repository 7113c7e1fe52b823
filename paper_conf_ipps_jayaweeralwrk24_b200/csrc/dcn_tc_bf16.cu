// dcn_tc_bf16.cu -- fused deformable convolution forward on the 5th-gen tensor cores.
//
// Computes Eq.2 with the bilinear kernel Eq.3, zero outside
// the image, offset groups and the DCNv2 mask (R6) as one implicit GEMM
//     Y[m, co] = bias[co] + sum_kd A[m, kd] * Wt[co, kd],   kd = tap * Cin + ci
// where A[m, kd] = m_k * X(p_o + p_k + dp_k) is produced on the fly (never in HBM).
//
// Persistent, stream-K scheduled: the (tile, k-iteration) space -- tiles of 128 output
// pixels x BLOCK_N output channels, k-iterations of 64 input channels x 1 tap -- is cut
// into one contiguous, equal range per CTA (grid = #SMs), so there is no wave tail.
// A tile split between CTAs is finished by whichever contributor arrives last on the
// tile's counter, summing the fp32 partials in fixed segment order (deterministic).
//
// Warp roles (14 warps):
//   0..7    A producers: bilinear gathers from NHWC bf16 x (16-byte vectors, fp32 weights
//           and lerp, RNE to bf16) into the canonical SWIZZLE_128B K-major smem layout.
//   8..11   epilogue: tcgen05.ld accumulators (TMEM lane = output row), + bias, bf16 NHWC
//           store, or fp32 partial + stream-K fixup.
//   12      TMA producer for the weight tile (B, K-major, SWIZZLE_128B).
//   13      TMEM allocator and single-thread tcgen05.mma issuer (M=128, N<=256, K=16),
//           fp32 accumulators double-buffered in TMEM when BLOCK_N <= 256.
// K order inside a tile: 64-channel chunks (outer) x taps (inner), so the taps of one
// chunk revisit the same input neighbourhood while it is hot in L1.  Per-(row, tap)
// sampling metadata (4 corner offsets, 4 mask-scaled weights) is built once per
// (tile, offset group) into shared memory and reused by every chunk of that group.
#include <algorithm>
#include <type_traits>
#include <cstdio>
#include <cstdlib>

#include "common.cuh"
#include "kernels.h"

namespace defcon {
namespace {

constexpr int BM = 128;          // rows per tile (UMMA M)
constexpr int BK = 64;           // bf16 elements per K chunk (= one 128-byte swizzle row)
constexpr int A_PLANE = BM * 128;   // one A operand plane: BM rows x 128 bytes
// Element type of x / W / y: bf16 (kind::f16, one plane, 64 channels per k-iteration) or fp32
// (kind::tf32 3xTF32: hi / lo planes, 32 channels per k-iteration).  A k-iteration covers one
// 128-byte row of channels either way.
template <bool F32>
struct Elem {
    static constexpr int ES = F32 ? 4 : 2;           // bytes per element
    static constexpr int CPI = 128 / ES;             // channels per k-iteration
    static constexpr int PLANES = F32 ? 2 : 1;       // operand planes (tf32 hi / lo)
    static constexpr int A_STAGE = A_PLANE * PLANES;
};
// Per-(row, tap) sampling metadata entry.  bf16 x: 16 bytes {byte offset of the top-left
// corner | 1 when the right-hand corners are a pixel further, byte offset of the bottom-left
// corner, bf16 weights (w0, w1), (w2, w3)} (invalid corners alias a valid in-bounds one and have
// weight 0); texture rows: float4 {u, v, mask, -}; fp32 x: 32 bytes {4 corner offsets, 4 fp32
// weights}.
template <bool F32>
__host__ __device__ constexpr int meta_entry() { return F32 ? 32 : 16; }
constexpr int META_ENTRY = 32;   // the largest entry (shape-support checks)
#ifndef DEFCON_NPW
#define DEFCON_NPW 8
#endif
constexpr int NPW = DEFCON_NPW;  // producer warps (8 or 16)
#ifndef DEFCON_LATE_LAST
#define DEFCON_LATE_LAST 0   // 1: the last row's next gathers after the full_a arrive, 2: all rows (DESIGN 12b)
#endif
constexpr int EPI_WARP0 = NPW;   // 4 epilogue warps: TMEM lane quarters 0..3
constexpr int TMA_WARP = NPW + 4;
constexpr int MMA_WARP = NPW + 5;
constexpr int NUM_THREADS = (NPW + 6) * 32;
constexpr int FEPI_WARPS = 8;    // producer warps that run the CTA's last epilogue
constexpr int NPT = NPW * 32;
constexpr int TPR = 4;               // producer threads per 128-byte A row (32 bytes each)
constexpr int ROWS = BM * TPR / NPT; // A rows per producer thread
constexpr int RPW = 32 / TPR;        // rows per warp per pass

#ifdef DEFCON_PROBE_KTRACE   // dev probe: per-k-iteration event clock64 stamps of CTA `KTRACE_CTA`
__device__ long long g_kt[24][64];
__device__ int g_kt_q;
#ifndef KTRACE_CTA
#define KTRACE_CTA 5
#endif
__device__ __forceinline__ void kt_stamp(int ev, int q) {
    if (blockIdx.x == KTRACE_CTA && q < 64) g_kt[ev][q] = clock64();
}
#define KT(ev, q) kt_stamp(ev, q)
#else
#define KT(ev, q) ((void)0)
#endif

#ifdef DEFCON_PROBE_TIMELINE   // dev probe: per-CTA phase timestamps (globaltimer, ns)
__device__ unsigned long long g_tl[256][16];
__device__ __forceinline__ void tl_stamp(int i) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    g_tl[blockIdx.x][i] = t;
}
#define TL(i) tl_stamp(i)
#else
#define TL(i) ((void)0)
#endif

struct TcArgs {
    const void* x;
    const float* offset;
    const float* mask;
    const float* bias;
    void* y;
    float* partials;       // [2 * gridDim.x][BLOCK_N / 4][BM][4] fp32
    int* counters;         // [num_tiles], zeroed before launch
    int H, W, Cin, Cout, Kw, Ho, Wo;
    int sh, sw, ph, pw, dh, dw;
    int G, Cg, M, KK;
    float bound_h;         // bounded deformation half-window (R12); < 0: unbounded
    int off_f16;           // offsets / mask in binary16 (tex2D++, R13)
    int ipt;               // k-iterations per tile = (Cin / CPI) * KK
    int es, cpi;           // element bytes, channels per k-iteration
    int n_tiles_n;         // tiles along Cout
    long long total_iters; // num_tiles * ipt
    unsigned long long tex;          // DEFCON_SAMPLER_TEX: stacked-image texture object, else 0
    int bias_in_smem;      // Cout <= BIAS_SMEM_MAX: bias (or zeros) staged in shared memory
    int pair;              // 1: CTA pairs (cta_group::2, M = 256 per MMA), tiles of 2 x BM rows
};

constexpr int BIAS_SMEM_MAX = 1024;

// Byte offset of the bias table behind the barriers / TMEM slot / fix flags (16-aligned).
__host__ __device__ constexpr int bias_smem_offset(int stages, int nbuf) {
    return (((3 * stages + 2 * nbuf) * 8 + 12) + 15) & ~15;
}

template <int BLOCK_N, bool PAIR = false, bool F32 = false>
struct TcCfg {
    static constexpr int UMMA_N = BLOCK_N > 256 ? 256 : BLOCK_N;
    static constexpr int N_MMA = BLOCK_N / UMMA_N;
    static constexpr int B_ROWS = PAIR ? BLOCK_N / 2 : BLOCK_N;   // B rows staged by this CTA
    static constexpr int B_PLANE = B_ROWS * 128;
    static constexpr int B_STAGE_BYTES = B_PLANE * Elem<F32>::PLANES;
    static constexpr int A_STAGE_BYTES = Elem<F32>::A_STAGE;
    static constexpr int STAGE_BYTES = A_STAGE_BYTES + B_STAGE_BYTES;
    static constexpr int NBUF = BLOCK_N <= 256 ? 2 : 1;      // TMEM accumulator buffers
    // F32: two accumulators per buffer -- hi*hi, and the small cross terms lo*hi + hi*lo in
    // their own (ACC_STRIDE = BLOCK_N columns further) -- summed in the epilogue
    static constexpr int NACC = F32 ? 2 : 1;
    static constexpr int ACC_STRIDE = BLOCK_N * NACC;      // columns per accumulator buffer
    static constexpr int TMEM_COLS = (ACC_STRIDE * NBUF) < 32 ? 32 : ACC_STRIDE * NBUF;
    static constexpr int TMA_BOX_N = B_ROWS > 256 ? 256 : B_ROWS;
};

// First output row of `tile` for this CTA: tiles are BM rows, or 2 x BM rows split between
// the two CTAs of a pair (rank r owns rows r*BM .. r*BM + BM - 1).
template <bool PAIR>
__device__ __forceinline__ int tile_m0(const TcArgs& a, int tile) {
    if (!PAIR) return (tile / a.n_tiles_n) * BM;
    return (tile / a.n_tiles_n) * (2 * BM) + (int)cluster_ctarank() * BM;
}

// Static stream-K partition: CTA b owns global iterations [it0(b), it0(b+1)).
__device__ __forceinline__ long long range_begin(long long T, int G, int b) {
    return (T * b) / G;
}
// The CTA whose range contains global iteration `it`.
__device__ __forceinline__ int cta_of(long long T, int G, long long it) {
    return (int)(((it + 1) * G - 1) / T);
}

// One segment = the part of one tile inside this CTA's range.
struct Segment {
    int tile;
    int kb, ke;          // k-iteration range within the tile
};


// Sampling metadata for (row, tap) of offset group g: the byte offset (into x) of
// channel 0 of each of the 4 bilinear corners and the 4 corner weights with the mask
// folded in.  Corners outside the image get weight 0 and the harmless in-bounds
// offset 0 (R8).  Built in two passes over a thread's entries -- all offset/mask
// loads first, then the arithmetic -- so a table costs one memory round trip, not one
// per entry.
struct MetaIn {
    float2 d;     // (dy, dx) offset (R4)
    float mk;     // mask (1 for DCNv1)
};


// Output pixel of tile row `row`: image n and the top-left tap position (R3).
struct RowPos {
    int n, yb, xb;
    bool ok;
};

__device__ __forceinline__ RowPos row_pos(const TcArgs& a, int m) {
    RowPos p;
    p.ok = m < a.M;
    const int mm = p.ok ? m : 0;
    const int hw = a.Ho * a.Wo;
    p.n = mm / hw;
    const int rem = mm - p.n * hw;
    const int ho = rem / a.Wo;
    p.yb = ho * a.sh - a.ph;
    p.xb = (rem - ho * a.Wo) * a.sw - a.pw;
    return p;
}

// One metadata entry (see meta_entry) for tap (i, j) of row rp, computed without branches so
// that a thread's entries are independent dependency chains the scheduler can interleave.
// Corners outside the image get weight 0 and an in-bounds address (R8).
struct MetaVal {
    uint4 lo, hi;   // hi: fp32 weights of the 32-byte format
};

template <bool COMPACT>
__device__ __forceinline__ MetaVal meta_value(const TcArgs& a, const RowPos& rp, int i, int j, const MetaIn& in,
                                              bool tex_row) {
    float2 d = in.d;
    if (a.bound_h >= 0.f) {   // bounded deformation (R12)
        const int Kh = a.KK / a.Kw;
        d.x = bound_offset(d.x, (i - 0.5f * (Kh - 1)) * a.dh, a.bound_h);
        d.y = bound_offset(d.y, (j - 0.5f * (a.Kw - 1)) * a.dw, a.bound_h);
    }
    const float mk = in.mk;
    const float py0 = (float)(rp.yb + i * a.dh) + d.x;
    const float px0 = (float)(rp.xb + j * a.dw) + d.y;
    const bool fin = rp.ok && py0 == py0 && px0 == px0;
    MetaVal r;
    if (tex_row) {
        // texture sampler: unnormalised texel coordinates (texel centres at +0.5, R7) in the
        // stacked-image texture (image n occupies rows n*(H+1) .. n*(H+1)+H-1, row
        // n*(H+1)+H is zero) and the mask.  Clamping to [-1, H] x [-1, W] keeps samples
        // beyond the image on zero texels.
        const float u = fminf(fmaxf(px0, -1.0f), (float)a.W) + 0.5f;
        const float v = (float)(rp.n * (a.H + 1)) + fminf(fmaxf(py0, -1.0f), (float)a.H) + 0.5f;
        r.lo = make_uint4(__float_as_uint(fin ? u : -4.f), __float_as_uint(fin ? v : -4.f),
                          __float_as_uint(fin ? mk : 0.f), 0u);
        r.hi = make_uint4(0u, 0u, 0u, 0u);
        return r;
    }
    // Anything beyond one pixel outside samples only zeros; clamping keeps the int conversion
    // defined for huge offsets (non-finite ones are mapped to a fully outside point).
    const float py = fin ? fminf(fmaxf(py0, -2.0f), (float)a.H + 1.0f) : -2.0f;
    const float px = fin ? fminf(fmaxf(px0, -2.0f), (float)a.W + 1.0f) : -2.0f;
    const int y0 = __float2int_rd(py), x0 = __float2int_rd(px);
    const float ly = py - (float)y0, lx = px - (float)x0;
    const bool vy0 = (unsigned)y0 < (unsigned)a.H, vy1 = (unsigned)(y0 + 1) < (unsigned)a.H;
    const bool vx0 = (unsigned)x0 < (unsigned)a.W, vx1 = (unsigned)(x0 + 1) < (unsigned)a.W;
    const float w0 = (vy0 && vx0) ? (1.f - ly) * (1.f - lx) * mk : 0.f;
    const float w1 = (vy0 && vx1) ? (1.f - ly) * lx * mk : 0.f;
    const float w2 = (vy1 && vx0) ? ly * (1.f - lx) * mk : 0.f;
    const float w3 = (vy1 && vx1) ? ly * lx * mk : 0.f;
    const uint32_t base = (uint32_t)(rp.n * a.H);
    const uint32_t pb = (uint32_t)(a.Cin * a.es);   // bytes per pixel
    const uint32_t rowb = (uint32_t)a.W * pb;
    if constexpr (COMPACT) {   // one valid column / row stands in for an invalid one (weight 0)
        const int ya = vy0 ? y0 : (vy1 ? y0 + 1 : 0);
        const int xa = vx0 ? x0 : (vx1 ? x0 + 1 : 0);
        const uint32_t o = (base + (uint32_t)ya) * rowb + (uint32_t)xa * pb;
        r.lo = make_uint4(o | ((vx0 && vx1) ? 1u : 0u), (vy0 && vy1) ? o + rowb : o, pack_bf16x2(w0, w1),
                          pack_bf16x2(w2, w3));
        r.hi = make_uint4(0u, 0u, 0u, 0u);
    } else {
        const uint32_t o00 = (base + (uint32_t)y0) * rowb + (uint32_t)x0 * pb;
        r.lo = make_uint4((vy0 && vx0) ? o00 : 0u, (vy0 && vx1) ? o00 + pb : 0u, (vy1 && vx0) ? o00 + rowb : 0u,
                          (vy1 && vx1) ? o00 + rowb + pb : 0u);
        r.hi = make_uint4(__float_as_uint(w0), __float_as_uint(w1), __float_as_uint(w2), __float_as_uint(w3));
    }
    return r;
}

constexpr int STG_TAPS = 5;   // entries per thread per round of the table build

// The whole (tile, group) table, built by the NPT = TPM * BM producer threads: thread t owns
// row t / TPM and taps t % TPM, + TPM, ... in rounds of STG_TAPS entries: all inputs of a round
// are loaded before any arithmetic, and the entries
// are computed as independent chains before any is stored.  Rows of warp w use the format of
// that warp's sampler.
constexpr int TPM = NPT / BM;    // producer threads per tile row in the metadata build
static_assert(NPT % BM == 0, "metadata build assumes whole producer threads per tile row");
template <int NTEX, int ME>
__device__ __forceinline__ void build_meta_table(const TcArgs& a, int m0, int g, uint8_t* meta, int t) {
    const int row = t / TPM;
    const RowPos rp = row_pos(a, m0 + row);
    const bool tex_row = ((row % (NPW * RPW)) / RPW) < NTEX;
    const long pix = (long)(m0 + row) * a.G + g;
    uint8_t* rmeta = meta + row * a.KK * ME;
    if (t == 0) KT(16, g_kt_q);
    const long ibase = pix * a.KK;
    int i0 = (t % TPM) / a.Kw, j0 = (t % TPM) - ((t % TPM) / a.Kw) * a.Kw;
#pragma unroll 1
    for (int tb = t % TPM; tb < a.KK; tb += TPM * STG_TAPS) {
        // inputs: every load unconditional (tap index clamped, rows past M read row 0's
        // pixel), validity applied afterwards -- no branches between the independent entries
        MetaIn in[STG_TAPS];
#pragma unroll
        for (int k = 0; k < STG_TAPS; ++k) {
            const int tk = min(tb + TPM * k, a.KK - 1);
            in[k].d = ld_offset2(a.offset, (ibase + tk) * 2, a.off_f16);
            in[k].mk = a.mask ? ld_mask1(a.mask, ibase + tk, a.off_f16) : 1.0f;
        }
        MetaVal v[STG_TAPS];
        int i = i0, j = j0;
#pragma unroll
        for (int k = 0; k < STG_TAPS; ++k) {
            v[k] = meta_value<ME == 16>(a, rp, i, j, in[k], tex_row);
            j += TPM;
            while (j >= a.Kw) {   // once per step for Kw >= TPM
                j -= a.Kw;
                ++i;
            }
        }
        i0 = i;
        j0 = j;
#pragma unroll
        for (int k = 0; k < STG_TAPS; ++k) {
            const int tk = tb + TPM * k;
            if (tk < a.KK) {
                *reinterpret_cast<uint4*>(rmeta + tk * ME) = v[k].lo;
                if (ME == 32 && !tex_row) *reinterpret_cast<uint4*>(rmeta + tk * ME + 16) = v[k].hi;
            }
        }
        if (t == 0) KT(18, g_kt_q);
    }
}

// Pull the offsets/mask of the tile a CTA processes next into L2 while the current one runs.
__device__ __forceinline__ void prefetch_meta_l2(const TcArgs& a, int m0, int t) {
    if (m0 < 0) return;
    const int rows = min(BM, a.M - m0);
    const size_t per_pix = (size_t)a.G * a.KK;
    const size_t es = a.off_f16 ? 2 : 4;
    const char* o0 = reinterpret_cast<const char*>(a.offset) + (size_t)m0 * per_pix * 2 * es;
    const int o_lines = (int)((rows * per_pix * 2 * es + 127) / 128);
    const char* k0 = a.mask ? reinterpret_cast<const char*>(a.mask) + (size_t)m0 * per_pix * es : nullptr;
    const int k_lines = a.mask ? (int)((rows * per_pix * es + 127) / 128) : 0;
    for (int l = t; l < o_lines + k_lines; l += NPT) {
        const char* p = l < o_lines ? o0 + (size_t)l * 128 : k0 + (size_t)(l - o_lines) * 128;
        asm volatile("prefetch.global.L2 [%0];" ::"l"(p));
    }
}

// The 4 corner vectors (8 channels each) of one A row and their weights.
struct RowLoad {
    U8x32 v[4];
    float4 w;
};
// bf16 x: the same, weights as two bf16 pairs (w0, w1), (w2, w3).
struct RowLoadB {
    U8x32 v[4];
    uint2 w;
};

// One 16-byte compact entry (store_meta_entry): corners 1 / 3 are corners 0 / 2 plus one pixel
// (pb bytes) when the entry's flag bit is set, else the same (weight-0) address.
__device__ __forceinline__ void issue_row_b(RowLoadB& L, const void* xbase, uint32_t meta_addr, uint32_t pb) {
    const uint4 e = ld_shared_v4(meta_addr);
    L.w = make_uint2(e.z, e.w);
    const uint32_t dx = (e.x & 1u) * pb;
    const uint32_t o0 = e.x & ~1u;
#ifdef DEFCON_PROBE_SAME_ADDR   // dev probe: every gather hits the same line (L1-resident)
    L.v[0] = ldg_nc_v8(xbase);
    L.v[1] = ldg_nc_v8(xbase);
    L.v[2] = ldg_nc_v8(xbase);
    L.v[3] = ldg_nc_v8(xbase);
    (void)dx; (void)o0;
#else
    L.v[0] = ldg_nc_v8(add_u32(xbase, o0));
    L.v[1] = ldg_nc_v8(add_u32(xbase, o0 + dx));
    L.v[2] = ldg_nc_v8(add_u32(xbase, e.y));
    L.v[3] = ldg_nc_v8(add_u32(xbase, e.y + dx));
#endif
}

// Eq.3 for 16 bf16 channels with bf16 weights: sum_q w_q * corner_q as mixed-precision FMAs
// (exact bf16 x bf16 products accumulated in fp32, FHFMA.BF16 -- the corners are used as
// stored, no unpack), RNE to bf16, into the two 16-byte swizzled slots of this thread's part
// of the A row.  Reading R20: the only rounding beyond the fp32 lerp is the weights' to bf16.
__device__ __forceinline__ void lerp_store_row_b(const RowLoadB& L, uint32_t dst_lo, uint32_t dst_hi) {
#ifdef DEFCON_PROBE_NO_MATH   // dev probe: no lerp, the 4 corners xor-ed (keeps every load live)
    uint32_t o[8];
#pragma unroll
    for (int h = 0; h < 8; ++h) o[h] = L.v[0].w[h] ^ L.v[1].w[h] ^ L.v[2].w[h] ^ L.v[3].w[h] ^ L.w.x;
    st_shared_v4(dst_lo, o[0], o[1], o[2], o[3]);
    st_shared_v4(dst_hi, o[4], o[5], o[6], o[7]);
    return;
#endif
    float acc[16];
    const uint32_t w01 = L.w.x, w23 = L.w.y;
#pragma unroll
    for (int h = 0; h < 8; ++h) {
        acc[2 * h] = fma_bf16h<0, 0>(L.v[0].w[h], w01, 0.f);
        acc[2 * h + 1] = fma_bf16h<1, 0>(L.v[0].w[h], w01, 0.f);
    }
#pragma unroll
    for (int h = 0; h < 8; ++h) {
        acc[2 * h] = fma_bf16h<0, 1>(L.v[1].w[h], w01, acc[2 * h]);
        acc[2 * h + 1] = fma_bf16h<1, 1>(L.v[1].w[h], w01, acc[2 * h + 1]);
    }
#pragma unroll
    for (int h = 0; h < 8; ++h) {
        acc[2 * h] = fma_bf16h<0, 0>(L.v[2].w[h], w23, acc[2 * h]);
        acc[2 * h + 1] = fma_bf16h<1, 0>(L.v[2].w[h], w23, acc[2 * h + 1]);
    }
#pragma unroll
    for (int h = 0; h < 8; ++h) {
        acc[2 * h] = fma_bf16h<0, 1>(L.v[3].w[h], w23, acc[2 * h]);
        acc[2 * h + 1] = fma_bf16h<1, 1>(L.v[3].w[h], w23, acc[2 * h + 1]);
    }
    st_shared_v4(dst_lo, pack_bf16x2(acc[0], acc[1]), pack_bf16x2(acc[2], acc[3]), pack_bf16x2(acc[4], acc[5]),
                 pack_bf16x2(acc[6], acc[7]));
    st_shared_v4(dst_hi, pack_bf16x2(acc[8], acc[9]), pack_bf16x2(acc[10], acc[11]),
                 pack_bf16x2(acc[12], acc[13]), pack_bf16x2(acc[14], acc[15]));
}

// fp32 x: the 4 corner vectors and fp32 weights of one 32-byte entry.
__device__ __forceinline__ void issue_row(RowLoad& L, const void* xbase, uint32_t meta_addr) {
    const uint4 o = ld_shared_v4(meta_addr);
    const uint4 wb = ld_shared_v4(meta_addr + 16);
    L.w = make_float4(__uint_as_float(wb.x), __uint_as_float(wb.y), __uint_as_float(wb.z),
                      __uint_as_float(wb.w));
    L.v[0] = ldg_nc_v8(add_u32(xbase, o.x));
    L.v[1] = ldg_nc_v8(add_u32(xbase, o.y));
    L.v[2] = ldg_nc_v8(add_u32(xbase, o.z));
    L.v[3] = ldg_nc_v8(add_u32(xbase, o.w));
}

// Texture-sampler counterpart of RowLoad: 16 channels = 4 texels of 4 channels, already
// bilinearly filtered by the texture unit, and the mask.
struct TexLoad {
    float4 t[4];
    float m;
};

__device__ __forceinline__ void issue_row_tex(TexLoad& L, cudaTextureObject_t tex, int layer,
                                              uint32_t meta_addr) {
    const uint4 c = ld_shared_v4(meta_addr);
    const float fx = __uint_as_float(c.x), fy = __uint_as_float(c.y);
    L.m = __uint_as_float(c.z);
#pragma unroll
    for (int i = 0; i < 4; ++i) L.t[i] = tex2DLayered<float4>(tex, fx, fy, layer + i);
}

__device__ __forceinline__ void tex_store_row(const TexLoad& L, uint32_t dst_lo, uint32_t dst_hi) {
    const float m = L.m;
    st_shared_v4(dst_lo, pack_bf16x2(L.t[0].x * m, L.t[0].y * m), pack_bf16x2(L.t[0].z * m, L.t[0].w * m),
                 pack_bf16x2(L.t[1].x * m, L.t[1].y * m), pack_bf16x2(L.t[1].z * m, L.t[1].w * m));
    st_shared_v4(dst_hi, pack_bf16x2(L.t[2].x * m, L.t[2].y * m), pack_bf16x2(L.t[2].z * m, L.t[2].w * m),
                 pack_bf16x2(L.t[3].x * m, L.t[3].y * m), pack_bf16x2(L.t[3].z * m, L.t[3].w * m));
}

// Sampler policy: LDG gathers + software lerp, or texture fetches with hardware filtering.
template <bool TEX>
struct Sampler;
template <>
struct Sampler<false> {
    using Load = RowLoadB;
    static __device__ __forceinline__ void issue(Load& L, const uint8_t* xb, unsigned long long, int,
                                                 uint32_t meta, uint32_t pb) {
        issue_row_b(L, xb, meta, pb);
    }
    static __device__ __forceinline__ void store(const Load& L, uint32_t lo, uint32_t hi) {
        lerp_store_row_b(L, lo, hi);
    }
};
template <>
struct Sampler<true> {
    using Load = TexLoad;
    static __device__ __forceinline__ void issue(Load& L, const uint8_t*, unsigned long long tex, int layer,
                                                 uint32_t meta, uint32_t) {
        issue_row_tex(L, (cudaTextureObject_t)tex, layer, meta);
    }
    static __device__ __forceinline__ void store(const Load& L, uint32_t lo, uint32_t hi) {
        tex_store_row(L, lo, hi);
    }
};

// fp32 x (3xTF32 path): the 4 corner vectors of 8 channels, fp32 bilinear sum (packed FFMA2,
// no widening), then the tf32 split written to the two A planes: hi = v with the low 13
// mantissa bits cleared, lo = v - hi (both exact; the MMAs take lo*hi + hi*lo + hi*hi).
__device__ __forceinline__ void lerp_store_row_f32(const RowLoad& L, uint32_t d0, uint32_t d1) {
    uint64_t acc[4];
    const float wq[4] = {L.w.x, L.w.y, L.w.z, L.w.w};
#pragma unroll
    for (int q = 0; q < 4; ++q) {
        const uint64_t w2 = f32x2_pack(wq[q], wq[q]);
#pragma unroll
        for (int h = 0; h < 4; ++h) {
            const uint64_t c = ((uint64_t)L.v[q].w[2 * h + 1] << 32) | L.v[q].w[2 * h];
            acc[h] = q == 0 ? f32x2_mul(c, w2) : f32x2_fma(c, w2, acc[h]);
        }
    }
    uint32_t hi[8], lo[8];
#pragma unroll
    for (int h = 0; h < 4; ++h) {
        const float v0 = __uint_as_float((uint32_t)(acc[h] & 0xFFFFFFFFull));
        const float v1 = __uint_as_float((uint32_t)(acc[h] >> 32));
        hi[2 * h] = __float_as_uint(v0) & 0xFFFFE000u;
        hi[2 * h + 1] = __float_as_uint(v1) & 0xFFFFE000u;
        lo[2 * h] = __float_as_uint(v0 - __uint_as_float(hi[2 * h]));
        lo[2 * h + 1] = __float_as_uint(v1 - __uint_as_float(hi[2 * h + 1]));
    }
    st_shared_v4(d0, hi[0], hi[1], hi[2], hi[3]);
    st_shared_v4(d1, hi[4], hi[5], hi[6], hi[7]);
    st_shared_v4(d0 + A_PLANE, lo[0], lo[1], lo[2], lo[3]);
    st_shared_v4(d1 + A_PLANE, lo[4], lo[5], lo[6], lo[7]);
}

struct SamplerF32 {
    using Load = RowLoad;
    static __device__ __forceinline__ void issue(Load& L, const uint8_t* xb, unsigned long long, int,
                                                 uint32_t meta, uint32_t) {
        issue_row(L, xb, meta);
    }
    static __device__ __forceinline__ void store(const Load& L, uint32_t lo, uint32_t hi) {
        lerp_store_row_f32(L, lo, hi);
    }
};

// CTA range -> segments helper (every role walks the same sequence).
__device__ __forceinline__ int count_segments(const TcArgs& a, long long it_begin, long long it_end) {
    if (it_end <= it_begin) return 0;
    return (int)((it_end - 1) / a.ipt - it_begin / a.ipt) + 1;
}

__device__ __forceinline__ Segment segment_j(const TcArgs& a, long long it_begin, long long it_end, int j) {
    Segment sg;
    sg.tile = (int)(it_begin / a.ipt) + j;
    const long long t0 = (long long)sg.tile * a.ipt;
    sg.kb = (int)(max(it_begin, t0) - t0);
    sg.ke = (int)(min(it_end, t0 + a.ipt) - t0);
    return sg;
}

// Processing order of a CTA's segments: the last one (the head of a tile whose remaining
// k-iterations belong to later CTAs) first, so its partial is published early; then the
// rest in order.  The tail segment of a split tile -- its "owner", which holds the tile's
// last k-iteration -- is then processed while the other contributors' partials are
// already in L2.
__device__ __forceinline__ int seg_order(int o, int nseg) {
    if (nseg <= 1) return o;
    return o == 0 ? nseg - 1 : o - 1;
}

__device__ __forceinline__ int ld_acquire_gpu(const int* p) {
    int v;
    asm volatile("ld.acquire.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

// Epilogue of one segment for NCOLS columns [col0, col0 + NCOLS) of row r (= TMEM lane).
// Whole tile: + bias -> bf16 -> y.  Split tile (stream-K): non-owner contributors publish an
// fp32 partial (slot = CTA index) and count themselves on the tile counter.  The owner, if
// every other contributor has arrived (the normal case, see seg_order), adds the partials in
// k order to its own TMEM accumulator and writes y; otherwise it publishes its accumulator too
// (slot = grid + CTA) and whoever arrives last sums all partials.  Fixed summation order in
// both cases: contributors by ascending k range, owner last -> deterministic.
// Output tile store: every warp owns 32 rows (its TMEM lane quarter); a group of CS = 32
// columns is packed to bf16, written to a 2 KB warp-private shared buffer in the 64-byte
// swizzled layout (conflict-free) and stored by one TMA bulk-tensor store (rows >= M and
// columns >= Cout are clipped by the TMA unit).  Two buffers alternate per warp.
constexpr int CS = 32;
#ifndef DEFCON_F32_EPI_NB
#define DEFCON_F32_EPI_NB 1   // fp32 y: one 4 KB scratch buffer per warp (the 3xTF32 kernel under the carveout cliff)
#endif
constexpr int EPI_SCRATCH_PER_WARP = 2 * 2048;   // bf16: two 2 KB buffers (32 rows x 64 B)
// fp32 y: two 4 KB buffers per warp (32 rows x 128 B, 128-byte swizzle)
// BLOCK_N = 512 (bf16): one 2 KB buffer per warp -- its 2-stage pipeline then stays under the
// shared-memory carveout step that would leave the gathers no L1 (C5 66.5 -> 64.9 us; DESIGN
// 12b item 15)
template <bool F32, int BLOCK_N = 256>
__host__ __device__ constexpr int epi_scratch_per_warp() {
    return F32 ? DEFCON_F32_EPI_NB * 4096 : BLOCK_N >= 512 ? EPI_SCRATCH_PER_WARP / 2 : EPI_SCRATCH_PER_WARP;
}

template <int NB = 2>   // 2 KB scratch buffers per warp
__device__ __forceinline__ void store_group_tma(const CUtensorMap* ymap, uint8_t* scratch, int gi,
                                                const uint32_t (&pk)[CS / 2], int col, int row0,
                                                int lane) {
    uint8_t* buf = scratch + (gi % NB) * 2048;
    if (gi >= NB) {                        // the store that used this buffer has read it
        if (lane == 0) bulk_wait_read<NB - 1>();
        __syncwarp();
    }
    const uint32_t base = smem_u32(buf) + lane * 64;
#pragma unroll
    for (int cc = 0; cc < 4; ++cc)
        st_shared_v4(base + ((cc ^ ((lane >> 1) & 3)) << 4), pk[4 * cc], pk[4 * cc + 1], pk[4 * cc + 2],
                     pk[4 * cc + 3]);
    fence_proxy_async_smem();
    __syncwarp();
    if (lane == 0) {
        tma_store_2d(ymap, buf, col, row0);
        bulk_commit();
    }
}

// fp32 y: 32 columns of this lane's row (128 B) into a 4 KB buffer in the 128-byte swizzled
// layout (16-byte unit c of row r at c ^ (r % 8)), stored by one 32 x 32 TMA box.
template <int NB = 2>   // 4 KB scratch buffers per warp
__device__ __forceinline__ void store_group_tma_f32(const CUtensorMap* ymap, uint8_t* scratch, int gi,
                                                    const float (&v)[CS], int col, int row0, int lane) {
    uint8_t* buf = scratch + (gi % NB) * 4096;
    if (gi >= NB) {
        if (lane == 0) bulk_wait_read<NB - 1>();
        __syncwarp();
    }
    const uint32_t base = smem_u32(buf) + lane * 128;
#pragma unroll
    for (int cc = 0; cc < 8; ++cc)
        st_shared_v4(base + ((cc ^ (lane & 7)) << 4), __float_as_uint(v[4 * cc]), __float_as_uint(v[4 * cc + 1]),
                     __float_as_uint(v[4 * cc + 2]), __float_as_uint(v[4 * cc + 3]));
    fence_proxy_async_smem();
    __syncwarp();
    if (lane == 0) {
        tma_store_2d(ymap, buf, col, row0);
        bulk_commit();
    }
}

template <int BLOCK_N, int NCOLS, bool PAIR, bool F32>
__device__ __forceinline__ void epilogue_segment(const TcArgs& a, const CUtensorMap* ymap, const Segment& sg,
                                                 uint32_t tacc, int r, int col0, int bar_id, int nthr,
                                                 bool leader, int* fix_flag, long long T, int nct,
                                                 const float* bias_s, uint8_t* scratch,
                                                 uint8_t* stage_smem = nullptr, size_t stage_bytes = 0,
                                                 int sid = 0) {
    constexpr int CH = 16;     // columns per partial write
    const int lane = threadIdx.x & 31;
    const int m0 = tile_m0<PAIR>(a, sg.tile);
    const int n0 = (sg.tile % a.n_tiles_n) * BLOCK_N;
    // pair mode: contributors are CTA pairs; this CTA's half of a tile has its own counter and
    // partial slots (slot of unit b = 2b + rank, i.e. the contributing CTA's index)
    const int rk = PAIR ? (int)cluster_ctarank() : 0;
    const int ctr = PAIR ? 2 * sg.tile + rk : sg.tile;
    auto slot_of = [&](int b) { return PAIR ? 2 * b + rk : b; };
    const int row = m0 + r;
    const int row0 = m0 + (r & ~31);
    const bool row_ok = row < a.M;
    const bool owner = sg.ke == a.ipt;
    const long long t0 = (long long)sg.tile * a.ipt;
    const int b_lo = cta_of(T, nct, t0);
    const int b_hi = cta_of(T, nct, t0 + a.ipt - 1);      // == owner CTA
    const int ncontrib = b_hi - b_lo;                    // contributors other than the owner
    const size_t slot_elems = (size_t)BLOCK_N * BM;
    const float4* parts = reinterpret_cast<const float4*>(a.partials);

    auto write_partial = [&](int slot) {
        float4* dst = reinterpret_cast<float4*>(a.partials + (size_t)slot * slot_elems);
#pragma unroll 1
        for (int c = col0; c < col0 + NCOLS; c += CH) {
            uint32_t v[CH];
            tmem_ld_32x32b_x16(tacc + c, v);
            if (F32) {   // + the cross-term accumulator
                uint32_t vx[CH];
                tmem_ld_32x32b_x16(tacc + BLOCK_N + c, vx);
                tmem_ld_wait();
#pragma unroll
                for (int u = 0; u < CH; ++u) v[u] = __float_as_uint(__uint_as_float(v[u]) + __uint_as_float(vx[u]));
            }
            tmem_ld_wait();
#pragma unroll
            for (int u = 0; u < CH / 4; ++u)
                __stcg(dst + (size_t)((c >> 2) + u) * BM + r,
                       make_float4(__uint_as_float(v[4 * u]), __uint_as_float(v[4 * u + 1]),
                                   __uint_as_float(v[4 * u + 2]), __uint_as_float(v[4 * u + 3])));
        }
        __threadfence();
    };
    // y = bias + sum(partials of contributors b_lo..b_hi-1) [+ own accumulator | owner slot],
    // in this fixed order whichever path runs, CS columns at a time.  With `st` the partial
    // float4s come from this thread's shared-memory staging slots (finish_staged: slot of
    // slab j, float4 u at st + (j * spj + u) * st_stride), else from L2.
    auto sum_group = [&](bool own_from_tmem, int c, int gi, const uint8_t* st, int st_stride, int spj,
                         int cbase) {
        uint32_t v[CS];
        if (own_from_tmem) {
            tmem_ld_32x32b_x32(tacc + c, v);
            if (F32) {   // + the cross-term accumulator
                uint32_t vx[CS];
                tmem_ld_32x32b_x32(tacc + BLOCK_N + c, vx);
                tmem_ld_wait();
#pragma unroll
                for (int u = 0; u < CS; ++u) v[u] = __float_as_uint(__uint_as_float(v[u]) + __uint_as_float(vx[u]));
            }
            tmem_ld_wait();
        }
        if (n0 + c >= a.Cout) return;      // warp-uniform
        const int nslab = (b_hi - b_lo) + (own_from_tmem ? 0 : 1);
        float acc[CS];
#pragma unroll
        for (int u = 0; u < CS; ++u) acc[u] = 0.f;
        if (row_ok) {
#pragma unroll 1
            for (int j = 0; j < nslab; ++j) {
                const int slot = b_lo + j < b_hi ? slot_of(b_lo + j) : (int)gridDim.x + slot_of(b_hi);
                float4 f[CS / 4];
#pragma unroll
                for (int u = 0; u < CS / 4; ++u)
                    f[u] = st ? *reinterpret_cast<const float4*>(st + (size_t)(j * spj + ((c - cbase) >> 2) + u) * st_stride)
                              : __ldcg(parts + (size_t)slot * (slot_elems / 4) + (size_t)((c >> 2) + u) * BM + r);
#pragma unroll
                for (int u = 0; u < CS / 4; ++u) {
                    acc[4 * u] += f[u].x; acc[4 * u + 1] += f[u].y;
                    acc[4 * u + 2] += f[u].z; acc[4 * u + 3] += f[u].w;
                }
            }
        }
        if (own_from_tmem) {
#pragma unroll
            for (int u = 0; u < CS; ++u) acc[u] += __uint_as_float(v[u]);
        }
#pragma unroll
        for (int u = 0; u < CS / 4; ++u) {
            const int co = n0 + c + 4 * u;
            float4 bb = make_float4(0.f, 0.f, 0.f, 0.f);
            if (bias_s) bb = *reinterpret_cast<const float4*>(bias_s + co);     // broadcast
            else if (a.bias && co < a.Cout) bb = __ldg(reinterpret_cast<const float4*>(a.bias + co));
            acc[4 * u] += bb.x; acc[4 * u + 1] += bb.y; acc[4 * u + 2] += bb.z; acc[4 * u + 3] += bb.w;
        }
        if (F32) {
            store_group_tma_f32<DEFCON_F32_EPI_NB>(ymap, scratch, gi, acc, n0 + c, row0, lane);
        } else {
            uint32_t pk[CS / 2];
#pragma unroll
            for (int u = 0; u < CS / 2; ++u) pk[u] = pack_bf16x2(acc[2 * u], acc[2 * u + 1]);
            store_group_tma<BLOCK_N >= 512 ? 1 : 2>(ymap, scratch, gi, pk, n0 + c, row0, lane);
        }
    };
    auto drain = [&]() {
        if (lane == 0) bulk_wait_all();
        __syncwarp();
    };
    auto finish = [&](bool own_from_tmem) {
        int gi = 0;
#pragma unroll 1
        for (int c = col0; c < col0 + NCOLS; c += CS, ++gi) sum_group(own_from_tmem, c, gi, nullptr, 0, 0, 0);
        drain();
    };
    // Staged variant (the producer-run last epilogue, when the pipeline's B stage buffers are
    // idle): the partial float4s of a pass of `pwc` columns are copied to shared memory with
    // cp.async first -- all in flight at once, no registers held -- so each pass costs about
    // one L2 round trip.  Thread `sid` of `nthr` owns slot sid of each float4 row.
    const int nslab_fast = b_hi - b_lo;
    int pwc = NCOLS;
    while (pwc > CS && (size_t)nslab_fast * (pwc / 4) * nthr * 16 > stage_bytes) pwc >>= 1;
    auto finish_staged = [&](uint8_t* st) {
        int gi = 0;
#pragma unroll 1
        for (int p0 = col0; p0 < col0 + NCOLS; p0 += pwc) {
            if (row_ok) {
                for (int j = 0; j < nslab_fast; ++j) {
                    const float4* src = parts + (size_t)slot_of(b_lo + j) * (slot_elems / 4) + (size_t)(p0 >> 2) * BM + r;
#pragma unroll 4
                    for (int u = 0; u < pwc / 4; ++u)
                        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(
                                         st + (size_t)((j * (pwc / 4) + u) * nthr + sid) * 16)),
                                     "l"(src + (size_t)u * BM)
                                     : "memory");
                }
                asm volatile("cp.async.commit_group;\n\tcp.async.wait_group 0;" ::: "memory");
            }
            if (sid == 0) TL(7);
#pragma unroll 1
            for (int c = p0; c < p0 + pwc; c += CS, ++gi)
                sum_group(true, c, gi, st + (size_t)sid * 16, nthr * 16, pwc / 4, p0);
        }
        drain();
    };
    const bool staged = stage_smem != nullptr && (size_t)nslab_fast * (pwc / 4) * nthr * 16 <= stage_bytes;

    if (owner && ncontrib == 0) {          // whole tile
        finish(true);
        return;
    }
    // The party that finishes a split tile resets its counter to 0, so the workspace is
    // zero again after every launch (no per-call memset; see defcon_dcn_forward).
    if (!owner) {                          // non-owner contributor: publish, count
        write_partial(blockIdx.x);
        named_bar_sync(bar_id, nthr);
        if (leader) *fix_flag = (atomicAdd(a.counters + ctr, 1) == ncontrib) ? 1 : 0;
        named_bar_sync(bar_id, nthr);
        const bool last = *fix_flag != 0;
        named_bar_sync(bar_id, nthr);      // fix_flag reused by the next segment
        if (last) {                        // owner took the slow path: finish from partials
            __threadfence();
            finish(false);
            if (leader) a.counters[ctr] = 0;
        }
        return;
    }
    // owner of a split tile
    if (leader) *fix_flag = (ld_acquire_gpu(a.counters + ctr) == ncontrib) ? 1 : 0;
    named_bar_sync(bar_id, nthr);
    const bool all_in = *fix_flag != 0;
    named_bar_sync(bar_id, nthr);
#ifndef DEFCON_PROBE_TL_META
    if (leader && stage_smem) TL(all_in ? 6 : 9);
#endif
    if (all_in) {                          // fast path: partials + own TMEM accumulator
        if (staged) finish_staged(stage_smem);
        else finish(true);
        if (leader) a.counters[ctr] = 0;
        if (leader && stage_smem) TL(8);
        return;
    }
    write_partial((int)gridDim.x + blockIdx.x);   // slow path: publish own accumulator as well
    named_bar_sync(bar_id, nthr);
    if (leader) *fix_flag = (atomicAdd(a.counters + ctr, 1) == ncontrib) ? 1 : 0;
    named_bar_sync(bar_id, nthr);
    const bool last = *fix_flag != 0;
    named_bar_sync(bar_id, nthr);
    if (last) {
        __threadfence();
        finish(false);
        if (leader) a.counters[ctr] = 0;
    }
}

// One producer warp's share of one segment: for every k-iteration, 2 A rows x 32 bytes per
// thread (one 256-bit gather per corner), with the next k-iteration's gathers (or texture fetches) issued row by row as
// soon as the row's registers are free (rolling prefetch).  Warps with TEXW use the texture
// sampler, the others LDG gathers + software lerp; the metadata table holds each row in the
// format its warp consumes (warp of row r = (r mod 64) / 8).
template <bool TEXW, int STAGES, int NTEX, bool PAIR, bool F32>
__device__ __forceinline__ void produce_segment(const TcArgs& a, const Segment& sg, int& q, uint8_t* meta,
                                                const uint32_t (&dst_lo)[ROWS], const uint32_t (&dst_hi)[ROWS],
                                                const uint32_t (&mrow)[ROWS], uint32_t a_s, uint64_t* empty,
                                                uint64_t* full_a, int t, int sub, int lane, int next_m0) {
    using Smp = typename std::conditional<F32, SamplerF32, Sampler<TEXW>>::type;
    using E = Elem<F32>;
    constexpr int ME = meta_entry<F32>();
    const uint32_t pb = (uint32_t)(a.Cin * a.es);   // bytes per x pixel
    const int m0 = tile_m0<PAIR>(a, sg.tile);
    int chunk = sg.kb / a.KK;
    int tap = sg.kb - chunk * a.KK;
    int g = (chunk * E::CPI) / a.Cg;
#ifdef DEFCON_PROBE_KTRACE
    if (t == 0) g_kt_q = q;
#endif
    if (t == 0) KT(12, q);
    named_bar_sync(1, NPT);          // previous table no longer read
#ifdef DEFCON_PROBE_TL_META
    if (t == 0) TL(9);
#endif
    if (t == 0) KT(13, q);
#ifdef DEFCON_PROBE_BUILD_TWICE   // dev probe: a second, warm build of the same table
    build_meta_table<NTEX, ME>(a, m0, g, meta, t, 0u);
    if (t == 0) KT(23, q);
#endif
    build_meta_table<NTEX, ME>(a, m0, g, meta, t);
    if (t == 0) KT(14, q);
    named_bar_sync(1, NPT);
    if (t == 0) KT(15, q);
    prefetch_meta_l2(a, next_m0, t);
    if (t == 0) TL(10 + (q ? 1 : 0));     // metadata table ready (first / later segment)
    // position of this thread's 16 channels: byte pointer (LDG) / texture layer (TEX)
    const uint8_t* xb = reinterpret_cast<const uint8_t*>(a.x) + 128 * chunk + 32 * sub;
    int layer = chunk * (BK / 4) + sub * 4;
    typename Smp::Load L[ROWS];
#pragma unroll
    for (int p = 0; p < ROWS; ++p) Smp::issue(L[p], xb, a.tex, layer, mrow[p] + tap * ME, pb);
    for (int kt = sg.kb; kt < sg.ke; ++kt, ++q) {
        int ntap = tap + 1, nchunk = chunk;
        if (ntap == a.KK) { ntap = 0; ++nchunk; }
        const bool has_next = kt + 1 < sg.ke;
        int ng = g;
        if (has_next && nchunk != chunk) ng = (nchunk * E::CPI) / a.Cg;
        const bool prefetch = has_next && ng == g;
        const uint8_t* nxb = nchunk != chunk ? xb + 128 : xb;
        const int nlayer = nchunk != chunk ? layer + BK / 4 : layer;

        const int s = q % STAGES;
        if (t == 0) KT(0, q);
        mbar_wait(&empty[s], ((uint32_t)(q / STAGES) & 1u) ^ 1u);
        if (t == 0) KT(1, q);
        const uint32_t stage = a_s + s * E::A_STAGE;
#pragma unroll
        for (int p = 0; p < ROWS; ++p) {    // rolling prefetch of the next k-iteration
            Smp::store(L[p], stage + dst_lo[p], stage + dst_hi[p]);
            if (t == 0) KT(8 + p, q);
            // the last row's gathers go out after the arrive: the proxy fence below lowers to
            // MEMBAR.ALL.CTA, which waits for this thread's outstanding loads
            if (prefetch && (DEFCON_LATE_LAST == 0 || (DEFCON_LATE_LAST == 1 && p + 1 < ROWS)))
                Smp::issue(L[p], nxb, a.tex, nlayer, mrow[p] + ntap * ME, pb);
        }
#ifdef DEFCON_PROBE_NO_FENCE   // dev probe (WRONG results): no proxy fence, relaxed arrive -- the
                               // cost of ordering the A stores before the MMA
        __syncwarp();
        if (lane == 0)
            asm volatile("mbarrier.arrive.relaxed.cta.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&full_a[s])) : "memory");
#else
        fence_proxy_async_smem();
        if (t == 0) KT(10, q);
        __syncwarp();
        if (lane == 0) {
            if (PAIR) mbar_arrive_cluster(&full_a[s], 0);   // the pair's MMA issuer is rank 0
            else mbar_arrive(&full_a[s]);
        }
#endif
        if (t == 0) KT(2, q);
        if (t == 224) KT(7, q);   // the last producer warp
        if (DEFCON_LATE_LAST && prefetch) {
#pragma unroll
            for (int p = DEFCON_LATE_LAST == 1 ? ROWS - 1 : 0; p < ROWS; ++p)
                Smp::issue(L[p], nxb, a.tex, nlayer, mrow[p] + ntap * ME, pb);
        }

        if (has_next && !prefetch) {          // offset group changes: new table
#ifndef DEFCON_PROBE_NO_REBUILD   // dev probe (WRONG results for G > 1): keep the first table
            named_bar_sync(1, NPT);
            build_meta_table<NTEX, ME>(a, m0, ng, meta, t);
            named_bar_sync(1, NPT);
#endif
            g = ng;
#pragma unroll
            for (int p = 0; p < ROWS; ++p) Smp::issue(L[p], nxb, a.tex, nlayer, mrow[p] + ntap * ME, pb);
        }
        layer = nlayer;
        tap = ntap;
        chunk = nchunk;
        xb = nxb;
    }
}

// F32: fp32 x / W / y on kind::tf32 with the 3xTF32 split (wmap = W hi plane, wmap_lo = W lo
// plane, both prepared by dcn_w_split_kernel); otherwise bf16 on kind::f16 (wmap_lo unused).
template <int BLOCK_N, int STAGES, int NTEX, bool PAIR, bool F32>
__global__ void __launch_bounds__(NUM_THREADS, 1)
    dcn_fwd_bf16_tc_kernel(const __grid_constant__ CUtensorMap wmap, const __grid_constant__ CUtensorMap wmap_lo,
                           const __grid_constant__ CUtensorMap ymap, const TcArgs a) {
    using Cfg = TcCfg<BLOCK_N, PAIR, F32>;
    constexpr int EPI_W = epi_scratch_per_warp<F32, BLOCK_N>();

    extern __shared__ __align__(1024) uint8_t smem_raw[];
    uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                               ~uintptr_t(1023));
    uint8_t* sA = smem;
    uint8_t* sB = smem + STAGES * Cfg::A_STAGE_BYTES;
    uint8_t* epi_scratch = sB + STAGES * Cfg::B_STAGE_BYTES;   // 4 epilogue warps x EPI_W
    uint8_t* meta = epi_scratch + 4 * EPI_W;
    uint64_t* bars = reinterpret_cast<uint64_t*>(meta + BM * a.KK * meta_entry<F32>());
    uint64_t* full_a = bars;
    // single CTAs: the producers' arrivals and the weight TMA's transaction bytes complete ONE
    // barrier per stage (NPW + 1 arrivals), so the MMA issuer waits once per k-iteration
#ifndef DEFCON_SPLIT_FULL
    constexpr bool MERGED = !PAIR;
#else
    constexpr bool MERGED = false;
#endif
    uint64_t* full_b = MERGED ? bars : bars + STAGES;
    uint64_t* empty = bars + 2 * STAGES;
    uint64_t* tmem_full = bars + 3 * STAGES;
    uint64_t* tmem_empty = tmem_full + Cfg::NBUF;
    uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tmem_empty + Cfg::NBUF);
    int* fix_flag = reinterpret_cast<int*>(tmem_slot + 1);     // [0] epilogue, [1] producers
    float* bias_s = reinterpret_cast<float*>(reinterpret_cast<uint8_t*>(bars) +
                                             bias_smem_offset(STAGES, Cfg::NBUF));

    const int warp = threadIdx.x >> 5;
    const int lane = threadIdx.x & 31;
    const long long T = a.total_iters;
    // stream-K units: CTAs, or CTA pairs (both CTAs of a pair walk the same range)
    const int rank = PAIR ? (int)cluster_ctarank() : 0;
    const int nct = PAIR ? (int)gridDim.x / 2 : (int)gridDim.x;
    const int unit = PAIR ? (int)blockIdx.x / 2 : (int)blockIdx.x;
    const long long it_begin = range_begin(T, nct, unit);
    const long long it_end = range_begin(T, nct, unit + 1);
    const int nseg = count_segments(a, it_begin, it_end);
    if (threadIdx.x == 0) TL(0);

    if (warp == TMA_WARP && lane == 0) {
        for (int s = 0; s < STAGES; ++s) {
            mbar_init(&full_a[s], PAIR ? 2 * NPW : MERGED ? NPW + 1 : NPW);   // pair: both CTAs' producers
            if (!MERGED) mbar_init(&full_b[s], 1);
            mbar_init(&empty[s], 1);
        }
        for (int b = 0; b < Cfg::NBUF; ++b) {
            mbar_init(&tmem_full[b], 1);
            mbar_init(&tmem_empty[b], PAIR ? 8 : 4);       // pair: both CTAs' epilogue warps
        }
        fence_barrier_init();
        tma_prefetch_desc(&wmap);
        if (F32) tma_prefetch_desc(&wmap_lo);
        tma_prefetch_desc(&ymap);
    }
    if (warp == MMA_WARP) {
        if (PAIR) tmem_alloc_pair<Cfg::TMEM_COLS>(tmem_slot);
        else tmem_alloc<Cfg::TMEM_COLS>(tmem_slot);
    }
    // Everything above overlaps the previous kernel's tail (PDL); inputs are read and
    // outputs / workspace written only after it has completed.
    griddep_wait();
    griddep_launch_dependents();
    if (a.bias_in_smem)
        for (int i = threadIdx.x; i < a.Cout; i += NUM_THREADS) bias_s[i] = a.bias ? __ldg(a.bias + i) : 0.f;
    tc_fence_before();
    __syncthreads();
    if (PAIR) cluster_sync_all();      // the peer's barriers are initialised before any remote arrive
    tc_fence_after();
    const uint32_t tmem_base = *tmem_slot;
    if (threadIdx.x == 0) TL(1);

    if (warp < NPW) {
        // ===================== A producers =====================
        const int t = threadIdx.x;
        const int sub = t & (TPR - 1);       // 32-byte quarter of the 128-byte row
        const uint32_t meta_s = smem_u32(meta);
        const uint32_t a_s = smem_u32(sA);
        uint32_t dst_lo[ROWS], dst_hi[ROWS], mrow[ROWS];
#pragma unroll
        for (int p = 0; p < ROWS; ++p) {
            const int row = (t / TPR) + p * (NPT / TPR);
            dst_lo[p] = row * 128 + (((2 * sub) ^ (row & 7)) << 4);
            dst_hi[p] = row * 128 + (((2 * sub + 1) ^ (row & 7)) << 4);
            mrow[p] = meta_s + row * a.KK * meta_entry<F32>();
        }
        int q = 0;                           // running k-iteration (stage) counter
        for (int o = 0; o < nseg; ++o) {
            const Segment sg = segment_j(a, it_begin, it_end, seg_order(o, nseg));
            const int next_m0 = o + 1 < nseg
                ? tile_m0<PAIR>(a, segment_j(a, it_begin, it_end, seg_order(o + 1, nseg)).tile) : -1;
            if (t == 0 && o < 4) TL(2 + 2 * o);
            if (warp < NTEX)
                produce_segment<true, STAGES, NTEX, PAIR, F32>(a, sg, q, meta, dst_lo, dst_hi, mrow, a_s, empty,
                                                               full_a, t, sub, lane, next_m0);
            else
                produce_segment<false, STAGES, NTEX, PAIR, F32>(a, sg, q, meta, dst_lo, dst_hi, mrow, a_s, empty,
                                                                full_a, t, sub, lane, next_m0);
            if (t == 0 && o < 4) TL(3 + 2 * o);
        }
        // The producers (4 lane quarters x NPW/4 column slices) run the last processed
        // segment's epilogue, which would otherwise be exposed at the end of the CTA's range.
        // Its store scratch reuses the A stages other producer threads wrote: ordered already
        // through full_a -> MMA -> tmem_full, a barrier the race checker can see makes it explicit.
        named_bar_sync(1, NPT);
        if (nseg > 0 && warp < FEPI_WARPS) {
            const int o = nseg - 1;
            const Segment sg = segment_j(a, it_begin, it_end, seg_order(o, nseg));
            const int buf = o % Cfg::NBUF;
            mbar_wait(&tmem_full[buf], (uint32_t)(o / Cfg::NBUF) & 1u);
            tc_fence_after();
            const int qd = warp & 3;
            const int r = qd * 32 + lane;
            const uint32_t tacc = tmem_base + ((uint32_t)(qd * 32) << 16) + (uint32_t)(buf * Cfg::ACC_STRIDE);
            constexpr int SLICE = BLOCK_N / (FEPI_WARPS / 4);
            if (t == 0) TL(12);
            // idle pipeline buffers: the per-warp store scratch and the staged stream-K partials.
            // Single CTAs: warps 0-3 take the epilogue warps' scratch (free once those have
            // released the accumulator of the CTA's previous segment), warps 4-7 the start of
            // the A stages, and the partials get everything behind that (A + B stages, one pass
            // at BLOCK_N = 256); pairs: A stages for the scratch, B stages for the partials.
            uint8_t* fscr = sA + warp * EPI_W;
            uint8_t* fstg = sB;
            size_t fstg_bytes = (size_t)STAGES * Cfg::B_STAGE_BYTES;
#ifndef DEFCON_FINAL_STAGE_B_ONLY
            if (!PAIR && STAGES * Cfg::A_STAGE_BYTES >= 4 * EPI_W) {
                if (nseg >= 2) {
                    const int op = nseg - 2;
                    mbar_wait(&tmem_empty[op % Cfg::NBUF], (uint32_t)(op / Cfg::NBUF) & 1u);
                }
                fscr = warp < 4 ? epi_scratch + warp * EPI_W : sA + (warp - 4) * EPI_W;
                fstg = sA + 4 * EPI_W;
                fstg_bytes = (size_t)STAGES * Cfg::A_STAGE_BYTES - 4 * EPI_W + (size_t)STAGES * Cfg::B_STAGE_BYTES;
            }
#endif
            epilogue_segment<BLOCK_N, SLICE, PAIR, F32>(a, &ymap, sg, tacc, r, (warp >> 2) * SLICE, 4,
                                                  FEPI_WARPS * 32,
                                                  t == 0, fix_flag + 1, T, nct, a.bias_in_smem ? bias_s : nullptr,
                                                  fscr, fstg, fstg_bytes, t);
            if (t == 0) TL(13);
        }
    } else if (warp < EPI_WARP0 + 4) {
        // ===================== epilogue (all processed segments but the last) ============
        const int qd = warp & 3;                    // TMEM lane quarter of this warp
        const int r = qd * 32 + lane;               // row within the tile (= TMEM lane)
        for (int o = 0; o + 1 < nseg; ++o) {
            const Segment sg = segment_j(a, it_begin, it_end, seg_order(o, nseg));
            const int buf = o % Cfg::NBUF;
            mbar_wait(&tmem_full[buf], (uint32_t)(o / Cfg::NBUF) & 1u);
            tc_fence_after();
            const uint32_t tacc = tmem_base + ((uint32_t)(qd * 32) << 16) + (uint32_t)(buf * Cfg::ACC_STRIDE);
            epilogue_segment<BLOCK_N, BLOCK_N, PAIR, F32>(a, &ymap, sg, tacc, r, 0, 2, 128,
                                                    threadIdx.x == EPI_WARP0 * 32, fix_flag, T, nct,
                                                    a.bias_in_smem ? bias_s : nullptr,
                                                    epi_scratch + (warp - EPI_WARP0) * EPI_W);
            tc_fence_before();
            __syncwarp();
            if (lane == 0) {
                if (PAIR) mbar_arrive_cluster(&tmem_empty[buf], 0);
                else mbar_arrive(&tmem_empty[buf]);
            }
        }
    } else if (warp == TMA_WARP) {
        // ===================== TMA producer (weights) =====================
        if (lane == 0) {
            int q = 0;
            for (int o = 0; o < nseg; ++o) {
                const Segment sg = segment_j(a, it_begin, it_end, seg_order(o, nseg));
                const int n0 = (sg.tile % a.n_tiles_n) * BLOCK_N;
                int chunk = sg.kb / a.KK;
                int tap = sg.kb - chunk * a.KK;
                for (int kt = sg.kb; kt < sg.ke; ++kt, ++q) {
                    const int s = q % STAGES;
                    mbar_wait(&empty[s], ((uint32_t)(q / STAGES) & 1u) ^ 1u);
#ifdef DEFCON_PROBE_NO_B   // dev probe: weights never reloaded (stale smem B)
                    mbar_arrive(&full_b[s]);
                    (void)n0;
#else
                    const int kd = tap * a.Cin + chunk * Elem<F32>::CPI;
                    if (PAIR) {   // this CTA's half of B; both halves complete on rank 0's barrier
                        if (rank == 0) mbar_arrive_expect_tx(&full_b[s], 2 * Cfg::B_STAGE_BYTES);
                        tma_load_2d_pair(sB + s * Cfg::B_STAGE_BYTES, &wmap, &full_b[s], kd,
                                         n0 + rank * Cfg::B_ROWS);
                    } else {
                        mbar_arrive_expect_tx(&full_b[s], Cfg::B_STAGE_BYTES);
#pragma unroll
                        for (int h = 0; h < BLOCK_N / Cfg::TMA_BOX_N; ++h) {
                            tma_load_2d(sB + s * Cfg::B_STAGE_BYTES + h * Cfg::TMA_BOX_N * 128, &wmap,
                                        &full_b[s], kd, n0 + h * Cfg::TMA_BOX_N);
                            if (F32)   // the W lo plane behind the hi plane
                                tma_load_2d(sB + s * Cfg::B_STAGE_BYTES + Cfg::B_PLANE + h * Cfg::TMA_BOX_N * 128,
                                            &wmap_lo, &full_b[s], kd, n0 + h * Cfg::TMA_BOX_N);
                        }
                    }
#endif
                    if (++tap == a.KK) { tap = 0; ++chunk; }
                }
            }
        }
    } else {
        // ===================== MMA issuer (pair: rank 0 only) =====================
        if (lane == 0 && (!PAIR || rank == 0)) {
            constexpr uint32_t idesc = make_idesc(F32 ? 2u /*TF32*/ : 1u /*BF16*/, PAIR ? 2 * BM : BM, Cfg::UMMA_N);
            int q = 0;
            for (int o = 0; o < nseg; ++o) {
                const Segment sg = segment_j(a, it_begin, it_end, seg_order(o, nseg));
                const int buf = o % Cfg::NBUF;
                if (PAIR) mbar_wait_cluster(&tmem_empty[buf], ((uint32_t)(o / Cfg::NBUF) & 1u) ^ 1u);
                else mbar_wait(&tmem_empty[buf], ((uint32_t)(o / Cfg::NBUF) & 1u) ^ 1u);
                tc_fence_after();
                const uint32_t d_base = tmem_base + (uint32_t)(buf * Cfg::ACC_STRIDE);
                for (int kt = sg.kb; kt < sg.ke; ++kt, ++q) {
                    const int s = q % STAGES;
                    const uint32_t ph = (uint32_t)(q / STAGES) & 1u;
                    if (PAIR) {
                        mbar_wait_cluster(&full_a[s], ph);
                        mbar_wait_cluster(&full_b[s], ph);
                    } else {
                        KT(3, q);
                        mbar_wait(&full_a[s], ph);
                        KT(4, q);
                        if (!MERGED) mbar_wait(&full_b[s], ph);
                        KT(5, q);
                    }
                    tc_fence_after();
                    const uint32_t a_addr = smem_u32(sA + s * Cfg::A_STAGE_BYTES);
                    const uint32_t b_addr = smem_u32(sB + s * Cfg::B_STAGE_BYTES);
#pragma unroll
                    for (int kk = 0; kk < 4; ++kk) {   // 4 K steps of 32 bytes per 128-byte row
                        const uint64_t adesc = make_sw128_desc(a_addr + kk * 32);
#pragma unroll
                        for (int h = 0; h < Cfg::N_MMA; ++h) {
                            const uint64_t bdesc =
                                make_sw128_desc(b_addr + h * Cfg::UMMA_N * 128 + kk * 32);
                            const uint32_t acc = (kt != sg.kb || kk != 0) ? 1u : 0u;
                            if (F32) {   // 3xTF32: lo*hi + hi*lo into the cross accumulator, hi*hi
                                // into the main one (each MMA rounds its accumulator: the
                                // tiny cross terms no longer cost the main sum two roundings)
                                const uint64_t adesc_lo = make_sw128_desc(a_addr + A_PLANE + kk * 32);
                                const uint64_t bdesc_lo =
                                    make_sw128_desc(b_addr + Cfg::B_PLANE + h * Cfg::UMMA_N * 128 + kk * 32);
                                const uint32_t dx = d_base + BLOCK_N + h * Cfg::UMMA_N;
                                mma_tf32_ss(dx, adesc_lo, bdesc, idesc, acc);
                                mma_tf32_ss(dx, adesc, bdesc_lo, idesc, 1u);
                                mma_tf32_ss(d_base + h * Cfg::UMMA_N, adesc, bdesc, idesc, acc);
                            } else if (PAIR) {
                                mma_bf16_ss_pair(d_base + h * Cfg::UMMA_N, adesc, bdesc, idesc, acc);
                            } else {
                                mma_bf16_ss(d_base + h * Cfg::UMMA_N, adesc, bdesc, idesc, acc);
                            }
                        }
                        if (kk == 0) KT(16, q);
                    }
                    KT(17, q);
                    if (PAIR) mma_commit_pair(&empty[s], 0x3);
                    else mma_commit(&empty[s]);
                    KT(6, q);
#ifdef DEFCON_PROBE_MMA_SERIAL   // dev probe: wait for this k-iteration's MMAs to complete (serialises)
                    mbar_wait_spin(&empty[s], ph);
                    KT(11, q);
#endif
                }
                if (PAIR) mma_commit_pair(&tmem_full[buf], 0x3);
                else mma_commit(&tmem_full[buf]);
            }
            TL(14);
        }
    }

    __syncwarp();
    tc_fence_before();
    __syncthreads();
    if (PAIR) cluster_sync_all();      // no CTA leaves while its peer may still touch its smem / TMEM
    if (warp == MMA_WARP) {
        tc_fence_after();
        if (PAIR) tmem_dealloc_pair<Cfg::TMEM_COLS>(tmem_base);
        else tmem_dealloc<Cfg::TMEM_COLS>(tmem_base);
    }
    if (threadIdx.x == 0) TL(15);
}

int num_sms() {
    static int n = 0;
    if (n == 0) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
        if (n <= 0) n = 148;
    }
    return n;
}

// ---- schedule tuning (SURVEY NEXT 3, P:276 / P:286: the paper tunes its tile size per layer).
// tools/autotune.py times every (BLOCK_N, CTA pair, grid cap) candidate per layer shape and per
// per-GPU batch and writes the winners to tuning_table.inc, compiled in here.  Shapes not in
// the table take the defaults (BLOCK_N from Cout, single CTAs, a full persistent grid).
// DEFCON_BLOCK_N / DEFCON_DCN_PAIR / DEFCON_MAX_CTAS override the table (the sweep, tests).
struct TcTuning {
    int block_n;    // 0: from Cout
    int pair;       // -1: default (single CTAs); 0 / 1 (BLOCK_N = 256 only)
    int max_ctas;   // 0: every SM
};
struct TuneEntry {
    int Cin, Cout, H, W, stride, G, nmin, nmax;
    TcTuning t;
};
static const TuneEntry kTuneTable[] = {
#include "tuning_table.inc"
    {0, 0, 0, 0, 0, 0, 0, 0, {0, -1, 0}}   // terminator
};

TcTuning tc_tuning(const DcnGeom& g) {
    TcTuning t{0, -1, 0};
    for (const TuneEntry* e = kTuneTable; e->Cin; ++e)
        if (e->Cin == g.Cin && e->Cout == g.Cout && e->H == g.H && e->W == g.W && e->stride == g.sh &&
            g.sw == g.sh && e->G == g.G && g.KK == 9 && g.N >= e->nmin && g.N <= e->nmax) {
            t = e->t;
            break;
        }
    if (const char* env = getenv("DEFCON_BLOCK_N")) t.block_n = atoi(env);
    if (const char* env = getenv("DEFCON_DCN_PAIR")) t.pair = atoi(env) != 0;
    if (const char* env = getenv("DEFCON_MAX_CTAS")) t.max_ctas = atoi(env);
    return t;
}

// BLOCK_N of the bf16 kernel for this shape: the tuned value, else the smallest tile of
// 64 / 128 / 256 / 512 columns covering Cout.
int tc_block_n(const DcnGeom& g) {
    const int bn = tc_tuning(g).block_n;
    if (bn == 64 || bn == 128 || bn == 256 || bn == 512) return bn;
    return g.Cout <= 64 ? 64 : g.Cout <= 128 ? 128 : g.Cout <= 256 ? 256 : 512;
}

template <int BLOCK_N>
struct Plan {
    int grid;
    int n_tiles;
    int n_tiles_n;
    int ipt;
    long long total;
    size_t counters_bytes;
    size_t partial_bytes;
};

// Pair mode (CTA pairs, cta_group::2): tiles of 2 x BM rows, stream-K over pairs.
// Co-resident 2-CTA clusters of the pair kernel (GPCs with an odd number of usable SMs leave
// one SM unpaired), set by the pair launcher from cudaOccupancyMaxActiveClusters.
static int g_pair_units = 0;

template <int BLOCK_N>
Plan<BLOCK_N> make_plan(const DcnGeom& g, bool pair = false, int cpi = BK) {
    Plan<BLOCK_N> p;
    const int rows = pair ? 2 * BM : BM;
    p.n_tiles_n = (g.Cout + BLOCK_N - 1) / BLOCK_N;
    p.n_tiles = ((g.M + rows - 1) / rows) * p.n_tiles_n;
    p.ipt = (g.Cin / cpi) * g.KK;
    p.total = (long long)p.n_tiles * p.ipt;
    // At least 4 k-iterations per CTA (pair); the tuning's grid cap (DEFCON_MAX_CTAS: tests use
    // it to force long persistent ranges and many whole tiles per CTA).
    const int per = pair ? 2 : 1;
    const int max_units = pair && g_pair_units > 0 ? g_pair_units : num_sms() / per;
    long long units = std::min<long long>(max_units, (p.total + 3) / 4);
    {
        const long long cap = tc_tuning(g).max_ctas;
        if (cap > 0) units = std::min(units, std::max<long long>(cap / per, 1));
    }
    p.grid = (int)std::max<long long>(units, 1) * per;
    // counters: one per tile (per tile half in pair mode); sized for both modes so a workspace
    // from defcon_dcn_workspace_size fits either
    const size_t ctrs = std::max<size_t>((size_t)(((g.M + BM - 1) / BM) * p.n_tiles_n),
                                         (size_t)(2 * ((g.M + 2 * BM - 1) / (2 * BM)) * p.n_tiles_n));
    p.counters_bytes = (ctrs * sizeof(int) + 255) & ~size_t(255);
    p.partial_bytes = (size_t)2 * p.grid * BLOCK_N * BM * sizeof(float);
    return p;
}

// Workspace layout: [0, partials_region) fp32 partial tiles, then the stream-K tile counters.
// The partial region has ONE size for every shape on this device (2 slots per CTA of a full
// persistent grid at the widest tile, BLOCK_N = 512), so the counters of every shape start at
// the same offset and no shape's partials ever land on another shape's counters: a workspace
// zero-filled once stays valid for any sequence of shapes it is large enough for (every launch
// leaves its counters at zero again).
size_t partials_region() {
    return ((size_t)2 * num_sms() * 512 * BM * sizeof(float) + 255) & ~size_t(255);
}

template <int BLOCK_N>
size_t workspace_impl(const DcnGeom& g) {
    return partials_region() + make_plan<BLOCK_N>(g, false).counters_bytes;
}

// fp32 path: W's tf32 hi / lo planes ([Cout][Kd] fp32 each) sit INSIDE the partial region,
// behind the partial tiles of the fp32 plan (BLOCK_N <= 128 needs a quarter of the region), so
// the counters keep their shape-independent offset and no plane ever lands on a counter.
size_t w_split_offset(size_t partial_bytes) { return (partial_bytes + 1023) & ~size_t(1023); }
size_t w_split_bytes(const DcnGeom& g) { return 2 * (size_t)g.Cout * g.KK * g.Cin * sizeof(float); }

// W -> tf32 hi plane (low 13 mantissa bits cleared) and lo plane (w - hi), both exact.
__global__ void __launch_bounds__(256) dcn_w_split_kernel(const float* __restrict__ w, float* __restrict__ whi,
                                                          float* __restrict__ wlo, long n) {
    griddep_wait();   // the previous launch may still read the planes of this workspace
    griddep_launch_dependents();
    for (long i = (long)blockIdx.x * blockDim.x + threadIdx.x; i < n / 4; i += (long)gridDim.x * blockDim.x) {
        const float4 v = __ldg(reinterpret_cast<const float4*>(w) + i);
        float4 h, l;
        h.x = __uint_as_float(__float_as_uint(v.x) & 0xFFFFE000u); l.x = v.x - h.x;
        h.y = __uint_as_float(__float_as_uint(v.y) & 0xFFFFE000u); l.y = v.y - h.y;
        h.z = __uint_as_float(__float_as_uint(v.z) & 0xFFFFE000u); l.z = v.z - h.z;
        h.w = __uint_as_float(__float_as_uint(v.w) & 0xFFFFE000u); l.w = v.w - h.w;
        reinterpret_cast<float4*>(whi)[i] = h;
        reinterpret_cast<float4*>(wlo)[i] = l;
    }
}

// CTA pairs (cta_group::2) for the BLOCK_N = 256 kernel when the tuning asks for them.
bool use_pair(const DcnGeom& g, const TexPlan* tex) {
    return !tex && tc_block_n(g) == 256 && tc_tuning(g).pair == 1;
}

template <int BLOCK_N, int STAGES, bool PAIR = false, bool F32 = false>
cudaError_t launch_impl(const DcnGeom& g, const DcnPtrs& p, void* ws, size_t ws_bytes,
                        const TexPlan* tex, bool hybrid, cudaStream_t stream, const char** detail) {
    using Cfg = TcCfg<BLOCK_N, PAIR, F32>;
    using E = Elem<F32>;
    constexpr int EPI_W = epi_scratch_per_warp<F32, BLOCK_N>();
    if (PAIR && g_pair_units == 0) {   // how many pairs fit at once (one CTA per SM)
        auto kp = dcn_fwd_bf16_tc_kernel<BLOCK_N, STAGES, 0, PAIR, false>;
        const size_t smem_q = 1024 + (size_t)STAGES * Cfg::STAGE_BYTES + 4 * EPI_SCRATCH_PER_WARP +
                              (size_t)BM * g.KK * meta_entry<false>() + bias_smem_offset(STAGES, Cfg::NBUF) +
                              (size_t)BIAS_SMEM_MAX * 4;
        cudaFuncSetAttribute(kp, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem_q);
        cudaLaunchConfig_t qc = {};
        qc.gridDim = dim3(num_sms());
        qc.blockDim = dim3(NUM_THREADS);
        qc.dynamicSmemBytes = smem_q;
        cudaLaunchAttribute qa[1];
        qa[0].id = cudaLaunchAttributeClusterDimension;
        qa[0].val.clusterDim.x = 2;
        qa[0].val.clusterDim.y = 1;
        qa[0].val.clusterDim.z = 1;
        qc.attrs = qa;
        qc.numAttrs = 1;
        int nclusters = 0;
        if (cudaOccupancyMaxActiveClusters(&nclusters, kp, &qc) != cudaSuccess || nclusters <= 0)
            nclusters = num_sms() / 2;
        cudaGetLastError();
        g_pair_units = std::min(nclusters, num_sms() / 2);
        if (getenv("DEFCON_DEBUG")) fprintf(stderr, "defcon: %d co-resident 2-CTA clusters\n", nclusters);
    }
    auto plan = make_plan<BLOCK_N>(g, PAIR, E::CPI);
    const size_t wsplit_off = w_split_offset(plan.partial_bytes);
    if (ws_bytes < partials_region() + plan.counters_bytes || ws == nullptr ||
        plan.partial_bytes > partials_region() || (F32 && wsplit_off + w_split_bytes(g) > partials_region())) {
        *detail = "workspace too small for the stream-K partials and counters";
        return cudaErrorInvalidValue;
    }
    PFN_encodeTiled encode = get_encode_tiled();
    if (!encode) {
        *detail = "cuTensorMapEncodeTiled entry point unavailable";
        return cudaErrorNotSupported;
    }
    const int Kd = g.KK * g.Cin;
    const auto dt = F32 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT32 : CU_TENSOR_MAP_DATA_TYPE_BFLOAT16;
    // W: bf16 as given, or (fp32) its tf32 hi / lo planes split into the workspace first
    void* w_hi = const_cast<void*>(p.weight);
    void* w_lo = w_hi;
    if (F32) {
        w_hi = static_cast<uint8_t*>(ws) + wsplit_off;
        w_lo = static_cast<float*>(w_hi) + (size_t)g.Cout * Kd;
        const long n = (long)g.Cout * Kd;   // a multiple of 4 (Cin % 32 == 0)
        const unsigned nb = (unsigned)std::min<long>((n / 4 + 255) / 256, 4L * num_sms());
        cudaError_t es = launch_pdl(dcn_w_split_kernel, dim3(nb), dim3(256), 0, stream,
                                    static_cast<const float*>(p.weight), static_cast<float*>(w_hi),
                                    static_cast<float*>(w_lo), n);
        if (es != cudaSuccess) {
            *detail = "dcn_w_split_kernel launch failed";
            return es;
        }
    }
    CUtensorMap wmap, wmap_lo;
    cuuint64_t dims[2] = {(cuuint64_t)Kd, (cuuint64_t)g.Cout};
    cuuint64_t strides[1] = {(cuuint64_t)Kd * E::ES};
    cuuint32_t box[2] = {(cuuint32_t)E::CPI, (cuuint32_t)Cfg::TMA_BOX_N};
    cuuint32_t estr[2] = {1, 1};
    CUresult cr = encode(&wmap, dt, 2, w_hi, dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                         CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                         CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (cr == CUDA_SUCCESS)
        cr = encode(&wmap_lo, dt, 2, w_lo, dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                    CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                    CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (cr != CUDA_SUCCESS) {
        *detail = "cuTensorMapEncodeTiled failed for the weight tensor";
        return cudaErrorInvalidValue;
    }
    // y [M][Cout], stored by the epilogue in 32 x 32 boxes (bf16: 64-byte swizzle; fp32: 128-byte)
    CUtensorMap ymap;
    cuuint64_t ydims[2] = {(cuuint64_t)g.Cout, (cuuint64_t)g.M};
    cuuint64_t ystrides[1] = {(cuuint64_t)g.Cout * E::ES};
    cuuint32_t ybox[2] = {(cuuint32_t)CS, 32u};
    cr = encode(&ymap, dt, 2, p.y, ydims, ystrides, ybox, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                F32 ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_64B, CU_TENSOR_MAP_L2_PROMOTION_NONE,
                CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (cr != CUDA_SUCCESS) {
        *detail = "cuTensorMapEncodeTiled failed for the output tensor";
        return cudaErrorInvalidValue;
    }
    TcArgs a;
    a.x = p.x;
    a.offset = p.offset;
    a.mask = p.mask;
    a.bias = p.bias;
    a.y = p.y;
    a.es = E::ES;
    a.cpi = E::CPI;
    a.partials = static_cast<float*>(ws);
    a.counters = reinterpret_cast<int*>(static_cast<uint8_t*>(ws) + partials_region());
    a.H = g.H; a.W = g.W; a.Cin = g.Cin; a.Cout = g.Cout; a.Kw = g.Kw; a.Ho = g.Ho; a.Wo = g.Wo;
    a.sh = g.sh; a.sw = g.sw; a.ph = g.ph; a.pw = g.pw; a.dh = g.dh; a.dw = g.dw;
    a.G = g.G; a.Cg = g.Cg; a.M = g.M; a.KK = g.KK;
    a.bound_h = g.bound_h;
    a.off_f16 = g.off_f16;
    a.ipt = plan.ipt;
    a.n_tiles_n = plan.n_tiles_n;
    a.total_iters = plan.total;
    a.tex = tex ? tex_plan_texture(tex) : 0ull;

    a.bias_in_smem = g.Cout <= BIAS_SMEM_MAX ? 1 : 0;
    a.pair = PAIR ? 1 : 0;
    // Stream-K tile counters are NOT reset here: the workspace is zero-filled once by its
    // owner and every launch leaves it zeroed (the finisher of each split tile resets it).
    const size_t smem = 1024 + (size_t)STAGES * Cfg::STAGE_BYTES + 4 * EPI_W + (size_t)BM * g.KK * meta_entry<F32>() +
                        bias_smem_offset(STAGES, Cfg::NBUF) + (a.bias_in_smem ? (size_t)g.Cout * 4 : 0)
#ifdef DEFCON_PROBE_SMEM_PAD   // dev probe: unused shared memory (the L1 it costs the gathers)
                        + DEFCON_PROBE_SMEM_PAD
#endif
        ;
    auto kern = F32 ? dcn_fwd_bf16_tc_kernel<BLOCK_N, STAGES, 0, false, F32>
                : PAIR ? dcn_fwd_bf16_tc_kernel<BLOCK_N, STAGES, 0, PAIR, false>
                : !tex ? dcn_fwd_bf16_tc_kernel<BLOCK_N, STAGES, 0, false, false>
                : hybrid ? dcn_fwd_bf16_tc_kernel<BLOCK_N, STAGES, NPW / 2, false, false>
                         : dcn_fwd_bf16_tc_kernel<BLOCK_N, STAGES, NPW, false, false>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) {
        *detail = "cudaFuncSetAttribute(MaxDynamicSharedMemorySize) failed";
        return e;
    }
    if (PAIR) {   // 2-CTA clusters (the pair shares one M = 256 MMA) + PDL
        e = cudaFuncSetAttribute(kern, cudaFuncAttributeNonPortableClusterSizeAllowed, 0);
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = dim3(plan.grid);
        cfg.blockDim = dim3(NUM_THREADS);
        cfg.dynamicSmemBytes = smem;
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
        e = cudaLaunchKernelEx(&cfg, kern, wmap, wmap_lo, ymap, a);
    } else {
        e = launch_pdl(kern, dim3(plan.grid), dim3(NUM_THREADS), smem, stream, wmap, wmap_lo, ymap, a);
    }
    if (e != cudaSuccess) *detail = "dcn_fwd_bf16_tc_kernel launch failed";
    return e;
}

}  // namespace

#ifdef DEFCON_PROBE_KTRACE
extern "C" int defcon_debug_ktrace(long long* host) {
    return (int)cudaMemcpyFromSymbol(host, g_kt, sizeof(g_kt));
}
#endif

#ifdef DEFCON_PROBE_TIMELINE
extern "C" int defcon_debug_timeline(unsigned long long* host) {
    return (int)cudaMemcpyFromSymbol(host, g_tl, sizeof(g_tl));
}
#endif

// Shared-memory budget: stages + metadata for up to 12 taps must fit in 227 KB.
bool dcn_tc_bf16_supported(const DcnGeom& g) {
    if (g.Cin % BK != 0 || g.Cg % BK != 0) return false;
    if (g.Cout % 16 != 0) return false;
    if ((long)BM * g.KK * META_ENTRY > 48 * 1024) return false;
    return true;
}

// The workspace bytes that must be zero before the first launch: the stream-K tile counters
// at [offset, offset + bytes) (every launch leaves them zero again).  The fp32 partials need
// no initialisation.
void dcn_tc_bf16_workspace_counters(const DcnGeom& g, size_t* offset, size_t* bytes) {
    *offset = partials_region();
    switch (tc_block_n(g)) {
        case 64: *bytes = make_plan<64>(g).counters_bytes; break;
        case 128: *bytes = make_plan<128>(g).counters_bytes; break;
        case 256: *bytes = make_plan<256>(g).counters_bytes; break;
        default: *bytes = make_plan<512>(g).counters_bytes; break;
    }
}

size_t dcn_tc_bf16_workspace(const DcnGeom& g) {
    switch (tc_block_n(g)) {
        case 64: return workspace_impl<64>(g);
        case 128: return workspace_impl<128>(g);
        case 256: return workspace_impl<256>(g);
        default: return workspace_impl<512>(g);
    }
}

cudaError_t launch_dcn_tc_bf16(const DcnGeom& g, const DcnPtrs& p, void* ws, size_t ws_bytes,
                               const TexPlan* tex, bool hybrid, cudaStream_t stream, const char** detail) {
    const int bn = tc_block_n(g);
    if (bn == 64) return launch_impl<64, 6>(g, p, ws, ws_bytes, tex, hybrid, stream, detail);
#ifndef DEFCON_STAGES_128
#define DEFCON_STAGES_128 3   // 4 -> 3: C3 37.3 -> 36.5 us (more L1 for the gathers)
#endif
    if (bn == 128) return launch_impl<128, DEFCON_STAGES_128>(g, p, ws, ws_bytes, tex, hybrid, stream, detail);
#ifndef DEFCON_STAGES_256
#define DEFCON_STAGES_256 3   // 2 -> 3 once the compact table freed 18 KB: C4 43.4 -> 42.0 us
#endif
#ifndef DEFCON_STAGES_PAIR
#define DEFCON_STAGES_PAIR 4
#endif
    if (bn == 256 && use_pair(g, tex))
        return launch_impl<256, DEFCON_STAGES_PAIR, true>(g, p, ws, ws_bytes, tex, hybrid, stream, detail);
    if (bn == 256) return launch_impl<256, DEFCON_STAGES_256>(g, p, ws, ws_bytes, tex, hybrid, stream, detail);
    return launch_impl<512, 2>(g, p, ws, ws_bytes, tex, hybrid, stream, detail);
}

// ---- fp32 on the tensor cores (DEFCON_FP32_3XTF32): same kernel, kind::tf32 with the 3xTF32
// split, 32 channels per k-iteration, N tiles of <= 128 columns (the B stage holds two planes).
template <int BLOCK_N>
static bool f32_planes_fit(const DcnGeom& g) {
    return w_split_offset(make_plan<BLOCK_N>(g, false, 32).partial_bytes) + w_split_bytes(g) <= partials_region();
}

bool dcn_tc_f32_supported(const DcnGeom& g) {
    if (g.Cin % 32 != 0 || g.Cg % 32 != 0) return false;
    if (g.Cout % 16 != 0) return false;
    if ((long)BM * g.KK * META_ENTRY > 48 * 1024) return false;
    return g.Cout <= 64 ? f32_planes_fit<64>(g) : f32_planes_fit<128>(g);   // Cout * Kd up to ~7M
}

size_t dcn_tc_f32_workspace(const DcnGeom& g) {
    return partials_region() + (g.Cout <= 64 ? make_plan<64>(g, false, 32).counters_bytes
                                              : make_plan<128>(g, false, 32).counters_bytes);
}

void dcn_tc_f32_workspace_counters(const DcnGeom& g, size_t* offset, size_t* bytes) {
    *offset = partials_region();
    *bytes = g.Cout <= 64 ? make_plan<64>(g, false, 32).counters_bytes : make_plan<128>(g, false, 32).counters_bytes;
}

cudaError_t launch_dcn_tc_f32(const DcnGeom& g, const DcnPtrs& p, void* ws, size_t ws_bytes, cudaStream_t stream,
                              const char** detail) {
    if (g.Cout <= 64) return launch_impl<64, 3, false, true>(g, p, ws, ws_bytes, nullptr, false, stream, detail);
    return launch_impl<128, 2, false, true>(g, p, ws, ws_bytes, nullptr, false, stream, detail);
}

}  // namespace defcon
