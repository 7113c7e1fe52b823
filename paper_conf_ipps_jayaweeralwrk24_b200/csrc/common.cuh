// common.cuh -- sm_100a device helpers shared by the libdefcon kernels:
// mbarrier, TMA, tcgen05 (TMEM alloc / MMA / commit / ld), proxy fences and
// bf16 packing.  Inline PTX only; no CUTLASS/CuTe dependency.
#pragma once

#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_fp16.h>
#include <cuda_runtime.h>
#include <stdint.h>

#define DEFCON_DEVICE __device__ __forceinline__

namespace defcon {

// ------------------------------------------------------------------ smem address
DEFCON_DEVICE uint32_t smem_u32(const void* p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

// ------------------------------------------------------------------ mbarrier
DEFCON_DEVICE void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count)
                 : "memory");
}

DEFCON_DEVICE void fence_barrier_init() {
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}

DEFCON_DEVICE void mbar_arrive(uint64_t* bar) {
    asm volatile(
        "{\n\t.reg .b64 st;\n\t"
        "mbarrier.arrive.shared::cta.b64 st, [%0];\n\t}" ::"r"(smem_u32(bar))
        : "memory");
}

DEFCON_DEVICE void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile(
        "{\n\t.reg .b64 st;\n\t"
        "mbarrier.arrive.expect_tx.shared::cta.b64 st, [%0], %1;\n\t}" ::"r"(smem_u32(bar)),
        "r"(bytes)
        : "memory");
}

#ifndef DEFCON_MBAR_HINT_NS
#define DEFCON_MBAR_HINT_NS 100000   // ns; 0 = the implementation default (measured ~0.5 % slower at C4)
#endif
DEFCON_DEVICE uint32_t mbar_try_wait(uint64_t* bar, uint32_t parity) {
    uint32_t ok;
#if DEFCON_MBAR_HINT_NS > 0
    // suspend-time hint: a waiting warp sleeps until the phase completes (or the hint elapses)
    // instead of re-issuing try_wait, leaving issue slots to the producer warps
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(ok)
        : "r"(smem_u32(bar)), "r"(parity), "n"(DEFCON_MBAR_HINT_NS)
        : "memory");
#else
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(ok)
        : "r"(smem_u32(bar)), "r"(parity)
        : "memory");
#endif
    return ok;
}

// Blocks until the barrier phase with the given parity has completed
// (a fresh barrier counts its "previous" phase, parity 1, as complete).
DEFCON_DEVICE void mbar_wait(uint64_t* bar, uint32_t parity) {
    while (!mbar_try_wait(bar, parity)) {
    }
}

// Spinning variant (mbarrier.test_wait, never suspends): for the single MMA-issuing thread,
// whose wake-up latency after a suspended try_wait is exposed as a tensor-pipe bubble.
DEFCON_DEVICE void mbar_wait_spin(uint64_t* bar, uint32_t parity) {
    uint32_t ok = 0;
    while (!ok) {
        asm volatile(
            "{\n\t.reg .pred p;\n\t"
            "mbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
            "selp.u32 %0, 1, 0, p;\n\t}"
            : "=r"(ok)
            : "r"(smem_u32(bar)), "r"(parity)
            : "memory");
    }
}

// ------------------------------------------------------------------ bounded deformation
// P:182 (section III-A-c), reading R12: the offset d of a tap at regular displacement r from the
// centre tap, restricted so that r + d stays in [-h, h] (the P x P window, h = (P-1)/2).
// h < 0: unbounded.  A NaN offset stays NaN (the samplers turn it into zeros).
DEFCON_DEVICE float bound_offset(float d, float r, float h) {
    if (h < 0.f || d != d) return d;
    return fminf(fmaxf(r + d, -h), h) - r;
}

// Offsets / mask in fp32 or binary16 (tex2D++, R13): element pair `i2` (dy, dx), mask `i`.
DEFCON_DEVICE float2 ld_offset2(const float* base, long i2, bool f16) {
    if (f16) return __half22float2(__ldg(reinterpret_cast<const __half2*>(base) + (i2 >> 1)));
    return __ldg(reinterpret_cast<const float2*>(base + i2));
}
DEFCON_DEVICE float ld_mask1(const float* base, long i, bool f16) {
    return f16 ? __half2float(__ldg(reinterpret_cast<const __half*>(base) + i)) : __ldg(base + i);
}
DEFCON_DEVICE void st_offset1(float* base, long i, float v, bool f16) {
    if (f16) reinterpret_cast<__half*>(base)[i] = __float2half_rn(v);
    else base[i] = v;
}

// ------------------------------------------------------------------ fences
// Make this thread's generic-proxy smem writes visible to the async proxy
// (tcgen05.mma operand reads, TMA).
DEFCON_DEVICE void fence_proxy_async_smem() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

DEFCON_DEVICE void named_bar_sync(uint32_t id, uint32_t nthreads) {
    asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}

// ------------------------------------------------------------------ programmatic dependent launch
// Kernels launched with cudaLaunchAttributeProgrammaticStreamSerialization may start while
// the previous kernel in the stream drains; griddep_wait() blocks until that kernel has
// completed and its writes are visible, so it must precede every access to data the
// previous kernel may produce (or consume: our outputs).
DEFCON_DEVICE void griddep_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
DEFCON_DEVICE void griddep_launch_dependents() {
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}

// Host side: launch `kern` with programmatic stream serialization (PDL) enabled.
template <typename... KArgs, typename... Args>
inline cudaError_t launch_pdl(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem,
                              cudaStream_t stream, Args... args) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.dynamicSmemBytes = smem;
    cfg.stream = stream;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, kern, args...);
}

// ------------------------------------------------------------------ TMA
DEFCON_DEVICE void tma_prefetch_desc(const CUtensorMap* map) {
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(map)) : "memory");
}

// 2-D tiled TMA load global -> shared, completion signalled on `bar` (tx bytes).
DEFCON_DEVICE void tma_load_2d(void* smem_dst, const CUtensorMap* map, uint64_t* bar, int c0,
                               int c1) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes"
        " [%0], [%1, {%3, %4}], [%2];" ::"r"(smem_u32(smem_dst)),
        "l"(reinterpret_cast<uint64_t>(map)), "r"(smem_u32(bar)), "r"(c0), "r"(c1)
        : "memory");
}

// 3-D tiled TMA load global -> shared (coordinates innermost first; out-of-bounds elements of the
// box are zero-filled), completion signalled on `bar` (tx bytes = the full box).
DEFCON_DEVICE void tma_load_3d(void* smem_dst, const CUtensorMap* map, uint64_t* bar, int c0, int c1,
                               int c2) {
    asm volatile(
        "cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes"
        " [%0], [%1, {%3, %4, %5}], [%2];" ::"r"(smem_u32(smem_dst)),
        "l"(reinterpret_cast<uint64_t>(map)), "r"(smem_u32(bar)), "r"(c0), "r"(c1), "r"(c2)
        : "memory");
}

// 1-D bulk copy global -> shared (bytes a multiple of 16, both addresses 16-byte aligned),
// completion signalled on `bar` (tx bytes).
DEFCON_DEVICE void bulk_load(void* smem_dst, const void* src, uint32_t bytes, uint64_t* bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     smem_u32(smem_dst)),
                 "l"(src), "r"(bytes), "r"(smem_u32(bar))
                 : "memory");
}

// 4-D tiled TMA load global -> shared (coordinates innermost first; out-of-bounds elements of the
// box are zero-filled), completion signalled on `bar` (tx bytes = the full box).
DEFCON_DEVICE void tma_load_4d(void* smem_dst, const CUtensorMap* map, uint64_t* bar, int c0, int c1,
                               int c2, int c3) {
    asm volatile(
        "cp.async.bulk.tensor.4d.shared::cluster.global.tile.mbarrier::complete_tx::bytes"
        " [%0], [%1, {%3, %4, %5, %6}], [%2];" ::"r"(smem_u32(smem_dst)),
        "l"(reinterpret_cast<uint64_t>(map)), "r"(smem_u32(bar)), "r"(c0), "r"(c1), "r"(c2), "r"(c3)
        : "memory");
}

// 2-D tiled TMA store shared -> global (bulk async-group completion).  Elements of the box
// outside the tensor are not written (row / column tails are clipped by the TMA unit).
DEFCON_DEVICE void tma_store_2d(const CUtensorMap* map, const void* smem_src, int c0, int c1) {
    asm volatile(
        "cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%2, %3}], [%1];" ::"l"(
            reinterpret_cast<uint64_t>(map)),
        "r"(smem_u32(smem_src)), "r"(c0), "r"(c1)
        : "memory");
}
DEFCON_DEVICE void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
// Wait until at most N committed bulk groups still READ their shared-memory source.
template <int N>
DEFCON_DEVICE void bulk_wait_read() {
    asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}
// Wait until every committed bulk group has completed (writes performed).
DEFCON_DEVICE void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }

// ------------------------------------------------------------------ tcgen05
template <uint32_t kCols>
DEFCON_DEVICE void tmem_alloc(uint32_t* smem_result) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     smem_u32(smem_result)),
                 "n"(kCols)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
}

template <uint32_t kCols>
DEFCON_DEVICE void tmem_dealloc(uint32_t taddr) {
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(taddr), "n"(kCols)
                 : "memory");
}

DEFCON_DEVICE void tc_fence_before() {
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
}
DEFCON_DEVICE void tc_fence_after() {
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
}

// D[tmem] (+)= A[smem] * B[smem]^T, kind::f16 (bf16 inputs, fp32 accumulate).
DEFCON_DEVICE void mma_bf16_ss(uint32_t d_tmem, uint64_t a_desc, uint64_t b_desc, uint32_t idesc,
                               uint32_t accumulate) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
        "l"(a_desc), "l"(b_desc), "r"(idesc), "r"(accumulate)
        : "memory");
}

// D[tmem] (+)= A[smem] * B[smem]^T, kind::tf32 (fp32 storage, tf32 multiply).
DEFCON_DEVICE void mma_tf32_ss(uint32_t d_tmem, uint64_t a_desc, uint64_t b_desc, uint32_t idesc,
                               uint32_t accumulate) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
        "l"(a_desc), "l"(b_desc), "r"(idesc), "r"(accumulate)
        : "memory");
}

// D[tmem] (+)= A[tmem] * B[smem desc]^T, kind::tf32 (the A operand read from tensor memory:
// M = 128 lanes, K = 8 consecutive 32-bit columns starting at a_tmem).
DEFCON_DEVICE void mma_tf32_ts(uint32_t d_tmem, uint32_t a_tmem, uint64_t b_desc, uint32_t idesc,
                               uint32_t accumulate) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::tf32 [%0], [%1], %2, %3, p;\n\t}" ::"r"(d_tmem),
        "r"(a_tmem), "l"(b_desc), "r"(idesc), "r"(accumulate)
        : "memory");
}

// registers -> tensor memory, 16 lanes x 256 bits, 4 repetitions along the columns: thread t
// writes lanes (t/4) and (t/4)+8 of the 16-lane block at `taddr`, columns 8c + 2(t%4) and
// 8c + 2(t%4) + 1 of repetition c: r[4c..4c+1] to the first lane, r[4c+2..4c+3] to the second.
DEFCON_DEVICE void tmem_st_16x256b_x4(uint32_t taddr, const uint32_t (&r)[16]) {
    asm volatile(
        "tcgen05.st.sync.aligned.16x256b.x4.b32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, "
        "%12, %13, %14, %15, %16};" ::"r"(taddr),
        "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7]), "r"(r[8]),
        "r"(r[9]), "r"(r[10]), "r"(r[11]), "r"(r[12]), "r"(r[13]), "r"(r[14]), "r"(r[15])
        : "memory");
}
DEFCON_DEVICE void tmem_st_16x256b_x2(uint32_t taddr, const uint32_t (&r)[8]) {
    asm volatile("tcgen05.st.sync.aligned.16x256b.x2.b32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8};" ::"r"(taddr),
                 "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7])
                 : "memory");
}
DEFCON_DEVICE void tmem_st_wait() { asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory"); }

// Arrive on `bar` when all previously issued tcgen05.mma of this thread complete.
DEFCON_DEVICE void mma_commit(uint64_t* bar) {
    asm volatile(
        "tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
            smem_u32(bar))
        : "memory");
}

// 32 lanes x 32 bit, 16 consecutive columns -> 16 registers per thread.
DEFCON_DEVICE void tmem_ld_32x32b_x16(uint32_t taddr, uint32_t (&r)[16]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x16.b32 "
        "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]),
          "=r"(r[7]), "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]),
          "=r"(r[14]), "=r"(r[15])
        : "r"(taddr)
        : "memory");
}

// 32 lanes x 32 bit, 32 consecutive columns -> 32 registers per thread.
DEFCON_DEVICE void tmem_ld_32x32b_x32(uint32_t taddr, uint32_t (&r)[32]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 "
        "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
        "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]),
          "=r"(r[7]), "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]),
          "=r"(r[14]), "=r"(r[15]), "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]),
          "=r"(r[21]), "=r"(r[22]), "=r"(r[23]), "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]),
          "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
        : "r"(taddr)
        : "memory");
}

DEFCON_DEVICE void tmem_ld_wait() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }

// Shared-memory matrix descriptor for a K-major operand tile stored in the
// canonical SWIZZLE_128B layout: rows of 128 bytes, 8-row groups 1024 bytes apart.
//   bits [0,14)  start address >> 4
//   bits [16,30) leading byte offset >> 4 (ignored for swizzled K-major; 1)
//   bits [32,46) stride byte offset >> 4 (1024 B between 8-row groups)
//   bits [46,48) descriptor version (1 on sm_100)
//   bits [61,64) layout type (2 = SWIZZLE_128B)
DEFCON_DEVICE uint64_t make_sw128_desc(uint32_t smem_addr) {
    uint64_t d = 0;
    d |= static_cast<uint64_t>((smem_addr >> 4) & 0x3FFF);
    d |= static_cast<uint64_t>(1) << 16;
    d |= static_cast<uint64_t>(1024 >> 4) << 32;
    d |= static_cast<uint64_t>(1) << 46;
    d |= static_cast<uint64_t>(2) << 61;
    return d;
}

// Instruction descriptor, kind::f16 / kind::tf32 with fp32 accumulation,
// both operands K-major, dense.
//   [4,6) c_format (1 = F32)  [7,10) a_format  [10,13) b_format
//   (0 = F16, 1 = BF16, 2 = TF32)  [15] a_major  [16] b_major (0 = K)
//   [17,23) N >> 3   [24,29) M >> 4
__host__ __device__ constexpr uint32_t make_idesc(uint32_t ab_format, uint32_t M, uint32_t N) {
    return (1u << 4) | (ab_format << 7) | (ab_format << 10) | ((N >> 3) << 17) | ((M >> 4) << 24);
}

// ------------------------------------------------------------------ bf16 helpers
DEFCON_DEVICE float bf16lo_to_f32(uint32_t w) { return __uint_as_float(w << 16); }
DEFCON_DEVICE float bf16hi_to_f32(uint32_t w) { return __uint_as_float(w & 0xFFFF0000u); }

// Pack two fp32 into bf16x2 with round-to-nearest-even; `lo` in the low half.
DEFCON_DEVICE uint32_t pack_bf16x2(float lo, float hi) {
    uint32_t r;
    asm("cvt.rn.bf16x2.f32 %0, %1, %2;" : "=r"(r) : "f"(hi), "f"(lo));
    return r;
}

DEFCON_DEVICE void st_shared_v4(uint32_t addr, uint32_t a, uint32_t b, uint32_t c, uint32_t d) {
    asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(addr), "r"(a), "r"(b), "r"(c),
                 "r"(d)
                 : "memory");
}

DEFCON_DEVICE uint32_t ld_shared_u32(uint32_t addr) {
    uint32_t v;
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(addr));
    return v;
}

DEFCON_DEVICE uint2 ld_shared_v2(uint32_t addr) {
    uint2 r;
    asm volatile("ld.shared.v2.u32 {%0,%1}, [%2];" : "=r"(r.x), "=r"(r.y) : "r"(addr));
    return r;
}

// d = x * w + c with x the bf16 in half XH of `x`, w the bf16 in half WH of `w` and c, d fp32:
// the bf16 x bf16 product is exact in fp32, one rounding for the sum (sm_100 mixed-precision
// fma.rn.f32.bf16 -> SASS FHFMA.BF16; no bf16 -> fp32 unpack instruction needed).
template <int XH, int WH>
DEFCON_DEVICE float fma_bf16h(uint32_t x, uint32_t w, float c) {
    float d;
    if constexpr (XH == 0 && WH == 0)
        asm("{.reg .b16 x0, x1, w0, w1;\n\tmov.b32 {x0, x1}, %1;\n\tmov.b32 {w0, w1}, %2;\n\t"
            "fma.rn.f32.bf16 %0, x0, w0, %3;}" : "=f"(d) : "r"(x), "r"(w), "f"(c));
    else if constexpr (XH == 1 && WH == 0)
        asm("{.reg .b16 x0, x1, w0, w1;\n\tmov.b32 {x0, x1}, %1;\n\tmov.b32 {w0, w1}, %2;\n\t"
            "fma.rn.f32.bf16 %0, x1, w0, %3;}" : "=f"(d) : "r"(x), "r"(w), "f"(c));
    else if constexpr (XH == 0 && WH == 1)
        asm("{.reg .b16 x0, x1, w0, w1;\n\tmov.b32 {x0, x1}, %1;\n\tmov.b32 {w0, w1}, %2;\n\t"
            "fma.rn.f32.bf16 %0, x0, w1, %3;}" : "=f"(d) : "r"(x), "r"(w), "f"(c));
    else
        asm("{.reg .b16 x0, x1, w0, w1;\n\tmov.b32 {x0, x1}, %1;\n\tmov.b32 {w0, w1}, %2;\n\t"
            "fma.rn.f32.bf16 %0, x1, w1, %3;}" : "=f"(d) : "r"(x), "r"(w), "f"(c));
    return d;
}

DEFCON_DEVICE uint4 ld_shared_v4(uint32_t addr) {
    uint4 r;
    asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
                 : "r"(addr));
    return r;
}

// 64-bit address = base + 32-bit unsigned byte offset (one IMAD.WIDE.U32).
DEFCON_DEVICE const void* add_u32(const void* base, uint32_t off) {
    uint64_t p;
    asm("mad.wide.u32 %0, %1, 1, %2;" : "=l"(p) : "r"(off), "l"(reinterpret_cast<uint64_t>(base)));
    return reinterpret_cast<const void*>(p);
}

// ------------------------------------------------------------------ CTA pair (cta_group::2)
// Two CTAs of a 2-CTA cluster run one M = 256 MMA: each holds 128 rows of A and half of B in
// its own shared memory and 128 rows of the accumulator in its own TMEM; only rank 0 issues.
DEFCON_DEVICE uint32_t cluster_ctarank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
// Every thread of both CTAs: release our prior writes, acquire the peer's.
DEFCON_DEVICE void cluster_sync_all() {
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
// Arrive on the barrier at the same shared-memory offset in CTA `cta` of the cluster.
DEFCON_DEVICE void mbar_arrive_cluster(uint64_t* bar, uint32_t cta) {
    asm volatile(
        "{\n\t.reg .b32 ra;\n\t"
        "mapa.shared::cluster.u32 ra, %0, %1;\n\t"
        "mbarrier.arrive.shared::cluster.b64 _, [ra];\n\t}" ::"r"(smem_u32(bar)),
        "r"(cta)
        : "memory");
}
// Release-arrive (cluster scope) on the barrier at the same offset in CTA `cta`: orders this
// thread's earlier distributed-shared-memory stores before the arrival.
DEFCON_DEVICE void mbar_arrive_release_cluster(uint64_t* bar, uint32_t cta) {
    asm volatile(
        "{\n\t.reg .b32 ra;\n\t"
        "mapa.shared::cluster.u32 ra, %0, %1;\n\t"
        "mbarrier.arrive.release.cluster.shared::cluster.b64 _, [ra];\n\t}" ::"r"(smem_u32(bar)),
        "r"(cta)
        : "memory");
}
// 16-byte store into CTA `cta`'s shared memory at the offset of local address `laddr`.
DEFCON_DEVICE void st_cluster_v4(uint32_t laddr, uint32_t cta, uint32_t a, uint32_t b, uint32_t c, uint32_t d) {
    asm volatile(
        "{\n\t.reg .b32 ra;\n\t"
        "mapa.shared::cluster.u32 ra, %0, %1;\n\t"
        "st.shared::cluster.v4.b32 [ra], {%2, %3, %4, %5};\n\t}" ::"r"(laddr),
        "r"(cta), "r"(a), "r"(b), "r"(c), "r"(d)
        : "memory");
}

// Wait for a phase whose arrivals may come from the peer CTA (cluster-scope acquire).
DEFCON_DEVICE void mbar_wait_cluster(uint64_t* bar, uint32_t parity) {
    uint32_t ok = 0;
    while (!ok) {
        asm volatile(
            "{\n\t.reg .pred p;\n\t"
            "mbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 p, [%1], %2;\n\t"
            "selp.u32 %0, 1, 0, p;\n\t}"
            : "=r"(ok)
            : "r"(smem_u32(bar)), "r"(parity)
            : "memory");
    }
}
template <uint32_t kCols>
DEFCON_DEVICE void tmem_alloc_pair(uint32_t* smem_result) {
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     smem_u32(smem_result)),
                 "n"(kCols)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
}
template <uint32_t kCols>
DEFCON_DEVICE void tmem_dealloc_pair(uint32_t taddr) {
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(taddr), "n"(kCols) : "memory");
}
// D[tmem] (+)= A * B^T over the pair: M = 256 (128 rows per CTA), B split by N across the CTAs.
DEFCON_DEVICE void mma_bf16_ss_pair(uint32_t d_tmem, uint64_t a_desc, uint64_t b_desc, uint32_t idesc,
                                    uint32_t accumulate) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
        "l"(a_desc), "l"(b_desc), "r"(idesc), "r"(accumulate)
        : "memory");
}
// Arrive (once) on the barrier at this offset in every CTA of `mask` when the issuing thread's
// prior pair MMAs complete.
DEFCON_DEVICE void mma_commit_pair(uint64_t* bar, uint16_t mask) {
    asm volatile(
        "tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(
            smem_u32(bar)),
        "h"(mask)
        : "memory");
}
// 2-D TMA load into this CTA's shared memory whose completion is counted on the barrier at the
// same offset in the pair's rank-0 CTA (bit 24 of the cluster shared address selects the peer).
DEFCON_DEVICE void tma_load_2d_pair(void* smem_dst, const CUtensorMap* map, uint64_t* bar, int c0, int c1) {
    asm volatile(
        "cp.async.bulk.tensor.2d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes"
        " [%0], [%1, {%3, %4}], [%2];" ::"r"(smem_u32(smem_dst)),
        "l"(reinterpret_cast<uint64_t>(map)), "r"(smem_u32(bar) & 0xFEFFFFFFu), "r"(c0), "r"(c1)
        : "memory");
}

// ------------------------------------------------------------------ packed fp32 (FFMA2)
// sm_100 executes two fp32 FMAs per instruction on a 64-bit register pair.
DEFCON_DEVICE uint64_t f32x2_pack(float lo, float hi) {
    uint64_t r;
    asm("mov.b64 %0, {%1, %2};" : "=l"(r) : "f"(lo), "f"(hi));
    return r;
}
DEFCON_DEVICE uint64_t f32x2_fma(uint64_t a, uint64_t b, uint64_t c) {
    uint64_t d;
    asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d) : "l"(a), "l"(b), "l"(c));
    return d;
}
DEFCON_DEVICE uint64_t f32x2_mul(uint64_t a, uint64_t b) {
    uint64_t d;
    asm("mul.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b));
    return d;
}
// bf16x2 word -> (lo, hi) fp32 pair (exact widening).
DEFCON_DEVICE uint64_t bf16x2_to_f32x2(uint32_t w) {
    return f32x2_pack(__uint_as_float(w << 16), __uint_as_float(w & 0xFFFF0000u));
}
// (lo, hi) fp32 pair -> bf16x2 word, round-to-nearest-even.
DEFCON_DEVICE uint32_t f32x2_to_bf16x2(uint64_t v) {
    uint32_t r;
    asm("{.reg .f32 a, b;\n\tmov.b64 {a, b}, %1;\n\tcvt.rn.bf16x2.f32 %0, b, a;}" : "=r"(r) : "l"(v));
    return r;
}

// 256-bit read-only global load (sm_100: LDG.E.256), p must be 32-byte aligned.
struct U8x32 {
    uint32_t w[8];
};
DEFCON_DEVICE U8x32 ldg_nc_v8(const void* p) {
    U8x32 r;
    asm volatile("ld.global.nc.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=r"(r.w[0]), "=r"(r.w[1]), "=r"(r.w[2]), "=r"(r.w[3]), "=r"(r.w[4]),
                   "=r"(r.w[5]), "=r"(r.w[6]), "=r"(r.w[7])
                 : "l"(p));
    return r;
}

DEFCON_DEVICE uint4 ldg_nc_v4(const void* p) {
    uint4 r;
    asm volatile("ld.global.nc.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
                 : "l"(p));
    return r;
}

}  // namespace defcon
