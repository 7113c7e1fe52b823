// api.cu -- the extern "C" boundary of libdefcon.so (declared in include/defcon.h):
// argument validation, kernel selection and launch, workspace sizing and the
// host-buffer end-to-end entry point.  No allocation on the call path, no host sync
// (except defcon_layer_forward_host), no CPU fallback.
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <mutex>
#include <algorithm>
#include <cstdlib>

#include "../../include/defcon.h"
#include "common.cuh"
#include "kernels.h"

namespace defcon {

static thread_local char g_detail[512] = "";

static int fail(int status, const char* fmt, ...) {
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(g_detail, sizeof(g_detail), fmt, ap);
    va_end(ap);
    return status;
}

static int cuda_fail(cudaError_t e, const char* what) {
    return fail(DEFCON_ERR_CUDA, "%s: %s", what, cudaGetErrorString(e));
}

static bool aligned16(const void* p) { return (reinterpret_cast<uintptr_t>(p) & 15u) == 0; }
static bool aligned32(const void* p) { return (reinterpret_cast<uintptr_t>(p) & 31u) == 0; }

static int out_size(int in, int k, int stride, int pad, int dil) {
    const long span = (long)in + 2L * pad - (long)dil * (k - 1) - 1;
    if (span < 0 || stride <= 0) return 0;
    return (int)(span / stride + 1);
}

PFN_encodeTiled get_encode_tiled() {
    static PFN_encodeTiled fn = nullptr;
    static bool tried = false;
    if (!tried) {
        tried = true;
        void* p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) ==
                cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = reinterpret_cast<PFN_encodeTiled>(p);
    }
    return fn;
}

// Shared validation of the conv geometry.
static int check_conv(const defcon_conv_t& cv) {
    if (cv.stride_h <= 0 || cv.stride_w <= 0 || cv.dil_h <= 0 || cv.dil_w <= 0)
        return fail(DEFCON_ERR_INVALID_ARG, "stride and dilation must be positive");
    if (cv.pad_h < 0 || cv.pad_w < 0) return fail(DEFCON_ERR_INVALID_ARG, "padding must be >= 0");
    if (cv.offset_groups <= 0) return fail(DEFCON_ERR_INVALID_ARG, "offset_groups must be > 0");
    if (cv.bound < 0) return fail(DEFCON_ERR_INVALID_ARG, "bound must be >= 0 (0 = unbounded)");
    if (cv.offset_dtype != DEFCON_F32 && cv.offset_dtype != DEFCON_F16)
        return fail(DEFCON_ERR_INVALID_ARG, "offset_dtype must be DEFCON_F32 or DEFCON_F16");
    return DEFCON_OK;
}

static int make_geom(int N, int H, int W, int Cin, int Cout, int Kh, int Kw,
                     const defcon_conv_t& cv, int dtype, DcnGeom* g) {
    if (N <= 0 || H <= 0 || W <= 0 || Cin <= 0 || Cout <= 0 || Kh <= 0 || Kw <= 0)
        return fail(DEFCON_ERR_INVALID_ARG, "sizes must be positive");
    int rc = check_conv(cv);
    if (rc) return rc;
    if (dtype != DEFCON_F32 && dtype != DEFCON_BF16) return fail(DEFCON_ERR_INVALID_ARG, "bad dtype");
    if (Cin % cv.offset_groups != 0)
        return fail(DEFCON_ERR_INVALID_ARG, "offset_groups (%d) must divide Cin (%d)", cv.offset_groups, Cin);
    g->N = N; g->H = H; g->W = W; g->Cin = Cin; g->Cout = Cout; g->Kh = Kh; g->Kw = Kw;
    g->Ho = out_size(H, Kh, cv.stride_h, cv.pad_h, cv.dil_h);
    g->Wo = out_size(W, Kw, cv.stride_w, cv.pad_w, cv.dil_w);
    if (g->Ho <= 0 || g->Wo <= 0) return fail(DEFCON_ERR_INVALID_ARG, "output grid is empty");
    g->sh = cv.stride_h; g->sw = cv.stride_w; g->ph = cv.pad_h; g->pw = cv.pad_w;
    g->dh = cv.dil_h; g->dw = cv.dil_w;
    g->G = cv.offset_groups;
    g->Cg = Cin / cv.offset_groups;
    g->bound_h = cv.bound > 0 ? 0.5f * (float)(cv.bound - 1) : -1.f;
    g->off_f16 = cv.offset_dtype == DEFCON_F16 ? 1 : 0;
    g->KK = Kh * Kw;
    const long M = (long)N * g->Ho * g->Wo;
    if ((long)N * H * W * Cin >= (1L << 31) || M * Cout >= (1L << 31) ||
        M * g->G * g->KK * 2 >= (1L << 31) || (long)Cout * g->KK * Cin >= (1L << 31))
        return fail(DEFCON_ERR_LIMIT, "tensor too large for 32-bit element indexing");
    // the samplers address x by 32-bit byte offsets from its base (sampling metadata)
    if ((long)N * H * W * Cin * (dtype == DEFCON_BF16 ? 2 : 4) >= (1L << 32))
        return fail(DEFCON_ERR_LIMIT, "x larger than 4 GiB (32-bit byte offsets)");
    g->M = (int)M;
    const int vec = dtype == DEFCON_BF16 ? 8 : 4;
    if (g->Cg % vec != 0)
        return fail(DEFCON_ERR_UNSUPPORTED, "Cin/G = %d must be a multiple of %d for this dtype",
                    g->Cg, vec);
    return DEFCON_OK;
}

enum class Path { SIMT_F32, SIMT_BF16, TC_BF16, TC_F32 };

static int select_path(const DcnGeom& g, int dtype, int sampler, int fp32_mode, Path* path) {
    if (sampler != DEFCON_SAMPLER_LDG && sampler != DEFCON_SAMPLER_TEX && sampler != DEFCON_SAMPLER_HYBRID)
        return fail(DEFCON_ERR_INVALID_ARG, "bad sampler");
    if (fp32_mode != DEFCON_FP32_3XTF32 && fp32_mode != DEFCON_FP32_SIMT)
        return fail(DEFCON_ERR_INVALID_ARG, "bad fp32_mode");
    if (sampler == DEFCON_SAMPLER_TEX || sampler == DEFCON_SAMPLER_HYBRID) {
        if (dtype != DEFCON_BF16 || !dcn_tc_bf16_supported(g))
            return fail(DEFCON_ERR_UNSUPPORTED,
                        "texture sampler is built for the bf16 tensor-core path (Cin/G %% 64 == 0)");
        *path = Path::TC_BF16;
        return DEFCON_OK;
    }
    if (dtype == DEFCON_BF16) {
        *path = dcn_tc_bf16_supported(g) ? Path::TC_BF16 : Path::SIMT_BF16;
    } else {
        if (fp32_mode == DEFCON_FP32_3XTF32) {
            if (!dcn_tc_f32_supported(g))
                return fail(DEFCON_ERR_UNSUPPORTED,
                            "3xTF32 tensor-core path needs Cin/G %% 32 == 0 and Cout %% 16 == 0");
            *path = Path::TC_F32;
        } else {
            *path = Path::SIMT_F32;
        }
    }
    return DEFCON_OK;
}

static size_t path_workspace(const DcnGeom& g, Path path) {
    return path == Path::TC_BF16 ? dcn_tc_bf16_workspace(g) : path == Path::TC_F32 ? dcn_tc_f32_workspace(g) : 0;
}
// The workspace byte range [*off, *off + *bytes) that must be zero before a launch.
static void path_workspace_counters(const DcnGeom& g, Path path, size_t* off, size_t* bytes) {
    *off = 0;
    *bytes = 0;
    if (path == Path::TC_BF16) dcn_tc_bf16_workspace_counters(g, off, bytes);
    if (path == Path::TC_F32) dcn_tc_f32_workspace_counters(g, off, bytes);
}

}  // namespace defcon

using namespace defcon;

extern "C" {

const char* defcon_status_string(int status) {
    switch (status) {
        case DEFCON_OK: return "DEFCON_OK";
        case DEFCON_ERR_INVALID_ARG: return "DEFCON_ERR_INVALID_ARG";
        case DEFCON_ERR_UNSUPPORTED: return "DEFCON_ERR_UNSUPPORTED";
        case DEFCON_ERR_MISALIGNED: return "DEFCON_ERR_MISALIGNED";
        case DEFCON_ERR_CUDA: return "DEFCON_ERR_CUDA";
        case DEFCON_ERR_LIMIT: return "DEFCON_ERR_LIMIT";
        default: return "DEFCON_ERR_UNKNOWN";
    }
}

const char* defcon_last_error_detail(void) { return g_detail; }

int defcon_abi_version(void) { return DEFCON_ABI_VERSION; }

static int branch_geom(int N, int H, int W, int C, int K, const defcon_conv_t& cv, int* Ho, int* Wo) {
    if (N <= 0 || H <= 0 || W <= 0 || C <= 0 || K <= 0)
        return fail(DEFCON_ERR_INVALID_ARG, "sizes must be positive");
    int rc = check_conv(cv);
    if (rc) return rc;
    *Ho = out_size(H, 3, cv.stride_h, cv.pad_h, cv.dil_h);
    *Wo = out_size(W, 3, cv.stride_w, cv.pad_w, cv.dil_w);
    if (*Ho <= 0 || *Wo <= 0) return fail(DEFCON_ERR_INVALID_ARG, "output grid is empty");
    if (C % 8 != 0) return fail(DEFCON_ERR_UNSUPPORTED, "offset branch needs C %% 8 == 0 (C = %d)", C);
    if ((long)N * H * W * C >= (1L << 31) || (long)N * *Ho * *Wo * C >= (1L << 31))
        return fail(DEFCON_ERR_LIMIT, "tensor too large for 32-bit element indexing");
    return DEFCON_OK;
}

int defcon_offset_workspace_size(int N, int H, int W, int C, int K, defcon_conv_t cv, size_t* bytes) {
    g_detail[0] = 0;
    if (!bytes) return fail(DEFCON_ERR_INVALID_ARG, "bytes is NULL");
    int Ho, Wo;
    int rc = branch_geom(N, H, W, C, K, cv, &Ho, &Wo);
    if (rc) return rc;
    size_t b[2];
    for (int bf = 0; bf < 2; ++bf)   // x's dtype is not an argument here: cover both
        b[bf] = offset_branch_workspace(N, H, W, C, Ho, Wo, K, cv.offset_groups, cv.stride_h, cv.stride_w,
                                        cv.pad_h, cv.pad_w, cv.dil_h, cv.dil_w, bf == 1);
    *bytes = std::max(b[0], b[1]);
    return DEFCON_OK;
}

int defcon_offset_dw_conv(const void* x, int N, int H, int W, int C, int x_dtype,
                          const float* dw_w, const float* dw_scale, const float* dw_shift,
                          const float* pw_w, const float* pw_b, int K, defcon_conv_t cv,
                          float* offset, float* mask, void* workspace, size_t workspace_bytes,
                          void* stream) {
    g_detail[0] = 0;
    int Ho, Wo;
    int rc = branch_geom(N, H, W, C, K, cv, &Ho, &Wo);
    if (rc) return rc;
    if (x_dtype != DEFCON_F32 && x_dtype != DEFCON_BF16) return fail(DEFCON_ERR_INVALID_ARG, "bad dtype");
    if (!x || !dw_w || !dw_scale || !dw_shift || !pw_w || !offset)
        return fail(DEFCON_ERR_INVALID_ARG, "NULL tensor pointer");
    const void* ptrs[] = {x, dw_w, dw_scale, dw_shift, pw_w, pw_b, offset, mask, workspace};
    for (const void* p : ptrs)
        if (p && !aligned16(p)) return fail(DEFCON_ERR_MISALIGNED, "tensor pointer not 16-byte aligned");
    const int G = cv.offset_groups;
    const int OC = G * K * K * (mask ? 3 : 2);
    if (OC > 256) return fail(DEFCON_ERR_LIMIT, "offset branch OC = %d > 256", OC);
    if ((long)N * Ho * Wo * OC >= (1L << 31))
        return fail(DEFCON_ERR_LIMIT, "tensor too large for 32-bit element indexing");
    const size_t need = offset_branch_workspace(N, H, W, C, Ho, Wo, K, cv.offset_groups, cv.stride_h, cv.stride_w,
                                                cv.pad_h, cv.pad_w, cv.dil_h, cv.dil_w, x_dtype == DEFCON_BF16);
    if (workspace_bytes < need || (need && !workspace))
        return fail(DEFCON_ERR_LIMIT, "workspace of %zu bytes < required %zu", workspace_bytes, need);
    cudaError_t e = launch_offset_branch(x, x_dtype == DEFCON_BF16, N, H, W, C, dw_w, dw_scale,
                                         dw_shift, pw_w, pw_b, K, G, mask != nullptr, cv.stride_h,
                                         cv.stride_w, cv.pad_h, cv.pad_w, cv.dil_h, cv.dil_w, Ho, Wo,
                                         offset, mask, static_cast<float*>(workspace),
                                         static_cast<cudaStream_t>(stream), cv.offset_dtype == DEFCON_F16);
    if (e == cudaErrorInvalidValue) return fail(DEFCON_ERR_LIMIT, "offset branch OC = %d unsupported", OC);
    if (e != cudaSuccess) return cuda_fail(e, "offset_branch launch");
    return DEFCON_OK;
}

int defcon_offset_packed_size(int C, int K, int offset_groups, int modulated, size_t* bytes) {
    g_detail[0] = 0;
    if (!bytes) return fail(DEFCON_ERR_INVALID_ARG, "bytes is NULL");
    if (C <= 0 || K <= 0 || offset_groups <= 0) return fail(DEFCON_ERR_INVALID_ARG, "sizes must be positive");
    if (C % 8 != 0) return fail(DEFCON_ERR_UNSUPPORTED, "offset branch needs C %% 8 == 0 (C = %d)", C);
    const int OC = offset_groups * K * K * (modulated ? 3 : 2);
    if (OC > 256) return fail(DEFCON_ERR_LIMIT, "offset branch OC = %d > 256", OC);
    *bytes = offset_branch_onepass_workspace(C, OC);
    return DEFCON_OK;
}

int defcon_offset_pack_params(int C, int K, int offset_groups, int modulated, const float* dw_w,
                              const float* dw_scale, const float* dw_shift, const float* pw_w, void* packed,
                              size_t packed_bytes, void* stream) {
    size_t need = 0;
    int rc = defcon_offset_packed_size(C, K, offset_groups, modulated, &need);
    if (rc) return rc;
    if (!dw_w || !dw_scale || !dw_shift || !pw_w || !packed) return fail(DEFCON_ERR_INVALID_ARG, "NULL pointer");
    const void* ptrs[] = {dw_w, dw_scale, dw_shift, pw_w, packed};
    for (const void* p : ptrs)
        if (!aligned16(p)) return fail(DEFCON_ERR_MISALIGNED, "pointer not 16-byte aligned");
    if (packed_bytes < need) return fail(DEFCON_ERR_LIMIT, "packed buffer of %zu bytes < required %zu", packed_bytes, need);
    const int OC = offset_groups * K * K * (modulated ? 3 : 2);
    cudaError_t e = launch_offset_pack(dw_w, dw_scale, dw_shift, pw_w, C, OC, packed, static_cast<cudaStream_t>(stream));
    if (e != cudaSuccess) return cuda_fail(e, "offset parameter pack launch");
    return DEFCON_OK;
}

int defcon_offset_dw_conv_packed(const void* x, int N, int H, int W, int C, int x_dtype, const void* packed,
                                 size_t packed_bytes, const float* pw_b, int K, defcon_conv_t cv, float* offset,
                                 float* mask, void* stream) {
    g_detail[0] = 0;
    int Ho, Wo;
    int rc = branch_geom(N, H, W, C, K, cv, &Ho, &Wo);
    if (rc) return rc;
    if (x_dtype != DEFCON_F32 && x_dtype != DEFCON_BF16) return fail(DEFCON_ERR_INVALID_ARG, "bad dtype");
    if (!x || !packed || !offset) return fail(DEFCON_ERR_INVALID_ARG, "NULL tensor pointer");
    const void* ptrs[] = {x, packed, pw_b, offset, mask};
    for (const void* p : ptrs)
        if (p && !aligned16(p)) return fail(DEFCON_ERR_MISALIGNED, "tensor pointer not 16-byte aligned");
    const int G = cv.offset_groups;
    const int OC = G * K * K * (mask ? 3 : 2);
    if (OC > 256) return fail(DEFCON_ERR_LIMIT, "offset branch OC = %d > 256", OC);
    if ((long)N * Ho * Wo * OC >= (1L << 31))
        return fail(DEFCON_ERR_LIMIT, "tensor too large for 32-bit element indexing");
    if (!offset_branch_is_onepass(N, H, W, C, Ho, Wo, K, G, cv.stride_h, cv.stride_w, cv.pad_h, cv.pad_w, cv.dil_h,
                                  cv.dil_w, x_dtype == DEFCON_BF16))
        return fail(DEFCON_ERR_UNSUPPORTED, "this shape runs the two-launch branch: use defcon_offset_dw_conv");
    if (packed_bytes < offset_branch_onepass_workspace(C, OC))
        return fail(DEFCON_ERR_LIMIT, "packed buffer of %zu bytes < required %zu", packed_bytes,
                    offset_branch_onepass_workspace(C, OC));
    cudaError_t e = launch_offset_branch(x, x_dtype == DEFCON_BF16, N, H, W, C, nullptr, nullptr, nullptr, nullptr,
                                         pw_b, K, G, mask != nullptr, cv.stride_h, cv.stride_w, cv.pad_h, cv.pad_w,
                                         cv.dil_h, cv.dil_w, Ho, Wo, offset, mask,
                                         static_cast<float*>(const_cast<void*>(packed)),
                                         static_cast<cudaStream_t>(stream), cv.offset_dtype == DEFCON_F16, true);
    if (e == cudaErrorInvalidValue) return fail(DEFCON_ERR_LIMIT, "offset branch OC = %d unsupported", OC);
    if (e != cudaSuccess) return cuda_fail(e, "offset_branch launch");
    return DEFCON_OK;
}

int defcon_dcn_workspace_size(int N, int H, int W, int Cin, int Cout, int Kh, int Kw,
                              defcon_conv_t cv, int dtype, int sampler, int fp32_mode,
                              size_t* bytes) {
    g_detail[0] = 0;
    if (!bytes) return fail(DEFCON_ERR_INVALID_ARG, "bytes is NULL");
    DcnGeom g;
    int rc = make_geom(N, H, W, Cin, Cout, Kh, Kw, cv, dtype, &g);
    if (rc) return rc;
    Path path;
    rc = select_path(g, dtype, sampler, fp32_mode, &path);
    if (rc) return rc;
    *bytes = path_workspace(g, path);
    return DEFCON_OK;
}

int defcon_dcn_forward(const void* x, int N, int H, int W, int Cin, const float* offset,
                       const float* mask, const void* weight, const float* bias, int Cout, int Kh,
                       int Kw, defcon_conv_t cv, int dtype, int sampler, int fp32_mode, void* y,
                       void* workspace, size_t workspace_bytes, defcon_tex_plan_t tex_plan,
                       void* stream) {
    g_detail[0] = 0;
    DcnGeom g;
    int rc = make_geom(N, H, W, Cin, Cout, Kh, Kw, cv, dtype, &g);
    if (rc) return rc;
    if (!x || !offset || !weight || !y) return fail(DEFCON_ERR_INVALID_ARG, "NULL tensor pointer");
    const void* ptrs[] = {x, offset, mask, weight, bias, y, workspace};
    for (const void* p : ptrs)
        if (p && !aligned16(p)) return fail(DEFCON_ERR_MISALIGNED, "tensor pointer not 16-byte aligned");
    Path path;
    rc = select_path(g, dtype, sampler, fp32_mode, &path);
    if (rc) return rc;
    // the tensor-core producers gather x with 32-byte vector loads (ld.global.nc.v8)
    if ((path == Path::TC_BF16 || path == Path::TC_F32) && !aligned32(x))
        return fail(DEFCON_ERR_MISALIGNED, "x must be 32-byte aligned for the tensor-core path");
    TexPlan* tp = nullptr;
    if (sampler == DEFCON_SAMPLER_TEX || sampler == DEFCON_SAMPLER_HYBRID) {
        tp = reinterpret_cast<TexPlan*>(tex_plan);
        if (!tex_plan_matches(tp, N, H, W, Cin, dtype == DEFCON_BF16))
            return fail(DEFCON_ERR_INVALID_ARG, "tex_plan missing or made for another shape/dtype");
    }
    const size_t need = path_workspace(g, path);
    if (need > 0 && (workspace == nullptr || workspace_bytes < need))
        return fail(DEFCON_ERR_LIMIT, "workspace of %zu bytes < required %zu", workspace_bytes, need);
    DcnPtrs p{x, offset, mask, weight, bias, y};
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    cudaError_t e;
    const char* detail = "dcn launch";
    if (tp) {
        e = tex_plan_stage(tp, x, st);
        if (e != cudaSuccess) return cuda_fail(e, "texture staging launch");
    }
    switch (path) {
        case Path::TC_BF16: e = launch_dcn_tc_bf16(g, p, workspace, workspace_bytes, tp,
                                                   sampler == DEFCON_SAMPLER_HYBRID, st, &detail); break;
        case Path::TC_F32: e = launch_dcn_tc_f32(g, p, workspace, workspace_bytes, st, &detail); break;
        case Path::SIMT_BF16: e = launch_dcn_simt(g, p, true, st); break;
        default: e = launch_dcn_simt(g, p, false, st); break;
    }
    if (e != cudaSuccess) return cuda_fail(e, detail);
    return DEFCON_OK;
}

int defcon_deform_columns(const void* x, int N, int H, int W, int Cin, const float* offset,
                          const float* mask, int Kh, int Kw, defcon_conv_t cv, int dtype, void* columns,
                          void* stream) {
    g_detail[0] = 0;
    DcnGeom g;
    int rc = make_geom(N, H, W, Cin, 1, Kh, Kw, cv, dtype, &g);
    if (rc) return rc;
    if (!x || !offset || !columns) return fail(DEFCON_ERR_INVALID_ARG, "NULL tensor pointer");
    const void* ptrs[] = {x, offset, mask, columns};
    for (const void* p : ptrs)
        if (p && !aligned16(p)) return fail(DEFCON_ERR_MISALIGNED, "tensor pointer not 16-byte aligned");
    if (!aligned32(x) || !aligned32(columns))   // 32-byte vector gathers and stores
        return fail(DEFCON_ERR_MISALIGNED, "x and columns must be 32-byte aligned");
    if ((long)g.M * g.KK * Cin >= (1L << 31))
        return fail(DEFCON_ERR_LIMIT, "column matrix too large for 32-bit element indexing");
    const int vec = dtype == DEFCON_BF16 ? 16 : 8;     // 32-byte pieces within one offset group
    if (g.Cg % vec != 0)
        return fail(DEFCON_ERR_UNSUPPORTED, "columns need Cin/G %% %d == 0 for this dtype", vec);
    cudaError_t e = launch_deform_columns(g, x, offset, mask, dtype == DEFCON_BF16, columns,
                                          static_cast<cudaStream_t>(stream));
    if (e != cudaSuccess) return cuda_fail(e, "deform_columns launch");
    return DEFCON_OK;
}

// ---------------------------------------------------------------- end-to-end host entry
static size_t align_up(size_t v) { return (v + 255) & ~size_t(255); }

// The host entry point pipelines the batch: images are independent, so the batch
// is cut into nchunk image ranges that flow H2D -> step 1 -> step 2 -> D2H on two internal
// streams, and the copy engines (one per direction) overlap with the kernels of the other
// chunk.  Device workspace: x and y for the whole batch (image slices stay 16-byte aligned),
// offsets / mask per chunk (their per-image size is not a 16-byte multiple), and one step-2
// workspace + one offset-branch workspace per internal stream.
constexpr int HOST_PIPE_STREAMS = 2;

static int host_chunks(int N) {
    int k = N < 4 ? N : 4;
    if (const char* env = getenv("DEFCON_HOST_CHUNKS")) {
        const int v = atoi(env);
        if (v > 0) k = v < N ? v : N;
    }
    k = k < 16 ? k : 16;   // HOST_MAX_CHUNKS
    return k > 0 ? k : 1;
}

struct LayerCarve {
    int nchunk, per;                    // chunks, images per chunk (last may be short)
    size_t xy, ws, tws, total;          // xy = per-chunk x, y, offset and mask regions
    size_t ctr_off, ctr_bytes;          // step-2 workspace bytes that must start at zero
};

// Per-chunk device regions of the host entry, each 256-byte aligned (so every chunk's x and y
// meet the kernels' alignment rules whatever the per-image sizes are).
struct ChunkCarve {
    size_t x, y, off, msk;   // region sizes
    size_t total() const { return x + y + off + msk; }
};

static ChunkCarve chunk_carve(const DcnGeom& g, int dtype, int Cout, int modulated, int nc) {
    const size_t es = dtype == DEFCON_BF16 ? 2 : 4;
    const size_t hw = (size_t)g.Ho * g.Wo;
    ChunkCarve c;
    c.x = align_up((size_t)nc * g.H * g.W * g.Cin * es);
    c.y = align_up((size_t)nc * hw * Cout * es);
    const size_t oes = g.off_f16 ? 2 : 4;   // offsets / mask element bytes
    c.off = align_up((size_t)nc * hw * g.G * g.KK * 2 * oes);
    c.msk = modulated ? align_up((size_t)nc * hw * g.G * g.KK * oes) : 0;
    return c;
}

static int layer_carve(int N, int H, int W, int Cin, int dtype, int Cout, int K,
                       const defcon_conv_t& cv, int modulated, int sampler, int fp32_mode,
                       DcnGeom* g, LayerCarve* c) {
    int rc = make_geom(N, H, W, Cin, Cout, K, K, cv, dtype, g);
    if (rc) return rc;
    Path path;
    rc = select_path(*g, dtype, sampler, fp32_mode, &path);
    if (rc) return rc;
    // the host entry owns no texture plan: texture samplers are device-entry only
    if (sampler != DEFCON_SAMPLER_LDG)
        return fail(DEFCON_ERR_UNSUPPORTED, "the host entry point supports DEFCON_SAMPLER_LDG only");
    c->nchunk = host_chunks(N);
    c->per = (N + c->nchunk - 1) / c->nchunk;
    c->nchunk = (N + c->per - 1) / c->per;
    c->xy = 0;
    for (int k = 0; k < c->nchunk; ++k)
        c->xy += chunk_carve(*g, dtype, Cout, modulated, std::min(c->per, N - k * c->per)).total();
    // step-2 / branch workspaces sized for the full batch cover every chunk
    c->ws = align_up(path_workspace(*g, path));
    path_workspace_counters(*g, path, &c->ctr_off, &c->ctr_bytes);
    c->tws = align_up(offset_branch_workspace(N, H, W, Cin, g->Ho, g->Wo, K, g->G, cv.stride_h, cv.stride_w, cv.pad_h,
                                              cv.pad_w, cv.dil_h, cv.dil_w, dtype == DEFCON_BF16));
    c->total = c->xy + HOST_PIPE_STREAMS * (c->ws + c->tws);
    return DEFCON_OK;
}

int defcon_layer_workspace_size(int N, int H, int W, int Cin, int dtype, int Cout, int K,
                                defcon_conv_t cv, int modulated, int sampler, int fp32_mode,
                                size_t* bytes) {
    g_detail[0] = 0;
    if (!bytes) return fail(DEFCON_ERR_INVALID_ARG, "bytes is NULL");
    DcnGeom g;
    LayerCarve c;
    int rc = layer_carve(N, H, W, Cin, dtype, Cout, K, cv, modulated, sampler, fp32_mode, &g, &c);
    if (rc) return rc;
    *bytes = c.total;
    return DEFCON_OK;
}

// Internal streams and events, created once per process on first use (the only resources the
// host entry point keeps); calls are serialised by a mutex.  Copies have streams of their own
// (one host-to-device, one device-to-host, each in chunk order) so the copy engines stream
// back to back while the compute streams work on earlier chunks; per-chunk events link them.
constexpr int HOST_MAX_CHUNKS = 16;
struct HostPipe {
    int dev = -1;
    cudaStream_t s[HOST_PIPE_STREAMS] = {};   // compute
    cudaStream_t h2d = nullptr, d2h = nullptr;
    cudaEvent_t start = nullptr, done[HOST_PIPE_STREAMS] = {}, h2d_done = nullptr, d2h_done = nullptr;
    cudaEvent_t in[HOST_MAX_CHUNKS] = {}, out[HOST_MAX_CHUNKS] = {};   // chunk k landed / computed
};
static std::mutex g_pipe_mu;
static HostPipe g_pipe;

static cudaError_t host_pipe_ready() {
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    if (g_pipe.dev == dev) return cudaSuccess;
    HostPipe p;
    p.dev = dev;
    for (int i = 0; i < HOST_PIPE_STREAMS; ++i) {
        if ((e = cudaStreamCreateWithFlags(&p.s[i], cudaStreamNonBlocking)) != cudaSuccess) return e;
        if ((e = cudaEventCreateWithFlags(&p.done[i], cudaEventDisableTiming)) != cudaSuccess) return e;
    }
    if ((e = cudaEventCreateWithFlags(&p.start, cudaEventDisableTiming)) != cudaSuccess) return e;
    if ((e = cudaStreamCreateWithFlags(&p.h2d, cudaStreamNonBlocking)) != cudaSuccess) return e;
    if ((e = cudaStreamCreateWithFlags(&p.d2h, cudaStreamNonBlocking)) != cudaSuccess) return e;
    if ((e = cudaEventCreateWithFlags(&p.h2d_done, cudaEventDisableTiming)) != cudaSuccess) return e;
    if ((e = cudaEventCreateWithFlags(&p.d2h_done, cudaEventDisableTiming)) != cudaSuccess) return e;
    for (int k = 0; k < HOST_MAX_CHUNKS; ++k) {
        if ((e = cudaEventCreateWithFlags(&p.in[k], cudaEventDisableTiming)) != cudaSuccess) return e;
        if ((e = cudaEventCreateWithFlags(&p.out[k], cudaEventDisableTiming)) != cudaSuccess) return e;
    }
    g_pipe = p;   // a previous device's objects are left to process teardown
    return cudaSuccess;
}

int defcon_layer_forward_host(const void* x_host, int N, int H, int W, int Cin, int dtype,
                              const float* dw_w, const float* dw_scale, const float* dw_shift,
                              const float* pw_w, const float* pw_b, const void* weight,
                              const float* bias, int Cout, int K, defcon_conv_t cv, int modulated,
                              int sampler, int fp32_mode, void* y_host, void* dev_workspace,
                              size_t dev_workspace_bytes, void* stream) {
    g_detail[0] = 0;
    if (!x_host || !y_host || !dev_workspace) return fail(DEFCON_ERR_INVALID_ARG, "NULL pointer");
    DcnGeom g;
    LayerCarve c;
    int rc = layer_carve(N, H, W, Cin, dtype, Cout, K, cv, modulated, sampler, fp32_mode, &g, &c);
    if (rc) return rc;
    if (dev_workspace_bytes < c.total)
        return fail(DEFCON_ERR_LIMIT, "device workspace %zu < required %zu", dev_workspace_bytes, c.total);
    if (out_size(H, 3, cv.stride_h, cv.pad_h, cv.dil_h) != g.Ho ||
        out_size(W, 3, cv.stride_w, cv.pad_w, cv.dil_w) != g.Wo)
        return fail(DEFCON_ERR_INVALID_ARG, "offset-branch grid differs from the DCN grid");
    std::lock_guard<std::mutex> lock(g_pipe_mu);
    cudaError_t e = host_pipe_ready();
    if (e != cudaSuccess) return cuda_fail(e, "host pipeline streams");
    uint8_t* cur = static_cast<uint8_t*>(dev_workspace);
    uint8_t* wsbase = cur + c.xy;
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    const size_t es = dtype == DEFCON_BF16 ? 2 : 4;
    const size_t hw = (size_t)g.Ho * g.Wo;
    const size_t x_img = (size_t)H * W * Cin * es, y_img = hw * Cout * es;
    // order the pipeline after the caller's prior work on `stream`
    if ((e = cudaEventRecord(g_pipe.start, st)) != cudaSuccess) return cuda_fail(e, "event record");
    for (int i = 0; i < HOST_PIPE_STREAMS; ++i)
        if ((e = cudaStreamWaitEvent(g_pipe.s[i], g_pipe.start, 0)) != cudaSuccess) return cuda_fail(e, "event wait");
    if ((e = cudaStreamWaitEvent(g_pipe.h2d, g_pipe.start, 0)) != cudaSuccess) return cuda_fail(e, "event wait");
    if ((e = cudaStreamWaitEvent(g_pipe.d2h, g_pipe.start, 0)) != cudaSuccess) return cuda_fail(e, "event wait");
    // Any failure after the first enqueue: drain the internal streams before returning, so no
    // copy still reads x_host / writes y_host once the caller sees the error.
    auto bail = [&](int status) {
        for (int i = 0; i < HOST_PIPE_STREAMS; ++i) cudaStreamSynchronize(g_pipe.s[i]);
        cudaStreamSynchronize(g_pipe.h2d);
        cudaStreamSynchronize(g_pipe.d2h);
        return status;
    };
    // per-range device regions
    struct Range {
        uint8_t *x, *y;
        float *off, *msk;
        int n0, nc;
    } rg[HOST_MAX_CHUNKS];
    for (int k = 0; k < c.nchunk; ++k) {
        Range& r = rg[k];
        r.n0 = k * c.per;
        r.nc = std::min(c.per, N - r.n0);
        const ChunkCarve cc = chunk_carve(g, dtype, Cout, modulated, r.nc);
        r.x = cur;
        r.y = r.x + cc.x;
        r.off = reinterpret_cast<float*>(r.y + cc.y);
        r.msk = modulated ? reinterpret_cast<float*>(r.y + cc.y + cc.off) : nullptr;
        cur += cc.total();
    }
    // the caller's workspace carries no zero-fill guarantee: clear step 2's tile counters once
    // per compute stream (self-cleaning after every launch)
    for (int si = 0; si < HOST_PIPE_STREAMS && si < c.nchunk; ++si)
        if (c.ws && c.ctr_bytes) {
            e = cudaMemsetAsync(wsbase + si * (c.ws + c.tws) + c.ctr_off, 0, c.ctr_bytes, g_pipe.s[si]);
            if (e != cudaSuccess) return bail(cuda_fail(e, "workspace clear"));
        }
    // every host-to-device copy first, back to back on the copy stream
    for (int k = 0; k < c.nchunk; ++k) {
        e = cudaMemcpyAsync(rg[k].x, static_cast<const uint8_t*>(x_host) + rg[k].n0 * x_img, rg[k].nc * x_img,
                            cudaMemcpyHostToDevice, g_pipe.h2d);
        if (e == cudaSuccess) e = cudaEventRecord(g_pipe.in[k], g_pipe.h2d);
        if (e != cudaSuccess) return bail(cuda_fail(e, "H2D copy of x"));
    }
    for (int k = 0; k < c.nchunk; ++k) {
        const int si = k % HOST_PIPE_STREAMS;
        cudaStream_t s = g_pipe.s[si];
        const Range& r = rg[k];
        uint8_t* wsd = c.ws ? wsbase + si * (c.ws + c.tws) : nullptr;
        void* twsd = wsbase + si * (c.ws + c.tws) + c.ws;
        e = cudaStreamWaitEvent(s, g_pipe.in[k], 0);   // compute after the range's copy
        if (e != cudaSuccess) return bail(cuda_fail(e, "event wait"));
        rc = defcon_offset_dw_conv(r.x, r.nc, H, W, Cin, dtype, dw_w, dw_scale, dw_shift, pw_w, pw_b, K, cv,
                                   r.off, r.msk, twsd, c.tws, s);
        if (rc) return bail(rc);
        rc = defcon_dcn_forward(r.x, r.nc, H, W, Cin, r.off, r.msk, weight, bias, Cout, K, K, cv, dtype,
                                sampler, fp32_mode, r.y, wsd, c.ws, nullptr, s);
        if (rc) return bail(rc);
        e = cudaEventRecord(g_pipe.out[k], s);
        if (e == cudaSuccess) e = cudaStreamWaitEvent(g_pipe.d2h, g_pipe.out[k], 0);   // copy after the compute
        if (e == cudaSuccess)
            e = cudaMemcpyAsync(static_cast<uint8_t*>(y_host) + r.n0 * y_img, r.y, r.nc * y_img,
                                cudaMemcpyDeviceToHost, g_pipe.d2h);
        if (e != cudaSuccess) return bail(cuda_fail(e, "D2H copy of y"));
    }
    for (int i = 0; i < HOST_PIPE_STREAMS; ++i) {
        if ((e = cudaEventRecord(g_pipe.done[i], g_pipe.s[i])) != cudaSuccess) return bail(cuda_fail(e, "event record"));
        if ((e = cudaStreamWaitEvent(st, g_pipe.done[i], 0)) != cudaSuccess) return bail(cuda_fail(e, "event wait"));
    }
    if ((e = cudaEventRecord(g_pipe.h2d_done, g_pipe.h2d)) != cudaSuccess ||
        (e = cudaStreamWaitEvent(st, g_pipe.h2d_done, 0)) != cudaSuccess ||
        (e = cudaEventRecord(g_pipe.d2h_done, g_pipe.d2h)) != cudaSuccess ||
        (e = cudaStreamWaitEvent(st, g_pipe.d2h_done, 0)) != cudaSuccess)
        return bail(cuda_fail(e, "event record / wait"));
    e = cudaStreamSynchronize(st);
    if (e != cudaSuccess) return bail(cuda_fail(e, "stream synchronize"));
    return DEFCON_OK;
}

int defcon_tex_plan_create(int N, int H, int W, int Cin, int dtype, defcon_tex_plan_t* plan) {
    g_detail[0] = 0;
    if (!plan) return fail(DEFCON_ERR_INVALID_ARG, "plan is NULL");
    *plan = nullptr;
    if (N <= 0 || H <= 0 || W <= 0 || Cin <= 0) return fail(DEFCON_ERR_INVALID_ARG, "sizes must be positive");
    if (dtype != DEFCON_F32 && dtype != DEFCON_BF16) return fail(DEFCON_ERR_INVALID_ARG, "bad dtype");
    if (Cin % 4 != 0) return fail(DEFCON_ERR_UNSUPPORTED, "texture plan needs Cin %% 4 == 0");
    int dev = 0, max_layers = 2048, max_w = 32768, max_h = 32768;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&max_layers, cudaDevAttrMaxTexture2DLayeredLayers, dev);
    cudaDeviceGetAttribute(&max_w, cudaDevAttrMaxTexture2DLayeredWidth, dev);
    cudaDeviceGetAttribute(&max_h, cudaDevAttrMaxTexture2DLayeredHeight, dev);
    if (Cin / 4 > max_layers || W > max_w || (long)N * (H + 1) > max_h)
        return fail(DEFCON_ERR_LIMIT, "layered texture limits exceeded (layers %d / %d, %d x %ld texels)",
                    Cin / 4, max_layers, W, (long)N * (H + 1));
    TexPlan* p = nullptr;
    cudaError_t e = tex_plan_create(N, H, W, Cin, dtype == DEFCON_BF16, &p);
    if (e != cudaSuccess) return cuda_fail(e, "texture plan allocation");
    *plan = reinterpret_cast<defcon_tex_plan_t>(p);
    return DEFCON_OK;
}

int defcon_tex_plan_destroy(defcon_tex_plan_t plan) {
    tex_plan_destroy(reinterpret_cast<TexPlan*>(plan));
    return DEFCON_OK;
}

int defcon_tex_filter_probe(const float* px, const float* py, float* out, int n, void* stream) {
    g_detail[0] = 0;
    if (!px || !py || !out || n <= 0) return fail(DEFCON_ERR_INVALID_ARG, "bad probe arguments");
    cudaError_t e = tex_filter_probe(px, py, out, n, static_cast<cudaStream_t>(stream));
    if (e != cudaSuccess) return cuda_fail(e, "texture filter probe");
    return DEFCON_OK;
}

}  // extern "C"
