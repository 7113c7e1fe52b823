// kernels.h -- internal host-side launch interface between api.cu and the
// kernel translation units.  Not part of the public C ABI (include/defcon.h).
#pragma once

#include <cuda.h>
#include <cuda_runtime.h>
#include <stddef.h>
#include <stdint.h>

namespace defcon {

// Geometry of one deformable-conv launch (all validated by api.cu).
struct DcnGeom {
    int N, H, W, Cin, Cout, Kh, Kw, Ho, Wo;
    int sh, sw, ph, pw, dh, dw;
    int G, Cg;   // offset groups, channels per group
    int M;       // N * Ho * Wo output pixels
    int KK;      // Kh * Kw taps
    float bound_h;   // bounded deformation half-window (P-1)/2 (R12); < 0: unbounded
    int off_f16;     // offsets / mask stored as binary16 (tex2D++, R13)
};

struct DcnPtrs {
    const void* x;
    const float* offset;
    const float* mask;   // nullptr => DCNv1
    const void* weight;
    const float* bias;   // nullptr => 0
    void* y;
};

// ---- step 1: lightweight offset branch (offset_branch.cu)
cudaError_t launch_offset_branch(const void* x, bool x_bf16, int N, int H, int W, int C,
                                 const float* dw_w, const float* dw_scale, const float* dw_shift,
                                 const float* pw_w, const float* pw_b, int K, int G, bool with_mask,
                                 int s_h, int s_w, int p_h, int p_w, int d_h, int d_w, int Ho, int Wo,
                                 float* offset, float* mask, float* t_ws, cudaStream_t stream,
                                 bool out_f16 = false, bool prepacked = false);
// true when step 1 runs as the one-pass kernel for this shape (its parameters can be pre-packed)
bool offset_branch_is_onepass(int N, int H, int W, int C, int Ho, int Wo, int K, int G, int sh, int sw, int ph,
                              int pw, int dh, int dw, bool x_bf16);
// workspace of defcon_offset_dw_conv: the one-pass kernel's packed parameters when it can run
// this shape (decided for the widest branch, OC = 3*G*K*K), else the two-pass t buffers
size_t offset_branch_workspace(int N, int H, int W, int C, int Ho, int Wo, int K, int G, int sh, int sw, int ph,
                               int pw, int dh, int dw, bool x_bf16);
// one pass per tile (offset_branch_onepass.cu): TMA-staged dw on CUDA cores -> t as tf32 hi/lo
// operand planes in smem -> 1x1 on tcgen05 3xTF32; t never leaves the SM
bool offset_branch_onepass_plan(int N, int H, int W, int C, int Ho, int Wo, int sh, int sw, int ph, int pw,
                                int dh, int dw, int OC, bool x_bf16);
size_t offset_branch_onepass_workspace(int C, int OC);   // packed per-chunk parameter blocks
cudaError_t launch_offset_branch_onepass(const void* x, bool x_bf16, int N, int H, int W, int C,
                                         const float* dw_w, const float* dw_scale, const float* dw_shift,
                                         const float* pw_w, const float* pw_b, int n_off, int n_msk,
                                         int s_h, int s_w, int p_h, int p_w, int d_h, int d_w, int Ho, int Wo,
                                         float* offset, float* mask, void* ws, cudaStream_t stream,
                                         bool out_f16, bool prepacked = false);
cudaError_t launch_offset_pack(const float* dw_w, const float* dw_scale, const float* dw_shift, const float* pw_w,
                               int C, int OC, void* packed, cudaStream_t stream);
// ---- sampling step alone: deformable columns [M][KK*Cin] (sampler.cu)
cudaError_t launch_deform_columns(const DcnGeom& g, const void* x, const float* offset, const float* mask,
                                  bool bf16, void* cols, cudaStream_t stream);

// ---- step 2, CUDA-core anchor (dcn_simt.cu): fp32 math for fp32 or bf16 storage
cudaError_t launch_dcn_simt(const DcnGeom& g, const DcnPtrs& p, bool bf16, cudaStream_t stream);

// ---- step 2, fused gather + tcgen05 implicit GEMM, bf16 (dcn_tc_bf16.cu)
bool dcn_tc_bf16_supported(const DcnGeom& g);
size_t dcn_tc_bf16_workspace(const DcnGeom& g);   // stream-K counters + fp32 partials
void dcn_tc_bf16_workspace_counters(const DcnGeom& g, size_t* offset, size_t* bytes);   // must start at zero
struct TexPlan;
cudaError_t launch_dcn_tc_bf16(const DcnGeom& g, const DcnPtrs& p, void* ws, size_t ws_bytes,
                               const TexPlan* tex, bool hybrid, cudaStream_t stream, const char** detail);

// ---- step 2 on the tensor cores in fp32: kind::tf32 3xTF32 (same fused kernel, dcn_tc_bf16.cu)
bool dcn_tc_f32_supported(const DcnGeom& g);
size_t dcn_tc_f32_workspace(const DcnGeom& g);   // partials + counters + W's tf32 hi / lo planes
void dcn_tc_f32_workspace_counters(const DcnGeom& g, size_t* offset, size_t* bytes);
cudaError_t launch_dcn_tc_f32(const DcnGeom& g, const DcnPtrs& p, void* ws, size_t ws_bytes, cudaStream_t stream,
                              const char** detail);

// ---- texture sampler resources (tex_plan.cu)
struct TexPlan;
cudaError_t tex_plan_create(int N, int H, int W, int C, bool half, TexPlan** out);
void tex_plan_destroy(TexPlan* p);
bool tex_plan_matches(const TexPlan* p, int N, int H, int W, int C, bool half);
unsigned long long tex_plan_texture(const TexPlan* p);            // texture object handle
cudaError_t tex_plan_stage(const TexPlan* p, const void* x, cudaStream_t stream);
cudaError_t tex_filter_probe(const float* px, const float* py, float* out, int n, cudaStream_t stream);

// ---- driver entry point for cuTensorMapEncodeTiled (api.cu)
typedef CUresult (*PFN_encodeTiled)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*,
                                    const cuuint64_t*, const cuuint64_t*, const cuuint32_t*,
                                    const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                                    CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
PFN_encodeTiled get_encode_tiled();

}  // namespace defcon
