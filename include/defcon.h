/*
 * defcon.h -- C ABI of libdefcon.so, the B200 (sm_100a) implementation of the
 * DEFCON inference hot path (Jayaweera et al., IPDPSW 2024; /root/reference/PAPER.md).
 *
 * The path ("two-step" deformable convolution):
 *   step 1  defcon_offset_dw_conv  -- the paper's lightweight offset branch
 *           (P:170 W1 depthwise 3x3 -> P:180 BN + ReLU -> W2 1x1), producing the
 *           offsets (and the DCNv2 modulation mask, reading R6/R11 in DESIGN.md).
 *   step 2  defcon_dcn_forward     -- the deformable convolution, Eq.2 with
 *           the bilinear kernel Eq.3, zero outside the image,
 *           offset groups, optional DCNv2 mask.
 *
 * Conventions (all entry points):
 *  - Every tensor pointer is a DEVICE pointer owned by the caller unless the
 *    parameter name ends in _host (pinned host memory, also caller-owned).
 *    The library never allocates on the call path; its only owned resources are
 *    texture plans (defcon_tex_plan_create / _destroy) and the two streams the host
 *    entry point pipelines on (created once, see defcon_layer_forward_host).
 *  - Tensors are dense, row-major, channel-last (NHWC), with the layouts given per
 *    argument.  Every tensor pointer must be 16-byte aligned; x on the bf16 tensor-core
 *    path (Cin/G % 64 == 0) and x / columns of defcon_deform_columns must be 32-byte
 *    aligned (they are read / written with 32-byte vectors).  Violations return
 *    DEFCON_ERR_MISALIGNED before any launch.
 *  - `stream` is a cudaStream_t passed as void* (NULL = legacy default stream).
 *    Calls are asynchronous on that stream; no host synchronisation happens,
 *    except in defcon_layer_forward_host (see there).
 *  - Errors are returned as status codes, never as aborts or exceptions.  All
 *    argument checks happen before any launch; a failed launch returns
 *    DEFCON_ERR_CUDA.  defcon_last_error_detail() gives a thread-local message.
 *    Faults inside a kernel surface at the caller's next synchronisation.
 *  - There is no CPU fallback and no alternative backend: if the device cannot
 *    run the sm_100a kernels the call returns DEFCON_ERR_CUDA.
 *  - Output size: Ho = floor((H + 2*pad_h - dil_h*(Kh-1) - 1) / stride_h) + 1
 *    ("computed similarly to a regular convolution"), likewise Wo.
 */
#ifndef DEFCON_H_
#define DEFCON_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define DEFCON_ABI_VERSION 2   /* 2: defcon_conv_t.bound */

typedef enum {
    DEFCON_OK = 0,
    DEFCON_ERR_INVALID_ARG = 1,  /* shape / enum / pointer argument invalid        */
    DEFCON_ERR_UNSUPPORTED = 2,  /* valid, but this build has no kernel for it     */
    DEFCON_ERR_MISALIGNED = 3,   /* a tensor pointer is not 16- (or 32-) byte aligned */
    DEFCON_ERR_CUDA = 4,         /* a CUDA runtime call or kernel launch failed    */
    DEFCON_ERR_LIMIT = 5         /* exceeds an index / texture / workspace limit   */
} defcon_status_t;

typedef enum {
    DEFCON_F32 = 0,   /* x, weight, y stored as float32                         */
    DEFCON_BF16 = 1,  /* x, weight, y stored as bfloat16 (fp32 accumulation)    */
    DEFCON_F16 = 2    /* offsets / mask only (defcon_conv_t.offset_dtype): the
                         16-bit offsets of the paper's tex2D++ (R13)      */
} defcon_dtype_t;

typedef enum {
    DEFCON_SAMPLER_LDG = 0,  /* software bilinear: vectorised NHWC gathers, fp32 weights */
    DEFCON_SAMPLER_TEX = 1,  /* hardware bilinear: tex2DLayered, border (zero) addressing,
                                the paper's texel-based optimisation.  bf16 x
                                is staged as binary16 texels (CUDA has no bf16 texel
                                format): |x| > 65504 becomes inf and |x| < 2^-24 flushes
                                to 0, so x must lie in the binary16 range; the filter
                                rounds fractions and weights to 1/256 (reading R14)    */
    DEFCON_SAMPLER_HYBRID = 2 /* half of the A-producer warps use TEX, half LDG, so the
                                texture units and the FMA pipes work in parallel (SURVEY
                                section 8(f) NEXT 1); needs a tex_plan like TEX         */
} defcon_sampler_t;

typedef enum {
    DEFCON_FP32_3XTF32 = 0,  /* fp32 path on the tensor cores, 3 x TF32 split products  */
    DEFCON_FP32_SIMT = 1     /* fp32 path on CUDA cores (FFMA), the simple anchor        */
} defcon_fp32_mode_t;

/* Regular-conv geometry shared by both steps (reading R3) and the number of
 * offset (deformable) groups G: input channels [g*Cin/G, (g+1)*Cin/G) share
 * offset field g (reading R5). */
typedef struct {
    int stride_h, stride_w;
    int pad_h, pad_w;
    int dil_h, dil_w;
    int offset_groups;
    /* Bounded deformation (section III-A-c; reading R12): P > 0 restricts every offset
     * so that the sampling point of tap (i, j) stays in the P x P window centred on the output
     * pixel's centre tap: per axis, with r = (i - (Kh-1)/2) * dil_h (resp. j, Kw, dil_w) and
     * h = (P-1)/2, the offset d is used as clamp(r + d, -h, h) - r (NaN stays NaN).  The paper
     * picks P = 7 (Fig. 5).  0 = unbounded.  Read by the DCN / columns calls only. */
    int bound;
    /* Storage of the offset / mask tensors: DEFCON_F32 (0) or DEFCON_F16 -- tex2D++, "16 bits
     * to compute the offset" (reading R13): the branch writes them as binary16 (round
     * to nearest), the DCN reads them and forms the sampling coordinates in fp32. */
    int offset_dtype;
} defcon_conv_t;

/* Opaque texture plan: owns one layered cudaArray + texture object per image. */
typedef struct defcon_tex_plan_s* defcon_tex_plan_t;

/*
 * Step 1 -- lightweight offset branch (Eq.9 P:172 for its cost).
 *   t[c]  = max(0, dw_scale[c] * sum_{a,b<3} dw_w[c][a][b] * x[n][ho*s-p+a*d][wo*s-p+b*d][c]
 *                 + dw_shift[c])                  (zero padding; BN folded, R10)
 *   u[o]  = pw_b[o] + sum_c pw_w[o][c] * t[c]     (o < OC)
 *   offset[n][ho][wo][g][k][0..1] = u[g*2*K*K + 2*k + {0: dy, 1: dx}]          (R4)
 *   mask  [n][ho][wo][g][k]       = sigmoid(u[2*G*K*K + g*K*K + k])           (R6, R11)
 * Arguments
 *   x        [N][H][W][C], dtype x_dtype
 *   dw_w     [C][3][3] fp32;  dw_scale, dw_shift [C] fp32 (BN folded with the conv bias)
 *   pw_w     [OC][C] fp32, OC = G*K*K*(mask ? 3 : 2);  pw_b [OC] fp32 or NULL (= 0)
 *   K        kernel size of the deformable conv that consumes the offsets (taps K*K)
 *   cv       stride/pad/dil of the depthwise 3x3 conv (its output grid must be the
 *            DCN's Ho x Wo, R10) and G = cv.offset_groups
 *   offset   [N][Ho][Wo][G][K*K][2] fp32 (written)
 *   mask     [N][Ho][Wo][G][K*K] fp32 (written) or NULL (DCNv1: no mask rows)
 *   workspace  device scratch of defcon_offset_workspace_size() bytes (the fp32 t between the
 *            depthwise and the 1x1 launches; distinct per concurrently running call)
 * Errors: INVALID_ARG for non-positive sizes, Ho/Wo <= 0, G <= 0; UNSUPPORTED if
 *   C % 8 != 0 (16-byte channel vectors); LIMIT if OC > 256, a tensor needs >= 2^31
 *   elements or the workspace is too small; MISALIGNED for unaligned pointers.
 */
int defcon_offset_dw_conv(const void* x, int N, int H, int W, int C, int x_dtype,
                          const float* dw_w, const float* dw_scale, const float* dw_shift,
                          const float* pw_w, const float* pw_b, int K, defcon_conv_t cv,
                          float* offset, float* mask, void* workspace, size_t workspace_bytes,
                          void* stream);

/* Device workspace defcon_offset_dw_conv needs: the fp32 intermediate t as two planes (tf32 hi /
 * lo, 2*N*Ho*Wo*C*4 bytes) and the pointwise weights likewise (2*256*C*4 bytes). */
int defcon_offset_workspace_size(int N, int H, int W, int C, int K, defcon_conv_t cv,
                                 size_t* bytes);

/*
 * Step 1 with parameters packed once (inference: the branch weights are constants).
 * defcon_offset_pack_params writes dw_w / dw_scale / dw_shift / pw_w (same layouts as
 * defcon_offset_dw_conv, OC = offset_groups*K*K*(modulated ? 3 : 2)) as the per-32-channel
 * blocks the one-pass kernel streams (W2 as tf32 hi / lo in the tensor-core operand image, dw
 * taps and folded BN) into `packed` (defcon_offset_packed_size() bytes, caller-owned device
 * memory, 16-byte aligned); it is asynchronous on `stream`.  defcon_offset_dw_conv_packed then
 * computes exactly what defcon_offset_dw_conv computes from those parameters (bit-identical
 * results) without re-packing them per call; `packed` is only read, so one buffer serves
 * concurrent calls.  modulated must match (mask != NULL).
 * Errors: as defcon_offset_dw_conv; UNSUPPORTED for shapes that run the two-launch branch
 * (input rows wider than the one-pass kernel's TMA box; use defcon_offset_dw_conv there);
 * LIMIT if packed_bytes is too small.
 */
int defcon_offset_packed_size(int C, int K, int offset_groups, int modulated, size_t* bytes);
int defcon_offset_pack_params(int C, int K, int offset_groups, int modulated, const float* dw_w,
                              const float* dw_scale, const float* dw_shift, const float* pw_w,
                              void* packed, size_t packed_bytes, void* stream);
int defcon_offset_dw_conv_packed(const void* x, int N, int H, int W, int C, int x_dtype,
                                 const void* packed, size_t packed_bytes, const float* pw_b, int K,
                                 defcon_conv_t cv, float* offset, float* mask, void* stream);

/*
 * Step 2 -- deformable convolution forward, Eq.2 + Eq.3:
 *   y[n][ho][wo][co] = bias[co] + sum_{i<Kh, j<Kw, ci<Cin} weight[co][i][j][ci]
 *                      * m[n][ho][wo][g][k] * X(n, ci, p_y, p_x)
 *   k = i*Kw + j, g = ci / (Cin/G),
 *   p_y = ho*stride_h - pad_h + i*dil_h + offset[n][ho][wo][g][k][0]
 *   p_x = wo*stride_w - pad_w + j*dil_w + offset[n][ho][wo][g][k][1]
 *   X = bilinear interpolation of channel ci of image n at (p_y, p_x), with the four
 *       neighbours floor(p)+{0,1}; neighbours outside [0,H)x[0,W) contribute 0
 *   m = mask, or 1 when mask == NULL (DCNv1)
 * Arguments
 *   x        [N][H][W][Cin], dtype `dtype`
 *   offset   [N][Ho][Wo][G][Kh*Kw][2] fp32 (dy, dx);  mask [N][Ho][Wo][G][Kh*Kw] fp32 or NULL
 *   weight   [Cout][Kh][Kw][Cin], dtype `dtype`;  bias [Cout] fp32 or NULL (= 0)
 *   sampler  DEFCON_SAMPLER_LDG (any dtype), DEFCON_SAMPLER_TEX or DEFCON_SAMPLER_HYBRID
 *            (bf16 tensor-core path; require tex_plan made for the same N, H, W, Cin, dtype;
 *            the plan's array is (re)filled from x on `stream` by this call)
 *   fp32_mode  used only when dtype == DEFCON_F32
 *   y        [N][Ho][Wo][Cout], dtype `dtype` (written)
 *   workspace / workspace_bytes: device scratch of at least defcon_dcn_workspace_size()
 *            bytes (may be NULL when that size is 0).  The tensor-core path uses it for
 *            stream-K tile counters and fp32 partial tiles.  The workspace must be
 *            ZERO-FILLED before its first use (e.g. one cudaMemset after allocation); every
 *            completed call leaves its tile counters zero again, so no per-call reset is
 *            launched (graph-capture friendly).  The counters sit at the same offset for
 *            every shape (behind a partial-tile region of one device-wide size), so one
 *            zero-filled workspace serves any sequence of shapes whose
 *            defcon_dcn_workspace_size() it covers.  A call that faults or is aborted
 *            mid-kernel can leave counters non-zero: zero-fill again after an error.  Calls
 *            that may run concurrently need distinct workspaces.  The kernels are launched with programmatic dependent launch: their
 *            prologue may overlap the previous kernel on `stream`, never its data.
 * Errors: INVALID_ARG for non-positive sizes, Ho/Wo <= 0, G not dividing Cin, bad enums,
 *   NULL required pointers; UNSUPPORTED for (Cin/G) % 8 != 0 (bf16) or % 4 != 0 (fp32),
 *   or a Cout not multiple of 16 on the tensor-core paths; LIMIT when N*H*W*Cin >= 2^31,
 *   x spans >= 4 GiB (the samplers use 32-bit byte offsets) or the workspace is too small;
 *   MISALIGNED for pointers not 16-byte aligned, or x not
 *   32-byte aligned on the bf16 tensor-core path.
 */
int defcon_dcn_forward(const void* x, int N, int H, int W, int Cin,
                       const float* offset, const float* mask,
                       const void* weight, const float* bias, int Cout, int Kh, int Kw,
                       defcon_conv_t cv, int dtype, int sampler, int fp32_mode,
                       void* y, void* workspace, size_t workspace_bytes,
                       defcon_tex_plan_t tex_plan, void* stream);

/*
 * The sampling step alone -- the deformable im2col of the "two-step" formulation
 * (P:69-76), Eq.3 with the mask (R6), zero outside the image:
 *   columns[(n*Ho + ho)*Wo + wo][k*Cin + ci] = m[n][ho][wo][g][k] * X(n, ci, p_y, p_x)
 * with k, g, p_y, p_x exactly as in defcon_dcn_forward below.  y = columns . W^T + bias
 * (W viewed as [Cout][Kh*Kw*Cin]) is then the layer output: this is the unfused
 * baseline's first step and the measurement of the sampling stage on its own.
 * Arguments
 *   x        [N][H][W][Cin], dtype `dtype` (DEFCON_BF16 or DEFCON_F32)
 *   offset, mask  as in defcon_dcn_forward (mask may be NULL: DCNv1)
 *   columns  [N*Ho*Wo][Kh*Kw*Cin], dtype `dtype` (written; bf16 rounded to nearest even
 *            from the fp32 bilinear sum)
 * Ownership: caller owns every buffer; asynchronous on `stream`; no workspace.
 * Errors: as defcon_dcn_forward (INVALID_ARG, UNSUPPORTED for (Cin/G) % 16 (bf16) or % 8
 *   (fp32) != 0 -- 32-byte gathers --, LIMIT when the column matrix has >= 2^31 elements,
 *   MISALIGNED).
 */
int defcon_deform_columns(const void* x, int N, int H, int W, int Cin,
                          const float* offset, const float* mask, int Kh, int Kw,
                          defcon_conv_t cv, int dtype, void* columns, void* stream);

/* Device workspace defcon_dcn_forward needs for these arguments (0 if none). */
int defcon_dcn_workspace_size(int N, int H, int W, int Cin, int Cout, int Kh, int Kw,
                              defcon_conv_t cv, int dtype, int sampler, int fp32_mode,
                              size_t* bytes);

/*
 * Whole layer with HOST buffers (the end-to-end entry point): copies x_host (pinned)
 * to the device, runs step 1 and step 2, copies y back to y_host and synchronises
 * `stream` before returning.  Parameters dw_* / pw_* / weight / bias are device
 * pointers (resident model weights), as in the two calls above.  Images are independent
 * (P:58 is per output pixel), so the batch is cut into min(N, 4) image ranges
 * (DEFCON_HOST_CHUNKS overrides, at most 16) that flow H2D -> step 1 -> step 2 -> D2H,
 * ordered after the caller's prior work on `stream`: the host-to-device and the
 * device-to-host copies each run on an internal stream of their own, back to back in
 * range order, the kernels of a range on one of two internal compute streams once its
 * copy has landed (per-range events), so the copy engines of both directions stay busy
 * while earlier ranges compute.  The internal streams / events are
 * created once per process on first use; concurrent calls are serialised.  Only
 * DEFCON_SAMPLER_LDG is accepted (UNSUPPORTED otherwise: the entry owns no texture plan).
 * Every per-chunk device region is 256-byte aligned whatever the per-image sizes.  If an
 * error occurs after the first copy was enqueued, the internal streams are synchronised
 * before returning, so no copy touches x_host / y_host after the call returns.
 * dev_workspace must hold defcon_layer_workspace_size() bytes (x, offsets, mask, y and
 * two step-1 / step-2 workspaces are carved out of it).  modulated != 0 selects DCNv2.
 * Per-image results equal defcon_dcn_forward on the same images up to the fp32
 * summation order of the stream-K partition, which depends on the batch size.
 */
int defcon_layer_forward_host(const void* x_host, int N, int H, int W, int Cin, int dtype,
                              const float* dw_w, const float* dw_scale, const float* dw_shift,
                              const float* pw_w, const float* pw_b,
                              const void* weight, const float* bias, int Cout, int K,
                              defcon_conv_t cv, int modulated, int sampler, int fp32_mode,
                              void* y_host, void* dev_workspace, size_t dev_workspace_bytes,
                              void* stream);

int defcon_layer_workspace_size(int N, int H, int W, int Cin, int dtype, int Cout, int K,
                                defcon_conv_t cv, int modulated, int sampler, int fp32_mode,
                                size_t* bytes);

/*
 * Texture plan for DEFCON_SAMPLER_TEX / HYBRID: ONE 2-D layered cudaArray
 * (layer l = channels 4l..4l+3; half4 texels for bf16 input, float4 for fp32) holding
 * the N images stacked along y with one zero row after each image (W x N*(H+1) texels
 * per layer), and a texture object with border (zero) addressing, linear filtering and
 * unnormalised coordinates.  Stacking images keeps the layer count at Cin/4, inside the
 * 2048-layer limit the paper notes, and the texture handle warp-uniform.
 * Errors: INVALID_ARG for bad sizes, UNSUPPORTED for Cin % 4 != 0, LIMIT for
 * Cin/4 > device max layers or H, W above the layered-texture limits, CUDA on
 * allocation failure.  destroy(NULL) is a no-op returning DEFCON_OK.
 */
int defcon_tex_plan_create(int N, int H, int W, int Cin, int dtype, defcon_tex_plan_t* plan);
int defcon_tex_plan_destroy(defcon_tex_plan_t plan);

/*
 * Texture-filter probe (measures the reading R14 on the device): samples a single
 * 2 x 2 float texel layer [[0, 0], [0, 1]] (border addressing, linear filter) at
 * the n coordinates (px[i], py[i]) given in texel units (no +0.5 applied), writing
 * the filtered values to out[i].  px, py, out are device fp32 arrays of length n.
 */
int defcon_tex_filter_probe(const float* px, const float* py, float* out, int n, void* stream);

const char* defcon_status_string(int status);
const char* defcon_last_error_detail(void);   /* thread-local, "" if none */
int defcon_abi_version(void);

#ifdef __cplusplus
}
#endif

#endif /* DEFCON_H_ */
