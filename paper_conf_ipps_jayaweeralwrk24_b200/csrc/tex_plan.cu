// tex_plan.cu -- texture resources for DEFCON_SAMPLER_TEX, the paper's texel-based
// optimisation re-evaluated on sm_100a.
//
// Layout (adapted): ONE 2-D *layered* cudaArray, layer l holding channels
// [4l, 4l+4) as one 4-component texel per pixel (half4 for bf16 inputs -- CUDA has no
// bf16 texel format -- float4 for fp32 inputs).  Instead of merging batch and channel
// into the layer index (which hits the 2048-layer limit at N*C/4 > 2048),
// the images are stacked along y with one zero row after each image: texel row
// n*(H+1) + y holds image n's row y, row n*(H+1) + H is zero.  The layer count stays
// Cin/4 and the texture handle is the same for every lane of a warp (bindless texture
// handles must be warp-uniform).  Bilinear taps that leave an image read the zero row
// (y) or the zero border (x); callers clamp coordinates into [-1, H] x [-1, W].
// The texture object uses unnormalised coordinates, linear (bilinear) filtering and
// border addressing with a zero border colour (the zero-outside rule, P:83 / P:201).
// The array is (re)filled from NHWC x by tex_stage_kernel through surface writes.
#include <cstdio>
#include <cstring>

#include "common.cuh"
#include "kernels.h"

namespace defcon {

struct TexPlan {
    int N, H, W, C, layers;
    bool half;                              // half4 texels (bf16 input) vs float4 (fp32)
    cudaArray_t array;
    cudaTextureObject_t tex;
    cudaSurfaceObject_t surf;
};

namespace {

// One thread per (stacked texel row, column, layer): 4 channels -> one texel; the row
// after each image is written as zeros.
template <bool HALF>
__global__ void tex_stage_kernel(const void* __restrict__ x, cudaSurfaceObject_t surf, int H, int W,
                                 int C, int layers, long total) {
    const long i = (long)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= total) return;
    const int l = (int)(i % layers);
    const long r = i / layers;                    // stacked (row, column)
    const int xw = (int)(r % W);
    const int ys = (int)(r / W);                  // stacked row n*(H+1) + y
    const int n = ys / (H + 1), y = ys - n * (H + 1);
    if (HALF) {
        ushort4 t = make_ushort4(0, 0, 0, 0);
        if (y < H) {
            const long pix = ((long)n * H + y) * W + xw;
            const uint2 u = __ldg(reinterpret_cast<const uint2*>(static_cast<const __nv_bfloat16*>(x) + pix * C + l * 4));
            // bf16 -> fp16 round to nearest (exact for |v| in the fp16 normal range)
            t = make_ushort4(__half_as_ushort(__float2half_rn(bf16lo_to_f32(u.x))),
                             __half_as_ushort(__float2half_rn(bf16hi_to_f32(u.x))),
                             __half_as_ushort(__float2half_rn(bf16lo_to_f32(u.y))),
                             __half_as_ushort(__float2half_rn(bf16hi_to_f32(u.y))));
        }
        surf2DLayeredwrite(t, surf, xw * (int)sizeof(ushort4), ys, l, cudaBoundaryModeTrap);
    } else {
        float4 f = make_float4(0.f, 0.f, 0.f, 0.f);
        if (y < H) {
            const long pix = ((long)n * H + y) * W + xw;
            f = __ldg(reinterpret_cast<const float4*>(static_cast<const float*>(x) + pix * C + l * 4));
        }
        surf2DLayeredwrite(f, surf, xw * (int)sizeof(float4), ys, l, cudaBoundaryModeTrap);
    }
}

}  // namespace

cudaError_t tex_plan_create(int N, int H, int W, int C, bool half, TexPlan** out) {
    *out = nullptr;
    TexPlan* p = new TexPlan();
    memset(p, 0, sizeof(*p));
    p->N = N; p->H = H; p->W = W; p->C = C; p->layers = C / 4; p->half = half;
    const cudaChannelFormatDesc fmt = half ? cudaCreateChannelDescHalf4() : cudaCreateChannelDesc<float4>();
    cudaError_t e = cudaMalloc3DArray(&p->array, &fmt, make_cudaExtent(W, (size_t)N * (H + 1), p->layers),
                                      cudaArrayLayered | cudaArraySurfaceLoadStore);
    if (e == cudaSuccess) {
        cudaResourceDesc rd;
        memset(&rd, 0, sizeof(rd));
        rd.resType = cudaResourceTypeArray;
        rd.res.array.array = p->array;
        cudaTextureDesc td;
        memset(&td, 0, sizeof(td));
        td.addressMode[0] = cudaAddressModeBorder;     // zero outside the image
        td.addressMode[1] = cudaAddressModeBorder;
        td.addressMode[2] = cudaAddressModeBorder;
        td.borderColor[0] = td.borderColor[1] = td.borderColor[2] = td.borderColor[3] = 0.f;
        td.filterMode = cudaFilterModeLinear;         // hardware bilinear
        td.readMode = cudaReadModeElementType;
        td.normalizedCoords = 0;
        e = cudaCreateTextureObject(&p->tex, &rd, &td, nullptr);
        if (e == cudaSuccess) e = cudaCreateSurfaceObject(&p->surf, &rd);
    }
    if (e != cudaSuccess) {
        tex_plan_destroy(p);
        return e;
    }
    *out = p;
    return cudaSuccess;
}

void tex_plan_destroy(TexPlan* p) {
    if (!p) return;
    if (p->surf) cudaDestroySurfaceObject(p->surf);
    if (p->tex) cudaDestroyTextureObject(p->tex);
    if (p->array) cudaFreeArray(p->array);
    delete p;
}

bool tex_plan_matches(const TexPlan* p, int N, int H, int W, int C, bool half) {
    return p && p->N == N && p->H == H && p->W == W && p->C == C && p->half == half;
}

unsigned long long tex_plan_texture(const TexPlan* p) { return p->tex; }

cudaError_t tex_plan_stage(const TexPlan* p, const void* x, cudaStream_t stream) {
    const long total = (long)p->N * (p->H + 1) * p->W * p->layers;
    const int threads = 256;
    const unsigned blocks = (unsigned)((total + threads - 1) / threads);
    if (p->half)
        tex_stage_kernel<true><<<blocks, threads, 0, stream>>>(x, p->surf, p->H, p->W, p->C, p->layers, total);
    else
        tex_stage_kernel<false><<<blocks, threads, 0, stream>>>(x, p->surf, p->H, p->W, p->C, p->layers, total);
    return cudaGetLastError();
}

// ---------------------------------------------------------------- filter probe
namespace {
__global__ void tex_probe_kernel(cudaTextureObject_t t, const float* px, const float* py, float* out, int n) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n) out[i] = tex2DLayered<float>(t, px[i], py[i], 0);
}
}  // namespace

// 2 x 2 single-layer float texture [[0, 0], [0, 1]] (row-major, y then x), linear filter,
// border addressing: out = filter(px, py) exposes the fixed-point fraction handling.
cudaError_t tex_filter_probe(const float* px, const float* py, float* out, int n, cudaStream_t stream) {
    cudaArray_t arr = nullptr;
    const cudaChannelFormatDesc fmt = cudaCreateChannelDesc<float>();
    cudaError_t e = cudaMalloc3DArray(&arr, &fmt, make_cudaExtent(2, 2, 1), cudaArrayLayered);
    if (e != cudaSuccess) return e;
    const float host[4] = {0.f, 0.f, 0.f, 1.f};
    cudaMemcpy3DParms cp;
    memset(&cp, 0, sizeof(cp));
    cp.srcPtr = make_cudaPitchedPtr(const_cast<float*>(host), 2 * sizeof(float), 2, 2);
    cp.dstArray = arr;
    cp.extent = make_cudaExtent(2, 2, 1);
    cp.kind = cudaMemcpyHostToDevice;
    e = cudaMemcpy3D(&cp);
    cudaTextureObject_t t = 0;
    if (e == cudaSuccess) {
        cudaResourceDesc rd;
        memset(&rd, 0, sizeof(rd));
        rd.resType = cudaResourceTypeArray;
        rd.res.array.array = arr;
        cudaTextureDesc td;
        memset(&td, 0, sizeof(td));
        td.addressMode[0] = td.addressMode[1] = td.addressMode[2] = cudaAddressModeBorder;
        td.filterMode = cudaFilterModeLinear;
        td.readMode = cudaReadModeElementType;
        td.normalizedCoords = 0;
        e = cudaCreateTextureObject(&t, &rd, &td, nullptr);
    }
    if (e == cudaSuccess) {
        tex_probe_kernel<<<(n + 255) / 256, 256, 0, stream>>>(t, px, py, out, n);
        e = cudaGetLastError();
        if (e == cudaSuccess) e = cudaStreamSynchronize(stream);
    }
    if (t) cudaDestroyTextureObject(t);
    cudaFreeArray(arr);
    return e;
}

}  // namespace defcon
