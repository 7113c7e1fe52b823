// mma_probe.cu -- tcgen05.mma issue/execution cost for thin-N shapes with SMEM (SS) operands:
// one CTA per SM issues `iters` MMAs (M = 128, N in {32, 64, 128, 256}; kind::tf32 K = 8 or
// kind::f16 K = 16) from SWIZZLE_128B K-major descriptors in a loop over K slices, commits,
// waits, and reports cycles per MMA.  Operand contents are irrelevant (zeros).
//   nvcc -std=c++17 -O3 -gencode arch=compute_100a,code=sm_100a -o tools/bin/mma_probe tools/mma_probe.cu -lcuda
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#include "../paper_conf_ipps_jayaweeralwrk24_b200/csrc/common.cuh"

using namespace defcon;

template <int N, bool TF32>
__global__ void __launch_bounds__(128, 1) probe(int iters, unsigned long long* out) {
    extern __shared__ __align__(1024) uint8_t dyn[];
    uint8_t* sm = dyn + ((1024u - (smem_u32(dyn) & 1023u)) & 1023u);
    __shared__ uint64_t done;
    __shared__ uint32_t tslot;
    const int warp = threadIdx.x >> 5;
    for (int i = threadIdx.x; i < (16384 + N * 128) / 4; i += blockDim.x) reinterpret_cast<uint32_t*>(sm)[i] = 0u;
    if (threadIdx.x == 0) {
        mbar_init(&done, 1);
        fence_barrier_init();
    }
    if (warp == 0) tmem_alloc<256>(&tslot);
    fence_proxy_async_smem();
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = tslot;
    if (threadIdx.x == 0) {
        const uint32_t a = smem_u32(sm), b = a + 16384;
        constexpr uint32_t idesc = make_idesc(TF32 ? 2u : 1u, 128, N);
        const long long t0 = clock64();
        for (int it = 0; it < iters; ++it) {
            const int kk = it & 3;   // 4 K slices of 32 bytes per 128-byte row
            const uint64_t da = make_sw128_desc(a + kk * 32), db = make_sw128_desc(b + kk * 32);
            if (TF32) mma_tf32_ss(tmem, da, db, idesc, it ? 1u : 0u);
            else mma_bf16_ss(tmem, da, db, idesc, it ? 1u : 0u);
        }
        const long long t1 = clock64();
        mma_commit(&done);
        mbar_wait(&done, 0);
        const long long t2 = clock64();
        if (blockIdx.x == 0) {
            out[0] = (unsigned long long)(t1 - t0);
            out[1] = (unsigned long long)(t2 - t0);
        }
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 0) {
        tc_fence_after();
        tmem_dealloc<256>(tmem);
    }
}

template <int N, bool TF32>
void run(int ctas_per_sm) {
    unsigned long long* d;
    cudaMalloc(&d, 16);
    const int iters = 4096;
    const size_t smem = 1024 + 16384 + N * 128;
    cudaFuncSetAttribute(probe<N, TF32>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    probe<N, TF32><<<148 * ctas_per_sm, 128, smem>>>(iters, d);
    cudaDeviceSynchronize();
    probe<N, TF32><<<148 * ctas_per_sm, 128, smem>>>(iters, d);
    cudaError_t e = cudaDeviceSynchronize();
    unsigned long long h[2];
    cudaMemcpy(h, d, 16, cudaMemcpyDeviceToHost);
    const double flop = 2.0 * 128 * N * (TF32 ? 8 : 16);
    printf("{\"kind\": \"%s\", \"M\": 128, \"N\": %d, \"ctas_per_sm\": %d, \"issue_cyc_per_mma\": %.1f, "
           "\"total_cyc_per_mma\": %.1f, \"flop_per_cyc_per_cta\": %.0f, \"err\": \"%s\"}\n",
           TF32 ? "tf32" : "bf16", N, ctas_per_sm, (double)h[0] / iters, (double)h[1] / iters,
           flop * iters / (double)h[1], cudaGetErrorString(e));
    cudaFree(d);
}

int main() {
    for (int c = 1; c <= 2; ++c) {
        run<32, true>(c);
        run<64, true>(c);
        run<128, true>(c);
        run<256, true>(c);
        run<32, false>(c);
        run<256, false>(c);
    }
    return 0;
}
