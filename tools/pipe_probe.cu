// pipe_probe.cu -- microbenchmark of the producer -> MMA-issuer -> producer mbarrier
// handshake used by dcn_fwd_bf16_tc_kernel, without any data movement or math.
// Variants isolate: tcgen05.commit vs plain mbarrier arrive for the "empty" signal,
// fence.proxy.async on/off, number of stages, try_wait vs test_wait spinning.
//   nvcc -std=c++17 -O3 -gencode arch=compute_100a,code=sm_100a -o pipe_probe pipe_probe.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#include "../paper_conf_ipps_jayaweeralwrk24_b200/csrc/common.cuh"

using namespace defcon;

// VAR bit 1: separate TMA warp role (waits empty, arrives full_b); MMA waits full_a + full_b
// VAR bit 2: 4 extra warps spin on a barrier that completes only at the end (epilogue role)
// VAR bit 4: producer body like dcn_fwd_bf16_tc_kernel: ROWS rows per thread, 8 threads
//            per 128-byte row, meta LDS.128 x2 per row (entries 288 B apart), STS.128 per row
// VAR bit 8: producers arrive with mbarrier.arrive.relaxed.cta
// VAR bit 16: skip the meta LDS (STS only)
template <int STAGES, bool COMMIT, bool FENCE, int NPW, int VAR>
__global__ void __launch_bounds__((NPW + 7) * 32, 1) probe(int iters, unsigned long long* cycles) {
    constexpr int ROWS = 128 * 8 / (NPW * 32);
    __shared__ uint64_t full[STAGES], fullb[STAGES], empty[STAGES], done;
    __shared__ uint32_t tslot;
    extern __shared__ __align__(1024) uint8_t dyn[];
    uint8_t* buf = dyn;                         // STAGES x 16 KB A tiles
    uint8_t* meta = dyn + STAGES * 16384;       // 128 rows x 9 taps x 32 B
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        for (int s = 0; s < STAGES; ++s) { mbar_init(&full[s], NPW); mbar_init(&fullb[s], 1); mbar_init(&empty[s], 1); }
        mbar_init(&done, 1);
        fence_barrier_init();
    }
    if (COMMIT && warp == NPW + 1) tmem_alloc<32>(&tslot);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const long long t0 = clock64();
    if (warp < NPW) {
        const int t = threadIdx.x, cvec = t & 7;
        int tap = 0;
        for (int q = 0; q < iters; ++q) {
            const int s = q % STAGES;
            uint4 acc[ROWS];
#pragma unroll
            for (int p = 0; p < ROWS; ++p) {
                acc[p] = make_uint4(q, q, q, q);
                if ((VAR & 4) && !(VAR & 16)) {
                    const int row = (t >> 3) + p * (NPW * 4);
                    const uint32_t e = smem_u32(meta) + (row * 9 + tap) * 32;
                    const uint4 o = ld_shared_v4(e);
                    const uint4 w = ld_shared_v4(e + 16);
                    acc[p].x ^= o.x + w.y; acc[p].y ^= o.y; acc[p].z += w.z; acc[p].w += o.w;
                }
            }
            if (++tap == 9) tap = 0;
            mbar_wait(&empty[s], ((uint32_t)(q / STAGES) & 1u) ^ 1u);
            if (VAR & 4) {
#pragma unroll
                for (int p = 0; p < ROWS; ++p) {
                    const int row = (t >> 3) + p * (NPW * 4);
                    st_shared_v4(smem_u32(buf + s * 16384 + row * 128 + ((cvec ^ (row & 7)) << 4)),
                                 acc[p].x, acc[p].y, acc[p].z, acc[p].w);
                }
            } else {
                st_shared_v4(smem_u32(buf + s * 16384 + threadIdx.x * 16), q, q, q, q);
            }
            if (FENCE) fence_proxy_async_smem();
            __syncwarp();
            if (lane == 0) {
                if (VAR & 8)
                    asm volatile("{\n\t.reg .b64 st;\n\tmbarrier.arrive.relaxed.cta.shared::cta.b64 st, [%0];\n\t}" ::"r"(smem_u32(&full[s])) : "memory");
                else
                    mbar_arrive(&full[s]);
            }
        }
    } else if (warp == NPW && (VAR & 1)) {
        if (lane == 0)
            for (int q = 0; q < iters; ++q) {
                const int s = q % STAGES;
                mbar_wait(&empty[s], ((uint32_t)(q / STAGES) & 1u) ^ 1u);
                mbar_arrive(&fullb[s]);
            }
    } else if (warp == NPW + 1 && lane == 0) {
        for (int q = 0; q < iters; ++q) {
            const int s = q % STAGES;
            const uint32_t ph = (uint32_t)(q / STAGES) & 1u;
            mbar_wait(&full[s], ph);
            if (VAR & 1) mbar_wait(&fullb[s], ph);
            tc_fence_after();
            if (COMMIT) mma_commit(&empty[s]); else mbar_arrive(&empty[s]);
        }
        mbar_arrive(&done);
    } else if (warp >= NPW + 2 && warp < NPW + 6 && (VAR & 2)) {
        mbar_wait(&done, 0);
    }
    __syncwarp();
    tc_fence_before();
    __syncthreads();
    if (threadIdx.x == 0) cycles[blockIdx.x] = clock64() - t0;
    if (COMMIT && warp == NPW + 1) { tc_fence_after(); tmem_dealloc<32>(tslot); }
}

template <int STAGES, bool COMMIT, bool FENCE, int NPW, int VAR = 0>
void run(const char* name) {
    unsigned long long* d;
    cudaMalloc(&d, 148 * 8);
    const int iters = 4000;
    const int smem = STAGES * 16384 + 128 * 9 * 32;
    cudaFuncSetAttribute(probe<STAGES, COMMIT, FENCE, NPW, VAR>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    probe<STAGES, COMMIT, FENCE, NPW, VAR><<<148, (NPW + 7) * 32, smem>>>(iters, d);
    cudaEvent_t a, b;
    cudaEventCreate(&a); cudaEventCreate(&b);
    cudaEventRecord(a);
    probe<STAGES, COMMIT, FENCE, NPW, VAR><<<148, (NPW + 7) * 32, smem>>>(iters, d);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b);
    unsigned long long h[148];
    cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
    printf("%-44s %8.1f ns/iter  %8.1f cycles/iter  (%s)\n", name, ms * 1e6 / iters,
           (double)h[0] / iters, cudaGetErrorString(cudaGetLastError()));
    cudaFree(d);
}

int main() {
    run<3, true, true, 8, 3>("8w: 1 STS + fence + arrive");
    run<3, true, true, 8, 3 | 4 | 16>("8w: 4 STS + fence + arrive");
    run<3, true, true, 8, 3 | 4>("8w: 4x(2 LDS + STS) + fence");
    run<3, true, false, 8, 3 | 4>("8w: 4x(2 LDS + STS) nofence");
    run<3, true, true, 8, 3 | 4 | 8>("8w: 4x(2 LDS + STS) fence relaxed-arrive");
    run<3, false, true, 8, 3 | 4>("8w: 4x(2 LDS + STS) fence, arrive-not-commit");
    run<3, true, true, 16, 3 | 4>("16w: 2x(2 LDS + STS) + fence");
    run<3, true, true, 4, 3 | 4>("4w: 8x(2 LDS + STS) + fence");
    return 0;
}
