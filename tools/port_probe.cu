// port_probe.cu -- does tcgen05.mma (SS operands) share the SM's shared-memory / L1 data port
// with LSU traffic?  One CTA per SM: thread 0 issues M128 x N x K16 bf16 MMAs back to back
// (SWIZZLE_128B K-major operands in smem) until 8 "load" warps finish a fixed amount of
// traffic of one kind; reports the MMA cycles per instruction and the LSU bytes per cycle.
//   mode 0 idle, 1 LDS.128, 2 STS.128, 3 LDG.256 L1-resident (16 KB), 4 LDG.256 L2 (4 MB),
//   5 LDG.256 L1-resident + STS.128 (1 per 2 loads: the DCN producer's mix)
//   nvcc -std=c++17 -O3 -gencode arch=compute_100a,code=sm_100a -o tools/bin/port_probe tools/port_probe.cu -lcuda
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#include "../paper_conf_ipps_jayaweeralwrk24_b200/csrc/common.cuh"

using namespace defcon;

constexpr int LW = 8;   // load warps

template <int N>
__global__ void __launch_bounds__(32 * (LW + 1), 1)
    probe(int mode, int iters, const uint8_t* g, size_t gbytes, unsigned long long* out, int random_ops) {
    extern __shared__ __align__(1024) uint8_t dyn[];
    uint8_t* sm = dyn + ((1024u - (smem_u32(dyn) & 1023u)) & 1023u);
    uint8_t* scratch = sm + 16384 + N * 128;
    __shared__ uint64_t done;
    __shared__ uint32_t tslot;
    __shared__ volatile int stop;
    __shared__ int ndone;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    for (int i = threadIdx.x; i < (16384 + N * 128 + 32768) / 4; i += blockDim.x) {
        // operands: zeros, or (RANDOM_OPS) bf16 pairs of N(0,1)-like magnitude with random mantissas
        uint32_t h = (uint32_t)i * 2654435761u ^ 0x9e3779b9u;
        h ^= h >> 15; h *= 2246822519u; h ^= h >> 13;
        const uint32_t lo = 0x3f00u | (h & 0x80ffu), hi = 0x3f00u | ((h >> 16) & 0x80ffu);
        reinterpret_cast<uint32_t*>(sm)[i] = random_ops ? (hi << 16 | lo) : 0u;
    }
    if (threadIdx.x == 0) {
        mbar_init(&done, 1);
        fence_barrier_init();
        stop = 0;
        ndone = 0;
    }
    if (warp == 0) tmem_alloc<256>(&tslot);
    fence_proxy_async_smem();
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = tslot;
    if (warp == 0) {
        if (lane == 0) {
            const uint32_t a = smem_u32(sm), b = a + 16384;
            constexpr uint32_t idesc = make_idesc(1u, 128, N);
            const long long t0 = clock64();
            long long cnt = 0;
            for (;;) {
#pragma unroll
                for (int u = 0; u < 16; ++u) {
                    const int kk = u & 3;
                    mma_bf16_ss(tmem, make_sw128_desc(a + kk * 32), make_sw128_desc(b + kk * 32), idesc,
                                (cnt | u) ? 1u : 0u);
                }
                cnt += 16;
                if (mode == 0 ? cnt >= 4096 : stop != 0) break;
            }
            mma_commit(&done);
            mbar_wait(&done, 0);
            const long long t2 = clock64();
            if (blockIdx.x == 0) {
                out[0] = (unsigned long long)(t2 - t0);
                out[1] = (unsigned long long)cnt;
            }
        }
    } else {
        const int lw = warp - 1;
        uint32_t acc = 0;
        const uint32_t sbase = smem_u32(scratch);
        const long long t0 = clock64();
        if (mode == 1) {
            for (int it = 0; it < iters; ++it) {
#pragma unroll
                for (int u = 0; u < 4; ++u) {
                    const uint4 v = ld_shared_v4(sbase + (((it * 4 + u) * LW + lw) * 512 + lane * 16) % 32768);
                    acc ^= v.x ^ v.y ^ v.z ^ v.w;
                }
            }
        } else if (mode == 2) {
            for (int it = 0; it < iters; ++it) {
#pragma unroll
                for (int u = 0; u < 4; ++u)
                    st_shared_v4(sbase + (((it * 4 + u) * LW + lw) * 512 + lane * 16) % 32768, it, u, lane, 0);
            }
        } else if (mode >= 3) {
            const uint32_t mask = (mode == 4 ? (uint32_t)gbytes : 16384u) - 1u;   // powers of two
            // lane -> line lane / 4, 32-byte quarter lane % 4: 8 full lines per warp instruction
            uint32_t off = ((uint32_t)(blockIdx.x * LW + lw) * 8 * 128 * 4 + (lane >> 2) * 128 + (lane & 3) * 32) & mask;
            for (int it = 0; it < iters; ++it) {
                U8x32 v[4];
#pragma unroll
                for (int u = 0; u < 4; ++u) v[u] = ldg_nc_v8(g + ((off + (uint32_t)u * 1024 * LW) & mask));
#pragma unroll
                for (int u = 0; u < 4; ++u) {
                    acc ^= v[u].w[0] ^ v[u].w[3] ^ v[u].w[7];
                    if (mode == 5 && (u & 1))
                        st_shared_v4(sbase + ((it * 2 + (u >> 1)) * LW * 512 + lw * 512 + lane * 16) % 32768,
                                     v[u].w[1], v[u].w[2], v[u].w[4], v[u].w[5]);
                }
                off = (off + 4 * 1024 * LW * 7) & mask;
            }
        }
        const long long t1 = clock64();
        if (acc == 0x12345678u) out[7] = acc;
        if (lane == 0) {
            if (blockIdx.x == 0 && lw == 0) out[2] = (unsigned long long)(t1 - t0);
            if (atomicAdd(&ndone, 1) == LW - 1) stop = 1;
        }
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 0) {
        tc_fence_after();
        tmem_dealloc<256>(tmem);
    }
}

template <int N>
void run(int mode, const uint8_t* g, size_t gbytes, unsigned long long* d, int rnd) {
    const int iters = 4096;
    const size_t smem = 1024 + 16384 + N * 128 + 32768;
    cudaFuncSetAttribute(probe<N>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    for (int rep = 0; rep < 2; ++rep) probe<N><<<148, 32 * (LW + 1), smem>>>(mode, iters, g, gbytes, d, rnd);
    cudaError_t e = cudaDeviceSynchronize();
    unsigned long long h[3];
    cudaMemcpy(h, d, 24, cudaMemcpyDeviceToHost);
    const double bytes_per_iter = (mode == 1 || mode == 2) ? 4.0 * 512 * LW : (mode >= 3 ? 4.0 * 1024 * LW : 0);
    const double sts_bytes = mode == 5 ? 2.0 * 512 * LW : 0;
    printf("{\"rnd\": %d, \"N\": %d, \"mode\": %d, \"mma_cyc_per_instr\": %.1f, \"mma_smem_B_per_cyc\": %.1f, "
           "\"lsu_B_per_cyc\": %.1f, \"sts_B_per_cyc\": %.1f, \"load_cycles\": %llu, \"err\": \"%s\"}\n",
           rnd, N, mode, (double)h[0] / h[1], (16384.0 / 4 + N * 32.0) * h[1] / h[0],
           h[2] ? bytes_per_iter * iters / h[2] : 0.0, h[2] ? sts_bytes * iters / h[2] : 0.0, h[2],
           cudaGetErrorString(e));
}

int main() {
    unsigned long long* d;
    cudaMalloc(&d, 64);
    cudaMemset(d, 0, 64);
    const size_t gbytes = 4u << 20;
    uint8_t* g;
    cudaMalloc(&g, gbytes);
    cudaMemset(g, 1, gbytes);
    for (int rnd = 0; rnd <= 1; ++rnd) {
        for (int mode = 0; mode <= 5; ++mode) run<256>(mode, g, gbytes, d, rnd);
        for (int mode = 0; mode <= 5; mode += 5) run<128>(mode, g, gbytes, d, rnd);
    }
    return 0;
}
