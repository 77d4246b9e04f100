// Microbenchmark: latency and throughput of the Rabin rolling step
// (PRMT -> LDS -> LOP3 chain with per-lane replicated tables in smem).
// Build: nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o mb tools/microbench_roll.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t lds(uint32_t a) {
    uint32_t v;
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a));
    return v;
}

template <int MODE>
__global__ void __launch_bounds__(1024, 1) k(uint32_t* out, int iters, long long* cyc) {
    extern __shared__ __align__(16) uint8_t smem[];
    const uint32_t win = (uint32_t)__cvta_generic_to_shared(smem);
    const uint32_t pad = (0x10000u - (win & 0xFFFFu)) & 0xFFFFu;
    const uint32_t base = win + pad;
    uint32_t* t32 = reinterpret_cast<uint32_t*>(smem + pad);
    for (int i = threadIdx.x; i < 16384; i += blockDim.x) t32[i] = i * 2654435761u;
    __syncthreads();
    const int lane = threadIdx.x & 31;
    const uint32_t laneR = base | (lane * 4), laneW = laneR + 128;
    uint32_t h = threadIdx.x * 7919u, w0 = threadIdx.x * 13u, o0 = threadIdx.x * 31u, bits = 0;
    long long t0 = clock64();
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            const uint32_t aR = __byte_perm(h, laneR, 0x7634);
            const uint32_t aW = __byte_perm(o0, laneW, 0x7604 | (k << 4));
            const uint32_t hs = __byte_perm(w0, h, 0x6540 | k);
            if (MODE == 0) {
                h = hs ^ lds(aR) ^ lds(aW);
            } else {  // no W lookup
                h = hs ^ lds(aR);
            }
            asm("{\n\t.reg .pred p;\n\tsetp.eq.u32 p, %1, 0;\n\t@p or.b32 %0, %0, %2;\n\t}"
                : "+r"(bits) : "r"(h & 0xFFF), "r"(1u << k));
        }
        w0 = w0 * 1664525u + 1013904223u;
        o0 ^= w0;
    }
    long long t1 = clock64();
    out[blockIdx.x * blockDim.x + threadIdx.x] = h ^ bits;
    if (threadIdx.x == 0 && blockIdx.x == 0) *cyc = t1 - t0;
}

int main() {
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    uint32_t* out;
    long long* cyc;
    cudaMalloc(&out, sizeof(uint32_t) * sms * 1024);
    cudaMalloc(&cyc, sizeof(long long));
    const int smem = 2 * 65536;
    cudaFuncSetAttribute(k<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaFuncSetAttribute(k<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    const int iters = 4096;
    for (int mode = 0; mode < 2; ++mode) {
        for (int threads : {32, 128, 256, 512, 1024}) {
            long long c = 0;
            for (int rep = 0; rep < 2; ++rep) {
                cudaEventRecord(a);
                if (mode == 0) k<0><<<sms, threads, smem>>>(out, iters, cyc);
                else k<1><<<sms, threads, smem>>>(out, iters, cyc);
                cudaEventRecord(b);
                cudaEventSynchronize(b);
            }
            float ms;
            cudaEventElapsedTime(&ms, a, b);
            cudaMemcpy(&c, cyc, sizeof(c), cudaMemcpyDeviceToHost);
            const double bytes = (double)sms * threads * iters * 4;
            printf("mode %d threads/SM %4d: %.1f cycles/byte/warp (clock64), %.1f GB/s chip\n", mode,
                   threads, (double)c / (iters * 4), bytes / (ms * 1e6));
        }
    }
    return 0;
}
