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

// MODE 2/3: 32-byte steps whose data comes from global memory, lanes owning
// contiguous 256-byte segments (stride load, as the scan kernel) / lanes
// reading interleaved 16-byte pieces (coalesced).
template <int MODE>
__global__ void __launch_bounds__(512, 2) kg(const uint4* __restrict__ in, uint32_t* out,
                                             int steps, long long* cyc) {
    extern __shared__ __align__(16) uint8_t smem[];
    const uint32_t win = (uint32_t)__cvta_generic_to_shared(smem);
    const uint32_t pad = (0x10000u - (win & 0xFFFFu)) & 0xFFFFu;
    const uint32_t base = win + pad;
    uint32_t* t32 = reinterpret_cast<uint32_t*>(smem + pad);
    for (int i = threadIdx.x; i < 16384; i += blockDim.x) t32[i] = i * 2654435761u;
    __syncthreads();
    const int lane = threadIdx.x & 31;
    const uint32_t laneR = base | (lane * 4), laneW = laneR + 128;
    const uint64_t gtid = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    const uint64_t gthreads = (uint64_t)gridDim.x * blockDim.x;
    uint32_t h = threadIdx.x * 7919u, bits = 0;
    uint32_t old[8] = {0, 0, 0, 0, 0, 0, 0, 0};
    long long t0 = clock64();
    for (int s = 0; s < steps; ++s) {
        uint4 a, b;
        if (MODE == 2) {  // lane-contiguous segments of steps*32 bytes
            const uint4* p = in + (gtid * steps + s) * 2;
            a = __ldg(p);
            b = __ldg(p + 1);
        } else {          // warp-interleaved (coalesced)
            const uint4* p = in + ((uint64_t)s * gthreads + gtid) * 2;
            a = __ldg(p);
            b = __ldg(p + 1);
        }
        uint32_t cur[8] = {a.x, a.y, a.z, a.w, b.x, b.y, b.z, b.w};
#pragma unroll
        for (int w = 0; w < 8; ++w) {
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                const uint32_t aR = __byte_perm(h, laneR, 0x7634);
                const uint32_t aW = __byte_perm(old[w], laneW, 0x7604 | (k << 4));
                const uint32_t hs = __byte_perm(cur[w], h, 0x6540 | k);
                h = hs ^ lds(aR) ^ lds(aW);
                asm("{\n\t.reg .pred p;\n\tsetp.eq.u32 p, %1, 0;\n\t@p or.b32 %0, %0, %2;\n\t}"
                    : "+r"(bits) : "r"(h & 0xFFF), "r"(1u << (4 * w + k)));
            }
        }
#pragma unroll
        for (int i = 0; i < 8; ++i) old[i] = cur[i];
    }
    long long t1 = clock64();
    out[gtid] = h ^ bits;
    if (gtid == 0) *cyc = t1 - t0;
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
    // global-memory variants: 148 x 512 threads x steps x 32 bytes
    const int steps = 64;
    const size_t nbytes = (size_t)sms * 512 * steps * 32;
    uint4* in;
    cudaMalloc(&in, nbytes);
    cudaMemset(in, 0x5a, nbytes);
    cudaFuncSetAttribute(kg<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaFuncSetAttribute(kg<3>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    for (int mode = 2; mode < 4; ++mode) {
        float ms = 0;
        for (int rep = 0; rep < 3; ++rep) {
            cudaEventRecord(a);
            if (mode == 2) kg<2><<<sms, 512, smem>>>(in, out, steps, cyc);
            else kg<3><<<sms, 512, smem>>>(in, out, steps, cyc);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            cudaEventElapsedTime(&ms, a, b);
        }
        printf("global mode %d (%s): %.1f GB/s (%.1f MB in %.1f us)\n", mode,
               mode == 2 ? "lane-contiguous" : "coalesced", nbytes / (ms * 1e6), nbytes / 1e6,
               ms * 1e3);
    }
    return 0;
}
