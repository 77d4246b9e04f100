// probe.cu -- measured integer-pipe throughput of this GPU (the roofline
// denominators of the SHA-1 and scan kernels: "Integer-op peak.
// Not in MEASURED_PEAKS: microbenchmark LOP3/SHF/IADD3 throughput on B200").
//
// Each probe kernel runs 8 independent dependency chains per thread of one
// instruction kind (inline PTX, asm volatile, so ptxas keeps every op),
// 16 ops per chain per loop trip, on a full grid (every SM at 2 x 1024
// threads), and reports thread-ops per second.  The SASS of each kernel is
// one opcode per op (checked with cuobjdump: LOP3.LUT, SHF.L.W.U32.HI,
// IADD3, IMAD, IMAD.HI.U32, PRMT, LEA.HI, and the LOP3 + IMAD mix).
#include <cuda_runtime.h>
#include <stdint.h>

#include "dedup.h"

namespace {

constexpr int kChains = 8;
constexpr int kUnroll = 16;
constexpr int kThreads = 1024;

enum Kind { kLop3 = 0, kShf, kIadd3, kImad, kImadHi, kPrmt, kLeaHi, kMixLopImad, kKinds };

template <int K>
__device__ __forceinline__ void op(uint32_t& x, uint32_t y, uint32_t z) {
    if constexpr (K == kLop3) {
        asm volatile("lop3.b32 %0, %0, %1, %2, 0x96;" : "+r"(x) : "r"(y), "r"(z));
    } else if constexpr (K == kShf) {
        asm volatile("shf.l.wrap.b32 %0, %0, %0, 5;" : "+r"(x));
    } else if constexpr (K == kIadd3) {
        asm volatile("{\n\t.reg .u32 t;\n\tadd.u32 t, %0, %1;\n\tadd.u32 %0, t, %2;\n\t}"
                     : "+r"(x) : "r"(y), "r"(z));
    } else if constexpr (K == kImad) {
        asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(x) : "r"(y), "r"(z));
    } else if constexpr (K == kImadHi) {
        asm volatile("mad.hi.u32 %0, %0, %1, %2;" : "+r"(x) : "r"(y), "r"(z));
    } else if constexpr (K == kPrmt) {
        asm volatile("prmt.b32 %0, %0, %1, 0x0123;" : "+r"(x) : "r"(y));
    } else if constexpr (K == kLeaHi) {  // rotl(x, 5) + y, one LEA.HI
        asm volatile("{\n\t.reg .u32 t;\n\tshf.l.wrap.b32 t, %0, %0, 5;\n\tadd.u32 %0, t, %1;\n\t}"
                     : "+r"(x) : "r"(y));
    }
}

template <int K>
__global__ void __launch_bounds__(kThreads, 2) probe_kernel(uint32_t* out, int trips, uint32_t s) {
    uint32_t x[kChains];
#pragma unroll
    for (int c = 0; c < kChains; ++c) x[c] = threadIdx.x * 2654435761u + c * s;
    const uint32_t y = s * 7u + 1u, z = s ^ 0x5bd1e995u;
    for (int t = 0; t < trips; ++t) {
#pragma unroll
        for (int u = 0; u < kUnroll; ++u) {
#pragma unroll
            for (int c = 0; c < kChains; ++c) {
                if constexpr (K == kMixLopImad) {
                    if (c & 1) op<kImad>(x[c], y, z);
                    else op<kLop3>(x[c], y, z);
                } else {
                    op<K>(x[c], y, z);
                }
            }
        }
    }
    uint32_t r = 0;
#pragma unroll
    for (int c = 0; c < kChains; ++c) r ^= x[c];
    if (r == 0x12345678u) out[threadIdx.x] = r;  // keeps the chains live
}

template <int K>
double run(int sms, int trips, uint32_t* out, cudaEvent_t e0, cudaEvent_t e1) {
    const int blocks = 2 * sms;
    probe_kernel<K><<<blocks, kThreads>>>(out, trips / 8, 1u);  // warm-up
    cudaEventRecord(e0);
    probe_kernel<K><<<blocks, kThreads>>>(out, trips, 1u);
    cudaEventRecord(e1);
    if (cudaEventSynchronize(e1) != cudaSuccess) return -1.0;
    float ms = 0;
    cudaEventElapsedTime(&ms, e0, e1);
    const double ops = (double)blocks * kThreads * trips * kUnroll * kChains;
    return ops / (ms * 1e-3) / 1e12;
}

}  // namespace

extern "C" dedup_status dedup_probe_int_rates(int32_t device, dedup_int_rates* out) {
    if (out == nullptr) return DEDUP_EINVAL;
    if (cudaSetDevice(device) != cudaSuccess) return DEDUP_ECUDA;
    int sms = 0, khz = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
    cudaDeviceGetAttribute(&khz, cudaDevAttrClockRate, device);
    uint32_t* buf = nullptr;
    cudaEvent_t e0 = nullptr, e1 = nullptr;
    if (cudaMalloc(&buf, kThreads * sizeof(uint32_t)) != cudaSuccess) return DEDUP_ENOMEM;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    const int trips = 4096;  // ~ 2 x 148 x 1024 x 4096 x 128 ops = 160 G ops per probe
    double r[kKinds];
    r[kLop3] = run<kLop3>(sms, trips, buf, e0, e1);
    r[kShf] = run<kShf>(sms, trips, buf, e0, e1);
    r[kIadd3] = run<kIadd3>(sms, trips, buf, e0, e1);
    r[kImad] = run<kImad>(sms, trips, buf, e0, e1);
    r[kImadHi] = run<kImadHi>(sms, trips, buf, e0, e1);
    r[kPrmt] = run<kPrmt>(sms, trips, buf, e0, e1);
    r[kLeaHi] = run<kLeaHi>(sms, trips, buf, e0, e1);
    r[kMixLopImad] = run<kMixLopImad>(sms, trips, buf, e0, e1);
    const cudaError_t err = cudaGetLastError();
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    cudaFree(buf);
    if (err != cudaSuccess) return DEDUP_ECUDA;
    for (double v : r)
        if (v <= 0) return DEDUP_ECUDA;
    out->lop3 = r[kLop3];
    out->shf = r[kShf];
    out->iadd3 = r[kIadd3];
    out->imad = r[kImad];
    out->imad_hi = r[kImadHi];
    out->prmt = r[kPrmt];
    out->lea_hi = r[kLeaHi];
    out->mix_lop3_imad = r[kMixLopImad];
    out->num_sms = sms;
    out->clock_mhz_attr = khz / 1000;
    return DEDUP_OK;
}
