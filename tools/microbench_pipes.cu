// microbench_pipes.cu -- which sm_100a pipe executes each integer opcode the
// SHA-1 and scan kernels use, and at what rate, alone and mixed.
// Standalone (not part of the product):
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/mbp tools/microbench_pipes.cu
//   /tmp/mbp            (prints T ops/s per kind; run under ncu with
//                        sm__inst_executed_pipe_{alu,fmaheavy,fmalite} for the pipe split)
// Every op is inline PTX in an asm volatile on one of 8 independent chains per
// thread; 2 x 1024 threads per SM.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

constexpr int kChains = 8;
constexpr int kUnroll = 24;
constexpr int kThreads = 1024;

enum Kind {
    kLop3, kImad, kAddReg, kAddImm, kMadOne, kLeaHi, kShf, kPrmt,
    kMixLopAddImm,      // LOP3 / add-immediate alternating
    kMixLopAddReg,      // LOP3 / add reg alternating
    kMixLopImadAddImm,  // LOP3, IMAD, add-imm round robin (3 pipes?)
    kMix2Lop1Imad1Add,  // LOP3, LOP3, IMAD, add-imm
    kMixLopImad,
    kKinds
};
const char* names[] = {"lop3", "imad", "add_reg", "add_imm", "mad_one", "lea_hi", "shf", "prmt",
                       "lop3|add_imm", "lop3|add_reg", "lop3|imad|add_imm",
                       "lop3|lop3|imad|add_imm", "lop3|imad"};

template <int K>
__device__ __forceinline__ void op(uint32_t& x, uint32_t y, uint32_t z) {
    if constexpr (K == kLop3) {
        asm volatile("lop3.b32 %0, %0, %1, %2, 0x96;" : "+r"(x) : "r"(y), "r"(z));
    } else if constexpr (K == kImad) {
        asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(x) : "r"(y), "r"(z));
    } else if constexpr (K == kAddReg) {  // (alone: ptxas fuses pairs into IADD3)
        asm volatile("add.u32 %0, %0, %1;" : "+r"(x) : "r"(y));
    } else if constexpr (K == kAddImm) {
        asm volatile("add.u32 %0, %0, 0x5A827999;" : "+r"(x));
    } else if constexpr (K == kMadOne) {
        asm volatile("mad.lo.u32 %0, %0, %1, 0x5A827999;" : "+r"(x) : "r"(z));
    } else if constexpr (K == kLeaHi) {
        asm volatile("{\n\t.reg .u32 t;\n\tshf.l.wrap.b32 t, %0, %0, 5;\n\tadd.u32 %0, t, %1;\n\t}"
                     : "+r"(x) : "r"(y));
    } else if constexpr (K == kShf) {
        asm volatile("shf.l.wrap.b32 %0, %0, %0, 5;" : "+r"(x));
    } else if constexpr (K == kPrmt) {
        asm volatile("prmt.b32 %0, %0, %1, 0x0123;" : "+r"(x) : "r"(y));
    }
}

template <int K>
__global__ void __launch_bounds__(kThreads, 2) probe(uint32_t* out, int trips, uint32_t s) {
    uint32_t x[kChains];
#pragma unroll
    for (int c = 0; c < kChains; ++c) x[c] = threadIdx.x * 2654435761u + c * s;
    const uint32_t y = s * 7u + 1u, z = s ^ 0x5bd1e995u;
    for (int t = 0; t < trips; ++t) {
#pragma unroll
        for (int u = 0; u < kUnroll; ++u) {
#pragma unroll
            for (int c = 0; c < kChains; ++c) {
                // mixes: each chain alternates kinds (no two foldable adds in a row)
                if constexpr (K == kMixLopAddImm) {
                    if (u & 1) op<kAddImm>(x[c], y, z); else op<kLop3>(x[c], y, z);
                } else if constexpr (K == kMixLopAddReg) {
                    if (u & 1) op<kAddReg>(x[c], y, z); else op<kLop3>(x[c], y, z);
                } else if constexpr (K == kMixLopImadAddImm) {
                    const int r = u % 3;  // LOP3, IMAD, add-imm, ...
                    if (r == 0) op<kLop3>(x[c], y, z);
                    else if (r == 1) op<kImad>(x[c], y, z);
                    else op<kAddImm>(x[c], y, z);
                } else if constexpr (K == kMix2Lop1Imad1Add) {
                    const int r = u & 3;  // LOP3, IMAD, LOP3, add-imm
                    if (r == 0 || r == 2) op<kLop3>(x[c], y, z);
                    else if (r == 1) op<kImad>(x[c], y, z);
                    else op<kAddImm>(x[c], y, z);
                } else if constexpr (K == kMixLopImad) {
                    if (u & 1) op<kImad>(x[c], y, z); else op<kLop3>(x[c], y, z);
                } else {
                    op<K>(x[c], y, z);
                }
            }
        }
    }
    uint32_t r = 0;
#pragma unroll
    for (int c = 0; c < kChains; ++c) r ^= x[c];
    if (r == 0x12345678u) out[threadIdx.x] = r;
}

template <int K>
void run(int sms, int trips, uint32_t* out) {
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    const int blocks = 2 * sms;
    probe<K><<<blocks, kThreads>>>(out, trips / 8, 1u);
    cudaEventRecord(e0);
    probe<K><<<blocks, kThreads>>>(out, trips, 1u);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms = 0;
    cudaEventElapsedTime(&ms, e0, e1);
    const double ops = (double)blocks * kThreads * trips * kUnroll * kChains;
    printf("%-24s %7.2f T ops/s  %.3f warp-inst/clk/SMSP\n", names[K], ops / (ms * 1e-3) / 1e12,
           ops / 32 / (ms * 1e-3) / (sms * 4) / 1.965e9);
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
}

template <int... Ks>
void run_all(int sms, int trips, uint32_t* out, std::integer_sequence<int, Ks...>) {
    (run<Ks>(sms, trips, out), ...);
}

int main() {
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    uint32_t* buf;
    cudaMalloc(&buf, kThreads * 4);
    run_all(sms, 2048, buf, std::make_integer_sequence<int, kKinds>{});
    printf("err %s\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
