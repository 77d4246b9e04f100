// sha1.cu -- row A4 of the hot path: SHA-1 (FIPS 180-4) of every chunk.
// "each GPU thread calculates the SHA-1 of one block. The
// result is saved in an array".
//
// Kept from the paper: one lane owns one chunk (SHA-1 is a sequential chain
// of 64-byte compressions, so a chunk cannot be split).  Changed for sm_100a:
//   * persistent warps pull chunks from a device work counter with one
//     warp-aggregated atomic; a lane that finishes its chunk picks up the next
//     one at the following 64-byte step, so lanes of a warp stay busy even
//     though chunk lengths vary from 32 B to megabytes (block-granular load
//     balancing instead of one launch thread per chunk);
//   * the 16-word message schedule lives in registers (fully unrolled
//     rounds, circular W[16]) and rotates are funnel shifts (SHF);
//   * unaligned chunk data is read with five 16-byte loads and realigned with
//     two select stages + one PRMT per word (PRMT also does the big-endian
//     byte swap).
#include <cuda_runtime.h>
#include <stdint.h>

#include "internal.h"

namespace dd {

namespace {

#ifndef DEDUP_SHA_THREADS
#define DEDUP_SHA_THREADS 512
#endif
constexpr int kShaThreads = DEDUP_SHA_THREADS;
constexpr int kShaWarps = kShaThreads / 32;
#ifndef DEDUP_SHA_MINB
#define DEDUP_SHA_MINB (kShaThreads >= 768 ? 1 : 768 / kShaThreads)
#endif
constexpr int kShaMinBlocks = DEDUP_SHA_MINB;
constexpr int kShaStateWords = 11;
#ifndef DEDUP_SHA_COMPACT_EVERY
#define DEDUP_SHA_COMPACT_EVERY 16
#endif
// iterations (64-byte blocks) between compaction points (measured, bench:
// 4 -> 715, 8 -> 736, 16 -> 744-749 GB/s)
constexpr uint32_t kCompactEvery = DEDUP_SHA_COMPACT_EVERY;
// Idle lanes of a warp refilled together (the work pull in sha1_kernel).
// Measured (1000 MiB of C2-like chunks / bench): 1 -> 592 GB/s / 719, 4 ->
// 623 / 733, 8 -> - / 720, 16 -> - / 648.
#ifndef DEDUP_SHA_REFILL_MIN
#define DEDUP_SHA_REFILL_MIN 4
#endif
constexpr int kRefillMin = DEDUP_SHA_REFILL_MIN;
constexpr uint32_t kFull = 0xFFFFFFFFu;

__device__ __forceinline__ uint32_t rotl(uint32_t x, int s) { return __funnelshift_l(x, x, s); }

#ifndef DEDUP_SHA_FMA
#define DEDUP_SHA_FMA 0
#endif

// Pipe balancing.  LOP3/SHF/LEA issue to the ALU pipe and IMAD/VIADD to the
// FMA pipe, each at half a warp instruction per clock per SMSP
// (B300_MICROARCH.md "Pipe rates").  As compiled, a round is LOP3 (f), LEA.HI
// (rotl5 + x), SHF (rotl30) on the ALU pipe and IMAD.IADD, IMAD (w + ...),
// VIADD (K) on the FMA pipe, and the schedule is 2 LOP3 + 1 SHF: ~432 ALU vs
// ~240 FMA ops per block (ncu: ALU 51 %, FMA-heavy ~1.6x less busy), so the
// block is ALU-bound.  A rotate by s is x * 2^s + (x >> (32 - s)) (the parts
// do not overlap), i.e. mad.lo(x, 2^s, mad.hi(x, 2^s, 0)): two FMA-pipe ops
// for one ALU op.  DEDUP_SHA_FMA bit 0 moves the 64 schedule rotl1 (-> ~368
// on each pipe), bit 1 the 80 rotl30.  The multipliers are kernel arguments
// (runtime values) so that ptxas cannot turn them back into shifts.
// Measured (1 GiB of 4 KiB chunks, B200): 0 -> 1750 GB/s, 1 -> 1626, 3 -> 1254:
// the kernel is issue/latency-bound, not ALU-pipe-bound, so extra instructions
// cost more than the pipe balance gains.  Default 0.
struct ShaMul {
    uint32_t one, two, p30;  // 1, 2, 2^30 at run time
};

__device__ __forceinline__ uint32_t mad_hi(uint32_t a, uint32_t b, uint32_t c) {
    uint32_t d;
    asm("mad.hi.u32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(c));
    return d;
}
__device__ __forceinline__ uint32_t mad_lo(uint32_t a, uint32_t b, uint32_t c) {
    uint32_t d;
    asm("mad.lo.u32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(c));
    return d;
}
// rotl(x, s) on the FMA pipe, m = 2^s (runtime)
__device__ __forceinline__ uint32_t rotl_fma(uint32_t x, uint32_t m) {
    return mad_lo(x, m, mad_hi(x, m, 0u));
}

// `one` is a runtime 1 (kernel argument): w * one + K compiles to an IMAD on
// the FMA pipe that ptxas cannot fold back onto the a -> a' dependency chain,
// leaving LEA.HI (rotl(a,5) + x) as the only op on it.
__device__ __forceinline__ void sha1_compress(uint32_t H[5], uint32_t W[16], ShaMul m) {
    const uint32_t one = m.one;
    uint32_t a = H[0], b = H[1], c = H[2], d = H[3], e = H[4];
#pragma unroll
    for (int t = 0; t < 80; ++t) {
        uint32_t w;
        if (t < 16) {
            w = W[t];
        } else {
            const uint32_t x = W[(t - 3) & 15] ^ W[(t - 8) & 15] ^ W[(t - 14) & 15] ^ W[t & 15];
            w = (DEDUP_SHA_FMA & 1) ? rotl_fma(x, m.two) : rotl(x, 1);
            W[t & 15] = w;
        }
        uint32_t f, K;
        if (t < 20) {
            f = (b & c) ^ (~b & d);
            K = 0x5A827999u;
        } else if (t < 40) {
            f = b ^ c ^ d;
            K = 0x6ED9EBA1u;
        } else if (t < 60) {
            f = (b & c) ^ (b & d) ^ (c & d);
            K = 0x8F1BBCDCu;
        } else {
            f = b ^ c ^ d;
            K = 0xCA62C1D6u;
        }
        // keep only rotl(a,5) + x on the a -> a' dependency chain
        const uint32_t x = (f + e) + (w * one + K);
        const uint32_t T = rotl(a, 5) + x;
        e = d;
        d = c;
        c = (DEDUP_SHA_FMA & 2) ? rotl_fma(b, m.p30) : rotl(b, 30);
        b = a;
        a = T;
    }
    H[0] += a;
    H[1] += b;
    H[2] += c;
    H[3] += d;
    H[4] += e;
}

// Raw 16-byte-aligned window [p & ~15, +80) holding the 64 message bytes at
// byte offset p.  With kGuard, vectors at or beyond lim16 read as zero.
template <bool kGuard>
__device__ __forceinline__ void load_raw(const uint8_t* __restrict__ bytes, uint64_t p,
                                         uint64_t lim16, uint32_t v[20]) {
    const uint64_t base = p & ~uint64_t(15);
    const bool need5 = (p & 15) != 0;
#pragma unroll
    for (int i = 0; i < 5; ++i) {
        uint4 x = make_uint4(0, 0, 0, 0);
        const uint64_t a = base + 16 * i;
        bool ok = (i < 4) || need5;
        if (kGuard) ok = ok && (a < lim16);
        if (ok) x = __ldg(reinterpret_cast<const uint4*>(bytes + a));
        v[4 * i] = x.x;
        v[4 * i + 1] = x.y;
        v[4 * i + 2] = x.z;
        v[4 * i + 3] = x.w;
    }
}

// Realign the raw window to byte offset (p & 15) and byte-swap to 16
// big-endian message words: two select stages for the word offset, one PRMT
// per word for the byte offset + endianness.
__device__ __forceinline__ void realign(uint32_t v[20], uint32_t o, uint32_t M[16]) {
    const uint32_t wsh = o >> 2;
#pragma unroll
    for (int i = 0; i < 18; ++i) v[i] = (wsh & 2) ? v[i + 2] : v[i];
#pragma unroll
    for (int i = 0; i < 17; ++i) v[i] = (wsh & 1) ? v[i + 1] : v[i];
    const uint32_t sel = 0x0123u + (o & 3) * 0x1111u;
#pragma unroll
    for (int j = 0; j < 16; ++j) M[j] = __byte_perm(v[j], v[j + 1], sel);
}

#ifndef DEDUP_SHA_LD64
#define DEDUP_SHA_LD64 0
#endif
// kLd64: the data window is read as nine 8-byte vectors from p & ~7 (one
// word-select stage instead of two; 4 more load instructions per block).
// Measured: isolated SHA-1 +0.5 %, bench 733 vs 746 GB/s -> off.
constexpr bool kLd64 = DEDUP_SHA_LD64 != 0;
constexpr int kRawWords = kLd64 ? 18 : 20;

template <bool kGuard>
__device__ __forceinline__ void load_raw64(const uint8_t* __restrict__ bytes, uint64_t p,
                                           uint64_t lim8, uint32_t v[18]) {
    const uint64_t base = p & ~uint64_t(7);
    const bool need9 = (p & 7) != 0;
#pragma unroll
    for (int i = 0; i < 9; ++i) {
        uint2 x = make_uint2(0, 0);
        const uint64_t a = base + 8 * i;
        bool ok = (i < 8) || need9;
        if (kGuard) ok = ok && (a < lim8);
        if (ok) x = __ldg(reinterpret_cast<const uint2*>(bytes + a));
        v[2 * i] = x.x;
        v[2 * i + 1] = x.y;
    }
}

__device__ __forceinline__ void realign64(uint32_t v[18], uint32_t o, uint32_t M[16]) {
    const uint32_t wsh = o >> 2;
#pragma unroll
    for (int i = 0; i < 17; ++i) v[i] = wsh ? v[i + 1] : v[i];
    const uint32_t sel = 0x0123u + (o & 3) * 0x1111u;
#pragma unroll
    for (int j = 0; j < 16; ++j) M[j] = __byte_perm(v[j], v[j + 1], sel);
}

template <bool kGuard>
__device__ __forceinline__ void load_any(const uint8_t* __restrict__ bytes, uint64_t p,
                                         uint64_t lim, uint32_t* v) {
    if constexpr (kLd64) load_raw64<kGuard>(bytes, p, lim, v);
    else load_raw<kGuard>(bytes, p, lim, v);
}

// Chunks of at least `long_bytes` are listed so that the SHA-1 kernel starts
// them first (longest-processing-time-first: a batch's latency is bounded by
// its longest chunk, a sequential chain of 64-byte compressions).
__global__ void long_list_kernel(const BatchDesc* __restrict__ desc,
                                 const uint32_t* __restrict__ cut_pos,
                                 const uint32_t* __restrict__ n_chunks_p, uint64_t cap,
                                 uint32_t long_bytes, uint32_t* counters,
                                 uint32_t* __restrict__ long_list) {
    const uint32_t n = (uint32_t)min((uint64_t)*n_chunks_p, cap);
    const uint64_t nbytes = desc->nbytes;
    for (uint32_t k = blockIdx.x * blockDim.x + threadIdx.x; k < n; k += gridDim.x * blockDim.x) {
        const uint64_t e = (k + 1 < n) ? (uint64_t)cut_pos[k + 1] : nbytes;
        if (e - cut_pos[k] >= long_bytes) long_list[atomicAdd(&counters[1], 1u)] = k;
    }
}

// counters[0]: work counter, counters[1]: number of long chunks.
//
// Tail compaction: once the work list is exhausted, lanes whose chunks are done
// idle while their warp keeps issuing for the lanes still hashing (long chunks
// outlive the bulk of a batch by up to ~4x).  Every kCompactEvery iterations
// the live warps of the CTA meet at a named barrier; if the list is exhausted,
// the active lanes' states (H, position, lengths) are packed through shared
// memory into the first ceil(active/32) warps and the other warps exit, so
// the issue slots of the tail go to lanes that do work.
__global__ void __launch_bounds__(kShaThreads, kShaMinBlocks)
sha1_kernel(const BatchDesc* __restrict__ desc,
            const uint32_t* __restrict__ cut_pos, const uint32_t* __restrict__ n_chunks_p,
            uint64_t cap, uint32_t long_bytes, uint32_t* counters,
            const uint32_t* __restrict__ long_list, uint8_t* __restrict__ digest, ShaMul mul) {
    __shared__ uint32_t s_state[kShaStateWords][kShaThreads];
    __shared__ uint32_t s_warp_active[kShaWarps];
    __shared__ uint32_t s_exhausted;
    const uint8_t* __restrict__ bytes = desc->bytes;
    const uint64_t nbytes = desc->nbytes;
    const uint32_t n = (uint32_t)min((uint64_t)*n_chunks_p, cap);
    const uint32_t n_long = *((volatile uint32_t*)&counters[1]);
    const uint32_t total = n + n_long;
    const uint32_t lane = threadIdx.x & 31;
    uint32_t wid = threadIdx.x >> 5;
    uint32_t live = blockDim.x >> 5;  // warps of this CTA still running (CTA-uniform)
    // vectors at or beyond lim read as zero (16- or 8-byte vectors)
    const uint64_t lim16 = kLd64 ? (nbytes + 7) & ~uint64_t(7) : (nbytes + 15) & ~uint64_t(15);
    int64_t k = -1;      // chunk owned by this lane
    uint64_t p = 0;      // byte offset of the next block's data
    uint32_t rem = 0;    // chunk bytes not yet consumed
    uint32_t len = 0;    // chunk length
    uint32_t phase = 0;  // 1: only the length block is left
    bool done = false;   // the work list is exhausted for this lane
    uint32_t H[5] = {0, 0, 0, 0, 0};
    uint32_t raw[kRawWords];  // prefetched data window of the next block
    for (uint32_t iter = 1;; ++iter) {
        // ---- pull work: long chunks first, then all others in order.  The
        // pull is a divergent stretch of the warp (ballot, atomic, chunk
        // bounds, first data window), so idle lanes wait until kRefillMin of
        // them are idle (or no lane is working) and are refilled together ----
        const uint32_t idle = __ballot_sync(kFull, !done && k < 0);
        const bool pull = idle != 0 && (kRefillMin <= 1 || __popc(idle) >= kRefillMin ||
                                         __ballot_sync(kFull, k >= 0) == 0);
        while (pull) {
            const bool need = !done && k < 0;
            const uint32_t m = __ballot_sync(kFull, need);
            if (!m) break;
            const int leader = __ffs(m) - 1;
            uint32_t base = 0;
            if ((int)lane == leader) base = atomicAdd(&counters[0], (uint32_t)__popc(m));
            base = __shfl_sync(kFull, base, leader);
            if (need) {
                const uint32_t w = base + __popc(m & ((1u << lane) - 1u));
                if (w >= total) {
                    done = true;
                } else {
                    const uint32_t idx = w < n_long ? long_list[w] : w - n_long;
                    const uint32_t s = cut_pos[idx];
                    const uint64_t e = (idx + 1 < n) ? (uint64_t)cut_pos[idx + 1] : nbytes;
                    const uint32_t L = (uint32_t)(e - s);
                    if (w < n_long || L < long_bytes) {  // else: already taken as long
                        k = idx;
                        p = s;
                        rem = len = L;
                        phase = 0;
                        H[0] = 0x67452301u;
                        H[1] = 0xEFCDAB89u;
                        H[2] = 0x98BADCFEu;
                        H[3] = 0x10325476u;
                        H[4] = 0xC3D2E1F0u;
                        load_any<true>(bytes, p, lim16, raw);
                    }
                }
            }
        }
        if (iter % kCompactEvery == 0 && live > 1) {
            // ---- CTA compaction point (all live warps arrive here together:
            // every warp runs exactly one iteration per step) ----
            const uint32_t act = __ballot_sync(kFull, k >= 0);
            const uint32_t nthr = live * 32;
            if (lane == 0) s_warp_active[wid] = __popc(act);
            // one read of the (monotone) work counter makes the decision
            // CTA-uniform: once it has passed the end, no lane can get new work
            if (threadIdx.x == 0)
                s_exhausted = *((volatile uint32_t*)&counters[0]) >= total ? 1u : 0u;
            asm volatile("bar.sync 1, %0;" ::"r"(nthr) : "memory");
            uint32_t before = 0, tot = 0;
            for (uint32_t i = 0; i < live; ++i) {
                const uint32_t c = s_warp_active[i];
                before += i < wid ? c : 0;
                tot += c;
            }
            const bool exhausted = s_exhausted != 0;
            const uint32_t new_live = (tot + 31) / 32;
            if (exhausted && new_live < live) {
                if (k >= 0) {
                    const uint32_t slot = before + __popc(act & ((1u << lane) - 1u));
#pragma unroll
                    for (int i = 0; i < 5; ++i) s_state[i][slot] = H[i];
                    s_state[5][slot] = (uint32_t)k;
                    s_state[6][slot] = (uint32_t)p;
                    s_state[7][slot] = (uint32_t)(p >> 32);
                    s_state[8][slot] = rem;
                    s_state[9][slot] = len;
                    s_state[10][slot] = phase;
                }
                asm volatile("bar.sync 1, %0;" ::"r"(nthr) : "memory");
                if (wid >= new_live) return;  // CTA-uniform per warp
                const uint32_t slot = wid * 32 + lane;
                if (slot < tot) {
#pragma unroll
                    for (int i = 0; i < 5; ++i) H[i] = s_state[i][slot];
                    k = s_state[5][slot];
                    p = (uint64_t)s_state[6][slot] | ((uint64_t)s_state[7][slot] << 32);
                    rem = s_state[8][slot];
                    len = s_state[9][slot];
                    phase = s_state[10][slot];
                    if (phase == 0 && rem > 0) load_any<true>(bytes, p, lim16, raw);
                } else {
                    k = -1;
                }
                done = true;
                live = new_live;
                // the slots are reused at the next compaction point only after
                // every remaining warp has read its state
                asm volatile("bar.sync 1, %0;" ::"r"(new_live * 32) : "memory");
            } else {
                // keep s_warp_active stable until everyone has read it
                asm volatile("bar.sync 1, %0;" ::"r"(nthr) : "memory");
            }
            if (tot == 0 && exhausted) return;
        } else if (live == 1 && __all_sync(kFull, done && k < 0)) {
            return;
        }
        if (k >= 0) {
            uint32_t M[16];
            bool fin = false;
            if (phase == 0) {
                if constexpr (kLd64) realign64(raw, (uint32_t)(p & 7), M);
                else realign(raw, (uint32_t)(p & 15), M);
                if (rem < 64) {
                    // final data block: rem (0..63) bytes, 0x80, zeros [, length]
#pragma unroll
                    for (int j = 0; j < 16; ++j) {
                        const int nv = (int)rem - 4 * j;
                        uint32_t w = M[j];
                        if (nv < 4) {
                            if (nv >= 0) {
                                const uint32_t keep =
                                    nv == 0 ? 0u : (0xFFFFFFFFu << (32 - 8 * nv));
                                w = (w & keep) | (0x80u << (24 - 8 * nv));
                            } else {
                                w = 0;
                            }
                        }
                        M[j] = w;
                    }
                    if (rem <= 55) {
                        M[14] = len >> 29;
                        M[15] = len << 3;
                        fin = true;
                    } else {
                        phase = 1;
                    }
                    rem = 0;
                } else {
                    p += 64;
                    rem -= 64;
                    // prefetch the next block's window while this one compresses
                    if (rem >= 64) load_any<false>(bytes, p, lim16, raw);
                    else if (rem > 0) load_any<true>(bytes, p, lim16, raw);
                }
            } else {
#pragma unroll
                for (int j = 0; j < 14; ++j) M[j] = 0;
                M[14] = len >> 29;
                M[15] = len << 3;
                fin = true;
            }
            sha1_compress(H, M, mul);
            if (fin) {
                uint32_t* out = reinterpret_cast<uint32_t*>(digest + 20 * (uint64_t)k);
#pragma unroll
                for (int i = 0; i < 5; ++i) out[i] = __byte_perm(H[i], 0, 0x0123);
                k = -1;
            }
        }
    }
}

}  // namespace

const char* sha1_unlaunchable() {
    if (!fits((const void*)long_list_kernel, 256, 0)) return "long_list_kernel";
    if (!fits((const void*)sha1_kernel, kShaThreads, 0)) return "sha1_kernel";
    return nullptr;
}

void launch_sha1(const BatchDesc* d, uint64_t max_bytes, const uint32_t* cut_pos,
                 const uint32_t* n_chunks, uint64_t cap, uint32_t long_bytes, uint32_t* counters,
                 uint32_t* long_list, uint8_t* digest, int num_sms, cudaStream_t s,
                 uint32_t lane_bytes) {
    cudaMemsetAsync(counters, 0, 2 * sizeof(uint32_t), s);
    // Persistent lanes pull chunks dynamically, so the grid only needs enough
    // lanes to finish the batch's bulk within its longest chunk's latency:
    // one lane per kShaLaneBytes of input keeps the per-batch footprint small
    // and leaves the SMs to the other in-flight batches.  A batch's SHA-1 CTA
    // lives until its longest chunk is hashed (a sequential chain); with
    // fewer lanes per byte the bulk of its chunks covers more of that tail.
    // Measured (bench, C2, 64 MiB batches): 4 KiB 540, 8 KiB 590, 16 KiB
    // 619, 24 KiB 620, 32 KiB 632-641 (40 slots), 64 KiB 494 GB/s.
#ifndef DEDUP_SHA_LANE_BYTES
#define DEDUP_SHA_LANE_BYTES 32768
#endif
    const uint64_t kShaLaneBytes = lane_bytes ? lane_bytes : DEDUP_SHA_LANE_BYTES;
    uint64_t lanes = max_bytes / kShaLaneBytes;
// At least 4 CTAs per batch: smaller batches then finish their SHA-1 sooner
// (a batch's latency is its lanes' serial chains) and keep up the in-flight
// volume.  Measured (C2 sweep, 40 slots): min 1024 -> 16 MiB 319, 32 MiB 458,
// 64 MiB 734 GB/s; 2048 -> 382, 566, 732; 4096 -> 389, 597, 705.
#ifndef DEDUP_SHA_MIN_LANES
#define DEDUP_SHA_MIN_LANES 2048
#endif
    if (lanes < DEDUP_SHA_MIN_LANES) lanes = DEDUP_SHA_MIN_LANES;
    uint64_t blocks = (lanes + kShaThreads - 1) / kShaThreads;
    if (blocks > (uint64_t)num_sms * kShaMinBlocks) blocks = (uint64_t)num_sms * kShaMinBlocks;
    uint64_t lb = (cap + 255) / 256;
    if (lb > (uint64_t)num_sms * 2) lb = (uint64_t)num_sms * 2;
    if (lb < 1) lb = 1;
    long_list_kernel<<<(unsigned)lb, 256, 0, s>>>(d, cut_pos, n_chunks, cap, long_bytes, counters,
                                                  long_list);
    sha1_kernel<<<(unsigned)blocks, kShaThreads, 0, s>>>(d, cut_pos, n_chunks, cap, long_bytes,
                                                         counters, long_list, digest,
                                                         ShaMul{1u, 2u, 1u << 30});
}

}  // namespace dd
