// sha1.cu -- row A4 of the hot path: SHA-1 (FIPS 180-4) of every chunk.
// "each GPU thread calculates the SHA-1 of one block. The
// result is saved in an array".
//
// Kept from the paper: one lane owns one chunk (SHA-1 is a sequential chain
// of 64-byte compressions, so a chunk cannot be split).  Changed for sm_100a:
//   * the chunks of a batch are counting-sorted by their number of 64-byte
//     compressions, longest first (sha_hist / sha_scan / sha_scatter: three
//     small kernels over the cut list), and a warp takes 32 consecutive
//     chunks of that order as one task: its lanes then run the same number
//     of compressions (up to the few blocks by which neighbours differ), so
//     the warp works in lock-step -- no per-lane work pulls, no divergent
//     final-block branches in the bulk, and the longest chunks start first
//     (a batch's latency is bounded by its longest chunk's serial chain);
//   * the bulk blocks (every lane's block is 64 data bytes) run without any
//     per-block test; only the last blocks of a task (padding, length,
//     lanes already done) take the guarded path;
//   * the 16-word message schedule lives in registers (fully unrolled
//     rounds, circular W[16]) and rotates are funnel shifts (SHF);
//   * unaligned chunk data is read as an 80-byte window of five 16-byte
//     vectors (the next block's window prefetched during the compression;
//     its first vector is this window's last, kept in registers, so a block
//     costs four loads: isolated SHA-1 1.82 -> 1.89 TB/s) and realigned with
//     two select stages + one PRMT per word (PRMT also does the big-endian
//     swap).
//     Measured alternative (C3, 672 MiB): staging the window in shared memory
//     with cp.async and reading it back with 17 LDS at the lane's offset saves
//     the 34 selects (isolated 805 vs 750 GB/s) but its 40 KiB per CTA keeps
//     SHA-1 CTAs off the SMs that hold a scan CTA: bench 744 vs 790 GB/s.
#include <cuda_runtime.h>
#include <stdint.h>

#include "internal.h"

namespace dd {

namespace {

constexpr int kShaThreads = 256;
constexpr int kShaMinBlocks = 4;  // CTAs per SM (launch bounds: <= 64 registers)
constexpr uint32_t kFull = 0xFFFFFFFFu;

// Sort keys: the number of compressions nb of a chunk; nb < kExact gets its
// own bucket, longer chunks share buckets of 64 compressions (4 KiB).
constexpr uint32_t kBuckets = 4096;
constexpr uint32_t kExact = 2048;
// workspace words: [0, kBuckets) histogram, [kBuckets, 2 kBuckets) cursors,
// [2 kBuckets] task counter, [kOrderOff, ..) the sorted chunk order
constexpr uint32_t kOrderOff = 2 * kBuckets + 64;

__device__ __forceinline__ uint32_t sha_blocks(uint64_t L) { return (uint32_t)((L + 9 + 63) >> 6); }
__device__ __forceinline__ uint32_t bucket_of(uint32_t nb) {
    const uint32_t b = nb < kExact ? nb : kExact + ((nb - kExact) >> 6);
    return b < kBuckets - 1 ? b : kBuckets - 1;
}

__device__ __forceinline__ uint32_t rotl(uint32_t x, int s) { return __funnelshift_l(x, x, s); }

// `one` is a runtime 1 (kernel argument): w * one + ... compiles to an IMAD
// on the FMA pipe, which balances the ALU pipe (LOP3 f, LEA.HI rotl5 + add,
// SHF rotl30, the schedule's LOP3/SHF) against the FMA pipe (the other adds;
// measured on B200: LOP3/SHF/LEA.HI/IMAD 16 lanes/clk/SMSP each, IMAD.HI 8).
// Measured alternative (C3 bench, 300 steps): the rotates as IMAD.HI +
// IMAD on the FMA pipe (x * 2^s + hi(x * 2^s)) -- rotl30: 773 GB/s, the
// schedule's rotl1: 781, SHF (kept): 805; IMAD.HI's half rate costs more
// than the ALU slot it frees.
__device__ __forceinline__ void sha1_compress(uint32_t H[5], uint32_t W[16], uint32_t one) {
    uint32_t a = H[0], b = H[1], c = H[2], d = H[3], e = H[4];
#pragma unroll
    for (int t = 0; t < 80; ++t) {
        uint32_t w;
        if (t < 16) {
            w = W[t];
        } else {
            const uint32_t xw = W[(t - 3) & 15] ^ W[(t - 8) & 15] ^ W[(t - 14) & 15] ^ W[t & 15];
            w = rotl(xw, 1);
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
        // x does not depend on a: the empty asm pins it (K included) so
        // that only LEA.HI (rotl(a, 5) + x) is on the a -> a' chain; ptxas
        // otherwise adds K after the LEA.HI, a 9-cycle round instead of 4
        uint32_t x = (f + e) + (w * one + K);
        asm volatile("" : "+r"(x));
        const uint32_t T = rotl(a, 5) + x;
        e = d;
        d = c;
        c = rotl(b, 30);
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
    DD_CHECK(kGuard || base + (need5 ? 80 : 64) <= lim16);
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

// The next block's window, base + 64: its vector 0 is this window's vector 4
// when that one was loaded (p & 15 != 0, the same for every block of a chunk),
// so only 4 vectors are loaded per block either way.
template <bool kGuard>
__device__ __forceinline__ void load_next(const uint8_t* __restrict__ bytes, uint64_t p,
                                          uint64_t lim16, uint32_t v[20], bool need5) {
    const uint64_t base = p & ~uint64_t(15);
    DD_CHECK(kGuard || base + (need5 ? 80 : 64) <= lim16);
    uint4 x0 = make_uint4(v[16], v[17], v[18], v[19]);
    if (!need5) {
        x0 = make_uint4(0, 0, 0, 0);
        if (!kGuard || base < lim16) x0 = __ldg(reinterpret_cast<const uint4*>(bytes + base));
    }
    v[0] = x0.x;
    v[1] = x0.y;
    v[2] = x0.z;
    v[3] = x0.w;
#pragma unroll
    for (int i = 1; i < 5; ++i) {
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

// a + (b - a) * m for m in {0, 1}, as two IMADs (inline PTX: ptxas would turn
// the arithmetic back into a SEL on the ALU pipe)
__device__ __forceinline__ uint32_t fma_select(uint32_t a, uint32_t b, uint32_t m) {
    uint32_t d, r;
    asm("mad.lo.u32 %0, %1, 0xFFFFFFFF, %2;" : "=r"(d) : "r"(a), "r"(b));
    asm("mad.lo.u32 %0, %1, %2, %3;" : "=r"(r) : "r"(d), "r"(m), "r"(a));
    return r;
}

// Realign the raw window to byte offset o = p & 15 and byte-swap to 16
// big-endian message words: two select stages for the word offset, one PRMT
// per word for the byte offset + endianness.
__device__ __forceinline__ void realign(const uint32_t raw[20], uint32_t o, uint32_t M[16]) {
    uint32_t v[20];
#pragma unroll
    for (int i = 0; i < 20; ++i) v[i] = raw[i];
    const uint32_t wsh = o >> 2;
    // word-select stages on the FMA pipe: v = v + (v' - v) * bit (IMAD x 2),
    // the ALU pipe being the kernel's binding pipe
    const uint32_t m2 = (wsh >> 1) & 1, m1 = wsh & 1;
#pragma unroll
    for (int i = 0; i < 18; ++i) v[i] = fma_select(v[i], v[i + 2], m2);
#pragma unroll
    for (int i = 0; i < 17; ++i) v[i] = fma_select(v[i], v[i + 1], m1);
    const uint32_t sel = 0x0123u + (o & 3) * 0x1111u;
#pragma unroll
    for (int j = 0; j < 16; ++j) M[j] = __byte_perm(v[j], v[j + 1], sel);
}

// FIPS 180-4 5.1.1 padding of the block whose data starts r bytes before the
// chunk end (r < 64): data bytes [0, r), 0x80 at r, zeros, and the 64-bit
// big-endian bit length in words 14-15 if `last`.  r < 0: the length-only
// block after a block with 56..63 data bytes.
__device__ __forceinline__ void pad_block(uint32_t M[16], int32_t r, bool last, uint32_t L) {
#pragma unroll
    for (int j = 0; j < 16; ++j) {
        const int32_t nv = r - 4 * j;
        uint32_t w = M[j];
        if (nv < 4) {
            if (nv >= 0) {
                const uint32_t keep = nv == 0 ? 0u : (0xFFFFFFFFu << (32 - 8 * nv));
                w = (w & keep) | (0x80u << (24 - 8 * nv));
            } else {
                w = 0;
            }
        }
        M[j] = w;
    }
    if (last) {
        M[14] = L >> 29;
        M[15] = L << 3;
    }
}

__device__ __forceinline__ void chunk_bounds(const uint32_t* __restrict__ cut_pos, uint32_t k,
                                             uint32_t n, uint64_t nbytes, uint32_t& s,
                                             uint32_t& L) {
    s = cut_pos[k];
    const uint64_t e = (k + 1 < n) ? (uint64_t)cut_pos[k + 1] : nbytes;
    L = (uint32_t)(e - s);
}

// Carry-over mode (row NEXT-2): the last chunk of a piece (from its last cut
// to the piece end) is OPEN -- it continues into the next piece, so only its
// full 64-byte blocks are compressed here and its state goes to carry_out.
__device__ __forceinline__ bool last_is_open(const BatchDesc* desc) {
    return (desc->carry & kCarryMode) && !(desc->carry & kCarryClose);
}
__device__ __forceinline__ uint32_t task_blocks(uint64_t L, bool open) {
    return open ? (uint32_t)(L >> 6) : sha_blocks(L);
}

// ---- counting sort of the chunks by compressions, longest first ----------
__global__ void sha_hist_kernel(const BatchDesc* __restrict__ desc,
                                const uint32_t* __restrict__ cut_pos,
                                const uint32_t* __restrict__ n_chunks_p, uint64_t cap,
                                uint32_t* __restrict__ ws) {
    const uint32_t n = (uint32_t)min((uint64_t)*n_chunks_p, cap);
    const uint64_t nbytes = desc->nbytes;
    const bool open_last = last_is_open(desc);
    for (uint32_t k = blockIdx.x * blockDim.x + threadIdx.x; k < n; k += gridDim.x * blockDim.x) {
        uint32_t s, L;
        chunk_bounds(cut_pos, k, n, nbytes, s, L);
        const uint32_t b = bucket_of(task_blocks(L, open_last && k + 1 == n));
        const uint32_t peers = __match_any_sync(__activemask(), b);
        if ((threadIdx.x & 31) == (uint32_t)(__ffs(peers) - 1)) atomicAdd(&ws[b], __popc(peers));
    }
}

// One CTA of 1024 threads: cursor[b] = chunks in buckets above b (descending
// order), task counter = 0.
__global__ void __launch_bounds__(1024) sha_scan_kernel(uint32_t* __restrict__ ws) {
    __shared__ uint32_t warp_sum[32];
    const uint32_t t = threadIdx.x, lane = t & 31, wid = t >> 5;
    // thread t owns the 4 buckets at descending positions 4t .. 4t + 3
    uint32_t h[4], sum = 0;
#pragma unroll
    for (int q = 0; q < 4; ++q) {
        h[q] = ws[kBuckets - 1 - (4 * t + q)];
        sum += h[q];
    }
    uint32_t incl = sum;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const uint32_t y = __shfl_up_sync(kFull, incl, d);
        if (lane >= (uint32_t)d) incl += y;
    }
    if (lane == 31) warp_sum[wid] = incl;
    __syncthreads();
    if (wid == 0) {
        uint32_t x = warp_sum[lane], xi = x;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const uint32_t y = __shfl_up_sync(kFull, xi, d);
            if (lane >= (uint32_t)d) xi += y;
        }
        warp_sum[lane] = xi - x;  // exclusive prefix of the warps
    }
    __syncthreads();
    uint32_t run = warp_sum[wid] + incl - sum;
#pragma unroll
    for (int q = 0; q < 4; ++q) {
        ws[kBuckets + kBuckets - 1 - (4 * t + q)] = run;
        run += h[q];
    }
    if (t == 0) ws[2 * kBuckets] = 0;
}

__global__ void sha_scatter_kernel(const BatchDesc* __restrict__ desc,
                                   const uint32_t* __restrict__ cut_pos,
                                   const uint32_t* __restrict__ n_chunks_p, uint64_t cap,
                                   uint32_t* __restrict__ ws) {
    const uint32_t n = (uint32_t)min((uint64_t)*n_chunks_p, cap);
    const uint64_t nbytes = desc->nbytes;
    uint32_t* order = ws + kOrderOff;
    const bool open_last = last_is_open(desc);
    for (uint32_t k = blockIdx.x * blockDim.x + threadIdx.x; k < n; k += gridDim.x * blockDim.x) {
        uint32_t s, L;
        chunk_bounds(cut_pos, k, n, nbytes, s, L);
        const uint32_t b = bucket_of(task_blocks(L, open_last && k + 1 == n));
        const uint32_t peers = __match_any_sync(__activemask(), b);
        const uint32_t lane = threadIdx.x & 31;
        const int leader = __ffs(peers) - 1;
        uint32_t base = 0;
        if ((int)lane == leader) base = atomicAdd(&ws[kBuckets + b], __popc(peers));
        base = __shfl_sync(peers, base, leader);
        order[base + __popc(peers & ((1u << lane) - 1u))] = k;
    }
}

// Persistent warps; a task = 32 consecutive chunks of the sorted order.
__global__ void __launch_bounds__(kShaThreads, kShaMinBlocks)
sha1_kernel(const BatchDesc* __restrict__ desc, const uint32_t* __restrict__ cut_pos,
            const uint32_t* __restrict__ n_chunks_p, uint64_t cap, uint32_t* ws,
            uint8_t* __restrict__ digest, uint32_t one) {
    const uint8_t* __restrict__ bytes = desc->bytes;
    const uint64_t nbytes = desc->nbytes;
    const uint64_t lim16 = (nbytes + 15) & ~uint64_t(15);  // vectors beyond read as zero
    const uint32_t n = (uint32_t)min((uint64_t)*n_chunks_p, cap);
    const uint32_t ntasks = (n + 31) >> 5;
    const uint32_t* __restrict__ order = ws + kOrderOff;
    const uint32_t lane = threadIdx.x & 31;
    const bool open_last = last_is_open(desc);
    // carry-over continuation: reported chunk 0 is the one continued from the
    // previous piece (hashed by carry_cont_kernel); the cut list's chunks follow
    const uint32_t shift = (desc->carry & kCarryCont) ? 1u : 0u;
    for (;;) {
        uint32_t task = 0;
        if (lane == 0) task = atomicAdd(&ws[2 * kBuckets], 1u);
        task = __shfl_sync(kFull, task, 0);
        if (task >= ntasks) return;
        const uint32_t idx = 32 * task + lane;
        const bool act = idx < n;
        uint32_t k = 0, s = 0, L = 0, nb = 0;
        bool open = false;
        if (act) {
            k = order[idx];
            chunk_bounds(cut_pos, k, n, nbytes, s, L);
            open = open_last && k + 1 == n;
            nb = task_blocks(L, open);
        }
        const uint32_t nb_max = __reduce_max_sync(kFull, nb);
        const uint32_t nb_min = __reduce_min_sync(kFull, act ? nb : kFull);
        // blocks [0, nbulk) hold 64 data bytes on every active lane.  Idle
        // lanes (the last task, past the last chunk) run them from byte 0 of
        // the batch: one bulk block less then keeps their unguarded window
        // loads below 64 nb_min - 112 <= the shortest active chunk, so inside
        // the batch (the guarded tail path takes that block)
        uint32_t nbulk = nb_min >= 3 ? nb_min - 2 : 0;
        if (32 * task + 31 >= n && nbulk > 0) --nbulk;
        const uint32_t o = s & 15;
        uint32_t H[5] = {0x67452301u, 0xEFCDAB89u, 0x98BADCFEu, 0x10325476u, 0xC3D2E1F0u};
        uint32_t raw[20];
        uint64_t p = s;
        if (nbulk > 0) load_raw<false>(bytes, p, lim16, raw);
        else load_raw<true>(bytes, p, lim16, raw);
        uint32_t M[16];
#ifdef DEDUP_SHA_U2
#pragma unroll 2
#endif
        for (uint32_t i = 0; i < nbulk; ++i) {
            realign(raw, o, M);
            p += 64;
            // prefetch the next block's window while this one compresses
            if (i + 1 < nbulk) load_next<false>(bytes, p, lim16, raw, o != 0);
            else load_next<true>(bytes, p, lim16, raw, o != 0);
            sha1_compress(H, M, one);
        }
        for (uint32_t i = nbulk; i < nb_max; ++i) {
            if (i < nb) {
                realign(raw, o, M);
                p += 64;
                if (i + 1 < nb) load_next<true>(bytes, p, lim16, raw, o != 0);
                pad_block(M, (int32_t)L - (int32_t)(64 * i), i + 1 == nb && !open, L);
                sha1_compress(H, M, one);
            }
        }
        if (act && !open) {
            uint32_t* out = reinterpret_cast<uint32_t*>(digest + 20 * (uint64_t)(k + shift));
#pragma unroll
            for (int i = 0; i < 5; ++i) out[i] = __byte_perm(H[i], 0, 0x0123);
        } else if (act) {  // the open chunk's state for the next piece
            CarryState* co = desc->carry_out;
#pragma unroll
            for (int i = 0; i < 5; ++i) co->H[i] = H[i];
            co->open_len = L;
            const uint32_t done = 64 * nb;
            co->left_n = L - done;
            for (uint32_t j = done; j < L; ++j) co->left[j - done] = bytes[s + j];
        }
    }
}

}  // namespace

void sha1_set_carveout(int pct) {
    for (const void* f : {(const void*)sha_hist_kernel, (const void*)sha_scan_kernel,
                          (const void*)sha_scatter_kernel, (const void*)sha1_kernel})
        cudaFuncSetAttribute(f, cudaFuncAttributePreferredSharedMemoryCarveout, pct);
}

const char* sha1_unlaunchable() {
    if (!fits((const void*)sha_hist_kernel, 256, 0)) return "sha_hist_kernel";
    if (!fits((const void*)sha_scan_kernel, 1024, 0)) return "sha_scan_kernel";
    if (!fits((const void*)sha_scatter_kernel, 256, 0)) return "sha_scatter_kernel";
    if (!fits((const void*)sha1_kernel, kShaThreads, 0)) return "sha1_kernel";
    return nullptr;
}

uint64_t sha1_ws_words(uint64_t cap) { return kOrderOff + cap; }

void launch_sha1(const BatchDesc* d, uint64_t max_bytes, const uint32_t* cut_pos,
                 const uint32_t* n_chunks, uint64_t cap, uint32_t* ws, uint8_t* digest,
                 int num_sms, cudaStream_t s, uint32_t lane_bytes) {
    cudaMemsetAsync(ws, 0, kBuckets * sizeof(uint32_t), s);
    uint64_t lb = (cap + 255) / 256;
    if (lb > (uint64_t)num_sms * 2) lb = (uint64_t)num_sms * 2;
    if (lb < 1) lb = 1;
    sha_hist_kernel<<<(unsigned)lb, 256, 0, s>>>(d, cut_pos, n_chunks, cap, ws);
    sha_scan_kernel<<<1, 1024, 0, s>>>(ws);
    sha_scatter_kernel<<<(unsigned)lb, 256, 0, s>>>(d, cut_pos, n_chunks, cap, ws);
    // Persistent warps take tasks dynamically, so the grid only needs enough
    // lanes to finish the batch's bulk within its longest chunk's latency:
    // one lane per lane_bytes of input keeps the per-batch footprint small
    // and leaves the SMs to the other in-flight batches.
    const uint64_t per_lane = lane_bytes ? lane_bytes : 16384;
    uint64_t lanes = max_bytes / per_lane;
    if (lanes < 2048) lanes = 2048;
    uint64_t blocks = (lanes + kShaThreads - 1) / kShaThreads;
    if (blocks > (uint64_t)num_sms * kShaMinBlocks) blocks = (uint64_t)num_sms * kShaMinBlocks;
    sha1_kernel<<<(unsigned)blocks, kShaThreads, 0, s>>>(d, cut_pos, n_chunks, cap, ws, digest,
                                                         1u);
}

}  // namespace dd
