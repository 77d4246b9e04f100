// carry.cu -- row NEXT-2, carry-over mode (dedup_config.carry_over): the whole
// byte stream of a dedup stream is ONE chunking domain, submitted in pieces cut
// anywhere (north_star: "the chunking is identical when the input is split
// at arbitrary batch cuts"; PARSEC's serial pipeline carries the unfinished
// tail of a buffer into the next, while the paper changed that fragmentation
// to fixed 1 MB batches).
//
// With min chunk = window = 32 the chunker's whole state at a piece boundary
// is O(1) and passed from piece to piece in device memory (CarryState):
//   * the stream's last 32 bytes (the windows that straddle the boundary:
//     the scan's first lane rolls them as its warm-up);
//   * the selection state: positions still blocked after the last cut (the
//     next piece's entry state of the greedy state machine);
//   * the OPEN chunk (from the last cut to the piece end): its SHA-1 state
//     after its full 64-byte blocks (sha1_kernel), its length and the < 64
//     bytes not yet compressed.
// Three kernels per piece, chained to the previous piece's batch by events
// (the batch slots are used round-robin, so the previous piece's state is
// the previous slot's CarryState):
//   carry_hist_kernel   this piece's last-32-bytes history (needs the
//                       previous history only for pieces shorter than 32 B);
//   carry_meta_kernel   the piece's reported chunks (the continued chunk,
//                       then the chunks between its cuts; the open one is
//                       reported by a later piece), their ids and starts, the
//                       exit state;
//   carry_cont_kernel   finishes the continued chunk: the previous piece's
//                       open state + this piece's bytes up to its first cut
//                       (one thread: a chunk is a sequential chain of
//                       compressions), or carries it through a piece without
//                       a cut.
#include <cuda_runtime.h>
#include <stdint.h>

#include "internal.h"

namespace dd {

namespace {

__device__ __forceinline__ uint32_t rotl(uint32_t x, int s) { return __funnelshift_l(x, x, s); }

// FIPS 180-4 6.1.2 on one 64-byte block given as 16 big-endian words.
__device__ void compress(uint32_t H[5], uint32_t W[16]) {
    uint32_t a = H[0], b = H[1], c = H[2], d = H[3], e = H[4];
#pragma unroll
    for (int t = 0; t < 80; ++t) {
        uint32_t w;
        if (t < 16) {
            w = W[t];
        } else {
            w = rotl(W[(t - 3) & 15] ^ W[(t - 8) & 15] ^ W[(t - 14) & 15] ^ W[t & 15], 1);
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
        const uint32_t T = rotl(a, 5) + f + e + K + w;
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

// 64 buffered bytes -> big-endian words -> compress
__device__ void compress_bytes(uint32_t H[5], const uint8_t* buf) {
    uint32_t W[16];
#pragma unroll
    for (int j = 0; j < 16; ++j)
        W[j] = ((uint32_t)buf[4 * j] << 24) | ((uint32_t)buf[4 * j + 1] << 16) |
               ((uint32_t)buf[4 * j + 2] << 8) | (uint32_t)buf[4 * j + 3];
    compress(H, W);
}

// The stream's last 32 bytes after this piece: history ++ bytes, last 32.
__global__ void carry_hist_kernel(const BatchDesc* __restrict__ desc) {
    const uint32_t j = threadIdx.x;  // 32 threads
    const uint64_t nbytes = desc->nbytes;
    const bool cont = (desc->carry & kCarryCont) != 0;
    const int64_t p = (int64_t)nbytes - 32 + j;
    uint8_t v = 0;
    if (p >= 0) v = desc->bytes[p];
    else if (cont) v = desc->carry_in->hist[32 + p];
    __syncwarp();  // every lane read carry_in before carry_out is written
    desc->carry_out->hist[j] = v;
}

// Reported chunks of the piece.  n = cuts of the piece (select), m = reported:
// the continued chunk (if the piece continues a stream and closes it: a cut
// in the piece, or the closing batch), then [cut_k, cut_k+1) for k < n - 1;
// [cut_{n-1}, end) is open (reported later), except in the closing batch
// (which has no bytes and no cuts).  extra[0..1] = bytes of chunk 0 that lie
// in earlier pieces (u64), extra[2] = end of the last reported chunk.
__global__ void carry_meta_kernel(const BatchDesc* __restrict__ desc,
                                  const uint32_t* __restrict__ n_cuts_p,
                                  const uint32_t* __restrict__ cut_pos, uint64_t cap,
                                  uint32_t* __restrict__ m_out, uint32_t* __restrict__ chunk_start,
                                  uint64_t* __restrict__ chunk_id, uint32_t* __restrict__ item_first,
                                  uint32_t* __restrict__ extra) {
    const uint32_t fl = desc->carry;
    const bool cont = (fl & kCarryCont) != 0, close = (fl & kCarryClose) != 0;
    const uint32_t n = (uint32_t)min((uint64_t)*n_cuts_p, cap);
    const uint64_t nbytes = desc->nbytes;
    const uint32_t has_cont = (cont && (n > 0 || close)) ? 1u : 0u;
    const uint32_t interior = n > 0 ? (close ? n : n - 1) : 0u;
    const uint32_t m = has_cont + interior;
    const uint64_t seq = desc->first_seq;
    for (uint32_t r = threadIdx.x; r < m; r += blockDim.x) {
        chunk_start[r] = (has_cont && r == 0) ? 0u : cut_pos[r - has_cont];
        chunk_id[r] = (seq << 32) | r;
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        *m_out = m;
        item_first[0] = m ? 0u : 0xFFFFFFFFu;
        // (extra[0..1], the carried bytes, come from carry_cont_kernel: the
        // previous piece's open length is final only after its SHA-1)
        extra[2] = n > 0 ? cut_pos[n - 1] : 0u;
        uint32_t ex = 0;  // positions still blocked after the piece
        if (n > 0) {
            const uint64_t E = (uint64_t)cut_pos[n - 1] + 32;
            ex = E > nbytes ? (uint32_t)(E - nbytes) : 0u;
        } else if (cont) {
            const uint32_t in = desc->carry_in->exit_state;
            ex = in > nbytes ? (uint32_t)(in - nbytes) : 0u;
        }
        desc->carry_out->exit_state = ex;
    }
}

// 16 big-endian message words at byte offset p of a 16-byte aligned buffer
// readable to its length rounded up to 16: five 16-byte loads, two word-select
// stages and a PRMT per word (as sha1_kernel).
__device__ __forceinline__ void load_block(const uint8_t* __restrict__ bytes, uint64_t p,
                                           uint32_t W[16]) {
    const uint64_t base = p & ~uint64_t(15);
    uint32_t v[20];
#pragma unroll
    for (int i = 0; i < 5; ++i) {
        uint4 x = make_uint4(0, 0, 0, 0);
        if (i < 4 || (p & 15)) x = __ldg(reinterpret_cast<const uint4*>(bytes + base + 16 * i));
        v[4 * i] = x.x;
        v[4 * i + 1] = x.y;
        v[4 * i + 2] = x.z;
        v[4 * i + 3] = x.w;
    }
    const uint32_t o = (uint32_t)(p & 15), wsh = o >> 2;
#pragma unroll
    for (int i = 0; i < 18; ++i) v[i] = (wsh & 2) ? v[i + 2] : v[i];
#pragma unroll
    for (int i = 0; i < 17; ++i) v[i] = (wsh & 1) ? v[i + 1] : v[i];
    const uint32_t sel = 0x0123u + (o & 3) * 0x1111u;
#pragma unroll
    for (int j = 0; j < 16; ++j) W[j] = __byte_perm(v[j], v[j + 1], sel);
}

// The continued chunk: the previous piece's open state + this piece's bytes
// up to its first cut (the whole piece if it has none).  Finished (digest =
// reported chunk 0, carried bytes to extra[0..1]) if the piece has a cut or
// closes the stream; else the open state moves on to carry_out.
__global__ void carry_cont_kernel(const BatchDesc* __restrict__ desc,
                                  const uint32_t* __restrict__ n_cuts_p,
                                  const uint32_t* __restrict__ cut_pos, uint64_t cap,
                                  uint8_t* __restrict__ digest, uint32_t* __restrict__ extra) {
    if (threadIdx.x != 0) return;
    const uint32_t fl = desc->carry;
    if (!(fl & kCarryCont)) return;
    const CarryState& in = *desc->carry_in;
    CarryState& out = *desc->carry_out;
    const uint32_t n = (uint32_t)min((uint64_t)*n_cuts_p, cap);
    const bool finish = n > 0 || (fl & kCarryClose);
    const uint8_t* __restrict__ bytes = desc->bytes;
    const uint64_t plen = n > 0 ? (uint64_t)cut_pos[0] : desc->nbytes;
    const uint64_t open_len = in.open_len;
    uint32_t H[5];
#pragma unroll
    for (int i = 0; i < 5; ++i) H[i] = in.H[i];
    uint8_t buf[64];
    uint32_t bn = in.left_n;
    for (uint32_t i = 0; i < bn; ++i) buf[i] = in.left[i];
    uint64_t pos = 0;
    if (bn > 0) {  // complete the buffered block first
        const uint64_t take = min((uint64_t)(64 - bn), plen);
        for (uint64_t i = 0; i < take; ++i) buf[bn + i] = bytes[i];
        bn += (uint32_t)take;
        pos = take;
        if (bn == 64) {
            compress_bytes(H, buf);
            bn = 0;
        }
    }
    if (bn == 0) {
        for (; pos + 64 <= plen; pos += 64) {  // full blocks straight from the piece
            uint32_t W[16];
            load_block(bytes, pos, W);
            compress(H, W);
        }
        for (; pos < plen; ++pos) buf[bn++] = bytes[pos];
    }
    const uint64_t total = open_len + plen;
    if (finish) {  // FIPS 180-4 5.1.1 padding with the chunk's total length
        buf[bn++] = 0x80;
        if (bn > 56) {
            while (bn < 64) buf[bn++] = 0;
            compress_bytes(H, buf);
            bn = 0;
        }
        while (bn < 56) buf[bn++] = 0;
        const uint64_t bits = total * 8;
        for (int k = 0; k < 8; ++k) buf[56 + k] = (uint8_t)(bits >> (56 - 8 * k));
        compress_bytes(H, buf);
        for (int i = 0; i < 5; ++i) {
            digest[4 * i] = (uint8_t)(H[i] >> 24);
            digest[4 * i + 1] = (uint8_t)(H[i] >> 16);
            digest[4 * i + 2] = (uint8_t)(H[i] >> 8);
            digest[4 * i + 3] = (uint8_t)H[i];
        }
        extra[0] = (uint32_t)open_len;  // bytes of chunk 0 in earlier pieces
        extra[1] = (uint32_t)(open_len >> 32);
    } else {
#pragma unroll
        for (int i = 0; i < 5; ++i) out.H[i] = H[i];
        out.open_len = total;
        out.left_n = bn;
        for (uint32_t i = 0; i < bn; ++i) out.left[i] = buf[i];
    }
}

}  // namespace

void launch_carry_hist(const BatchDesc* d, cudaStream_t s) {
    carry_hist_kernel<<<1, 32, 0, s>>>(d);
}

void launch_carry_meta(const BatchDesc* d, const uint32_t* n_cuts, const uint32_t* cut_pos,
                       uint64_t cap, uint32_t* m_out, uint32_t* chunk_start, uint64_t* chunk_id,
                       uint32_t* item_first, uint32_t* extra, cudaStream_t s) {
    carry_meta_kernel<<<8, 256, 0, s>>>(d, n_cuts, cut_pos, cap, m_out, chunk_start, chunk_id,
                                        item_first, extra);
}

void launch_carry_cont(const BatchDesc* d, const uint32_t* n_cuts, const uint32_t* cut_pos,
                       uint64_t cap, uint8_t* digest, uint32_t* extra, cudaStream_t s) {
    carry_cont_kernel<<<1, 32, 0, s>>>(d, n_cuts, cut_pos, cap, digest, extra);
}

}  // namespace dd
