// archive.cpp -- row NEXT-3 of SURVEY.md section 8(f): the CPU-side consumer
// of the GPU stages, i.e. the paper's Dedup stages 4-5 on the host: "In CPU,
// we used the result of the kernel function to run the compression on each
// block and generate the compressed data" and "it reorders
// the batches and writes it in the output".  Host code (no kernels):
// the GPU rows produce everything it reads -- chunk starts (A3), digests
// (A4), duplicate flags (A7/A8) and the LZSS matches (NEXT-1).
//
// Archive format (reading A1 in DESIGN.md; the paper prints none):
//   per chunk, in stream order:
//     'U' digest[20] u32 raw_len u32 tok_len tokens[tok_len]   unique chunk
//     'D' digest[20]                                          duplicate
//   tokens: groups of up to 8 tokens, each group preceded by a flag byte
//   (bit k set: token k is a literal byte; clear: a 2-byte match
//   (offset & 0xFFF) | ((length - 3) << 12), little-endian).  The encoder is
//   the classic greedy LZSS pass over FindMatch's output: at chunk position
//   i, a match of length >= 3 is emitted and i advances by its length, else
//   byte i is emitted as a literal.  The decoder recovers a match's source
//   c from the offset (c - bs) mod W and the chunk position (reading L2).
#include <cstdint>
#include <cstring>
#include <string>
#include <unordered_map>
#include <vector>

#include "dedup.h"

namespace {

constexpr uint32_t kMinMatch = 3;  // MAX_UNCODED + 1 (matches of <= 2 bytes are literals)

void put32(uint8_t* p, uint32_t v) { std::memcpy(p, &v, 4); }
uint32_t get32(const uint8_t* p) {
    uint32_t v;
    std::memcpy(&v, p, 4);
    return v;
}

// Greedy LZSS tokens of one chunk [0, n) into out (capacity cap); returns
// the token bytes or -1 if they do not fit.
int64_t encode_chunk(const uint8_t* p, uint32_t n, const uint8_t* mlen, const uint16_t* moff,
                     uint8_t* out, uint64_t cap) {
    uint64_t o = 0, flag_at = 0;
    int nt = 8;
    for (uint32_t i = 0; i < n;) {
        if (nt == 8) {  // new group
            if (o + 1 > cap) return -1;
            flag_at = o;
            out[o++] = 0;
            nt = 0;
        }
        const uint32_t L = mlen[i];
        if (L >= kMinMatch) {
            if (o + 2 > cap) return -1;
            const uint16_t t = (uint16_t)((moff[i] & 0xFFFu) | ((L - kMinMatch) << 12));
            out[o++] = (uint8_t)(t & 0xFF);
            out[o++] = (uint8_t)(t >> 8);
            i += L;
        } else {
            if (o + 1 > cap) return -1;
            out[flag_at] |= (uint8_t)(1u << nt);
            out[o++] = p[i];
            i += 1;
        }
        ++nt;
    }
    return (int64_t)o;
}

}  // namespace

struct dedup_archive_decoder {
    std::unordered_map<std::string, std::vector<uint8_t>> chunks;  // digest -> bytes
    uint32_t window = 4096;
    std::string err;
};

extern "C" {

int64_t dedup_archive_encode(const uint8_t* data, uint64_t nbytes, const uint32_t* starts,
                             uint32_t n_chunks, const uint8_t* digest, const uint8_t* is_dup,
                             const uint8_t* match_len, const uint16_t* match_off,
                             uint32_t window, uint32_t max_coded, uint8_t* out,
                             uint64_t out_cap) {
    if (window != 4096 || max_coded < kMinMatch || max_coded > kMinMatch + 15)
        return DEDUP_EINVAL;
    if (nbytes > 0 && (data == nullptr || starts == nullptr || n_chunks == 0 || starts[0] != 0))
        return DEDUP_EINVAL;
    uint64_t o = 0;
    for (uint32_t k = 0; k < n_chunks; ++k) {
        const uint64_t s = starts[k];
        const uint64_t e = k + 1 < n_chunks ? starts[k + 1] : nbytes;
        if (e <= s || e > nbytes) return DEDUP_EINVAL;
        const uint8_t* dg = digest + 20ull * k;
        if (is_dup[k]) {
            if (o + 21 > out_cap) return DEDUP_ENOMEM;
            out[o] = 'D';
            std::memcpy(out + o + 1, dg, 20);
            o += 21;
            continue;
        }
        if (o + 29 > out_cap) return DEDUP_ENOMEM;
        out[o] = 'U';
        std::memcpy(out + o + 1, dg, 20);
        put32(out + o + 21, (uint32_t)(e - s));
        const int64_t t = encode_chunk(data + s, (uint32_t)(e - s), match_len + s,
                                       match_off + s, out + o + 29, out_cap - o - 29);
        if (t < 0) return DEDUP_ENOMEM;
        put32(out + o + 25, (uint32_t)t);
        o += 29 + (uint64_t)t;
    }
    return (int64_t)o;
}

dedup_archive_decoder* dedup_archive_decoder_new(uint32_t window) {
    if (window != 4096) return nullptr;
    auto* d = new dedup_archive_decoder();
    d->window = window;
    return d;
}

void dedup_archive_decoder_free(dedup_archive_decoder* d) { delete d; }

int64_t dedup_archive_decode(dedup_archive_decoder* d, const uint8_t* in, uint64_t in_len,
                             uint8_t* out, uint64_t out_cap) {
    if (d == nullptr || (in_len && in == nullptr)) return DEDUP_EINVAL;
    const uint32_t W = d->window;
    uint64_t q = 0, o = 0;
    while (q < in_len) {
        const uint8_t tag = in[q];
        if (q + 21 > in_len) return DEDUP_EINVAL;
        std::string key(reinterpret_cast<const char*>(in + q + 1), 20);
        if (tag == 'D') {
            auto it = d->chunks.find(key);
            if (it == d->chunks.end()) return DEDUP_EINVAL;  // reference before its chunk
            if (o + it->second.size() > out_cap) return DEDUP_ENOMEM;
            std::memcpy(out + o, it->second.data(), it->second.size());
            o += it->second.size();
            q += 21;
            continue;
        }
        if (tag != 'U' || q + 29 > in_len) return DEDUP_EINVAL;
        const uint32_t n = get32(in + q + 21), tl = get32(in + q + 25);
        if (q + 29 + tl > in_len || o + n > out_cap) return DEDUP_EINVAL;
        const uint8_t* t = in + q + 29;
        uint8_t* blk = out + o;
        uint64_t a = 0;
        uint32_t i = 0;
        while (i < n) {
            if (a >= tl) return DEDUP_EINVAL;
            const uint8_t flags = t[a++];
            for (int k = 0; k < 8 && i < n; ++k) {
                if (flags & (1u << k)) {
                    if (a >= tl) return DEDUP_EINVAL;
                    blk[i++] = t[a++];
                } else {
                    if (a + 2 > tl) return DEDUP_EINVAL;
                    const uint32_t tok = t[a] | ((uint32_t)t[a + 1] << 8);
                    a += 2;
                    const uint32_t off = tok & 0xFFFu, L = (tok >> 12) + kMinMatch;
                    // the c in [i - W, i) with c mod W == off (reading L2)
                    const uint32_t back = (i - off) % W == 0 ? W : (i - off) % W;
                    if (back > i || L > back || i + L > n) return DEDUP_EINVAL;
                    std::memcpy(blk + i, blk + i - back, L);  // c + L <= i: no overlap
                    i += L;
                }
            }
        }
        d->chunks.emplace(std::move(key), std::vector<uint8_t>(blk, blk + n));
        o += n;
        q += 29 + tl;
    }
    return (int64_t)o;
}

}  // extern "C"
