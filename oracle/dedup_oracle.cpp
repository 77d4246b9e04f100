// ============================================================================
// dedup_oracle.cpp -- TEST INFRASTRUCTURE ONLY.
//
// A plain, slow, sequential CPU oracle for the GPU Dedup hot path of
// Rockenbach et al., "Stream Processing on Multi-Cores with GPUs: Parallel
// Programming Models' Challenges" (IPDPSW 2019).  Citations "P:NNN" are
// lines of /root/reference/PAPER.md (Section IV-B "Dedup").
//
// Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
// --impl reference legs may load this library.  It shares no code, headers,
// tables or constants generator with the CUDA path
// (paper_conf_ipps_rockenbachsgmtd19_b200/csrc); neither includes the other.
//
// What it computes:
//   1. Rabin fingerprint of a 32-byte window: fp(w) = (sum_k w[k] t^{8(31-k)})
//      mod P(t), P(t) = t^32 + poly over GF(2)        ("rabin fingerprint";
//      readings O1-O5 in DESIGN.md).  Two forms are here: the plain Horner
//      definition (oracle_fp_window) and the rolling recurrence the chunker
//      uses (PARSEC rabinseg style); tests pin one against the other and both
//      against a Python long division.
//   2. Chunking of one item (= one fixed-size batch of P:197 / P:213):
//      restart-based greedy cut selection, chunk starts = the paper's startPos
//      (Fig. 2).
//   3. SHA-1 (FIPS 180-4) of every chunk.
//   4. Global duplicate check in stream order (reading O11/O12):
//      std::unordered_map digest -> first id, id = (seq << 32) | chunk index.
//   5. Output per item in seq order.
// ============================================================================
#include <atomic>
#include <chrono>
#include <cstdint>
#include <cstring>
#include <string>
#include <thread>
#include <unordered_map>
#include <vector>

extern "C" {

// ----------------------------------------------------------------------------
// GF(2) polynomial helpers.  A 32-bit word x holds a polynomial of degree < 32
// (bit j = coefficient of t^j).  P(t) = t^32 + poly, so t^32 == poly (mod P).
// ----------------------------------------------------------------------------
static uint32_t gf_mul_t(uint32_t x, uint32_t poly) {
    // x * t mod P: shift left by one; the t^32 term that falls out is replaced
    // by poly.
    uint32_t carry = x >> 31;
    x <<= 1;
    if (carry) x ^= poly;
    return x;
}

static uint32_t gf_mul_tk(uint32_t x, unsigned k, uint32_t poly) {
    for (unsigned i = 0; i < k; ++i) x = gf_mul_t(x, poly);
    return x;
}

// Plain definition: Horner over bits, MSB of the first
// byte is the highest-degree coefficient (reading O4).
uint32_t oracle_fp_window(const uint8_t* w, uint32_t len, uint32_t poly) {
    uint32_t h = 0;
    for (uint32_t k = 0; k < len; ++k) {
        for (int bit = 7; bit >= 0; --bit) {
            h = gf_mul_t(h, poly) ^ ((w[k] >> bit) & 1u);
        }
    }
    return h;
}

// Rolling-hash tables: R[b] = b t^32 mod P (reduction of the
// byte shifted out of the top), Wt[b] = b t^{8(window-1)} mod P (contribution
// of the byte leaving the window).
void oracle_rabin_tables(uint32_t poly, uint32_t window, uint32_t* R, uint32_t* Wt) {
    for (uint32_t b = 0; b < 256; ++b) {
        R[b] = gf_mul_tk(b, 32, poly);
        Wt[b] = gf_mul_tk(b, 8 * (window - 1), poly);
    }
}

typedef struct {
    uint32_t window;        // 32 (reading O2)
    uint32_t poly;          // 0x45c2b6a1 (reading O1)
    uint32_t anchor_mask;   // 0xFFF (reading O3)
    uint32_t anchor_value;  // 0
    uint32_t min_chunk;     // >= window; 32 (reading O6)
    uint32_t max_chunk;     // 0 = none (reading O7)
    uint32_t literal_window;  // 1: PARSEC's rabininit(rf_win = 0) table (reading O5-L)
} oracle_params;

// Fingerprint of the window ending at every byte i (inclusive) of p, with the
// hash started fresh at byte 0 (no subtraction during the first `window`
// bytes).  out[i] = fp(p[i-window+1 .. i]) for i >= window-1.
void oracle_rolling_fp(const uint8_t* p, uint64_t n, uint32_t poly, uint32_t window,
                       uint32_t* out) {
    uint32_t R[256], Wt[256];
    oracle_rabin_tables(poly, window, R, Wt);
    uint32_t h = 0;
    for (uint64_t i = 0; i < n; ++i) {
        if (i >= window) h ^= Wt[p[i - window]];  // byte leaves the window
        uint32_t x = h >> 24;
        h = (h << 8) | p[i];                        // byte enters
        h ^= R[x];                                  // reduce the t^32.. overflow
        out[i] = h;
    }
}

// Chunk one item p[0..n) ("saved all the indexes
// where the algorithm would fragment the data"; P:199 startPos).
//   c = 0; while c < n: emit c; restart the hash at c; the cut is the smallest
//   e in [c+min_chunk, n) with (fp(p[e-window..e-1]) & mask) == value, or the
//   forced cut e = c+max_chunk (max_chunk != 0, e < n); else e = n.
// Returns the number of chunks; starts[] receives item-relative chunk starts.
//
// literal_window (row NEXT-2, reading O5-L): PARSEC's chunker as
// called with a window-table length of 0, rabinwintab[x] = x * t^0 = x: the
// byte leaving the window is XORed in at degree 0 instead of removed, so the
// hash at a position depends on every byte since the last cut (restart).
uint64_t oracle_chunk_item(const uint8_t* p, uint64_t n, const oracle_params* prm,
                           uint32_t* starts, uint64_t cap) {
    uint32_t R[256], Wt[256];
    oracle_rabin_tables(prm->poly, prm->window, R, Wt);
    if (prm->literal_window)
        for (uint32_t b = 0; b < 256; ++b) Wt[b] = b;
    const uint32_t W = prm->window;
    uint64_t count = 0;
    uint64_t c = 0;
    while (c < n) {
        if (count < cap) starts[count] = (uint32_t)c;
        ++count;
        uint64_t e = n;
        uint32_t h = 0;  // restart (PARSEC rabinseg re-run after each cut)
        for (uint64_t i = c; i < n; ++i) {
            if (i - c >= W) h ^= Wt[p[i - W]];
            uint32_t x = h >> 24;
            h = (h << 8) | p[i];
            h ^= R[x];
            uint64_t cut = i + 1;  // candidate cut position after byte i
            if (cut >= n) break;
            uint64_t len = cut - c;
            if (prm->max_chunk != 0 && len >= prm->max_chunk) { e = cut; break; }
            if (len >= prm->min_chunk && len >= W &&
                (h & prm->anchor_mask) == prm->anchor_value) {
                e = cut;
                break;
            }
        }
        c = e;
    }
    return count;
}

// ----------------------------------------------------------------------------
// SHA-1, FIPS 180-4 section 6.1, written out plainly.
// ----------------------------------------------------------------------------
static uint32_t rotl32(uint32_t x, unsigned s) { return (x << s) | (x >> (32 - s)); }

static void sha1_compress(uint32_t H[5], const uint8_t blk[64]) {
    uint32_t W[80];
    for (int t = 0; t < 16; ++t)
        W[t] = ((uint32_t)blk[4 * t] << 24) | ((uint32_t)blk[4 * t + 1] << 16) |
               ((uint32_t)blk[4 * t + 2] << 8) | (uint32_t)blk[4 * t + 3];
    for (int t = 16; t < 80; ++t) W[t] = rotl32(W[t - 3] ^ W[t - 8] ^ W[t - 14] ^ W[t - 16], 1);
    uint32_t a = H[0], b = H[1], c = H[2], d = H[3], e = H[4];
    for (int t = 0; t < 80; ++t) {
        uint32_t f, K;
        if (t < 20)      { f = (b & c) ^ (~b & d);          K = 0x5A827999u; }
        else if (t < 40) { f = b ^ c ^ d;                   K = 0x6ED9EBA1u; }
        else if (t < 60) { f = (b & c) ^ (b & d) ^ (c & d); K = 0x8F1BBCDCu; }
        else             { f = b ^ c ^ d;                   K = 0xCA62C1D6u; }
        uint32_t T = rotl32(a, 5) + f + e + K + W[t];
        e = d; d = c; c = rotl32(b, 30); b = a; a = T;
    }
    H[0] += a; H[1] += b; H[2] += c; H[3] += d; H[4] += e;
}

void oracle_sha1(const uint8_t* msg, uint64_t len, uint8_t out[20]) {
    uint32_t H[5] = {0x67452301u, 0xEFCDAB89u, 0x98BADCFEu, 0x10325476u, 0xC3D2E1F0u};
    uint64_t full = len / 64;
    for (uint64_t i = 0; i < full; ++i) sha1_compress(H, msg + 64 * i);
    // Padding (FIPS 180-4 5.1.1): 0x80, zeros, 64-bit big-endian bit length.
    uint8_t tail[128];
    std::memset(tail, 0, sizeof(tail));
    uint64_t rem = len - 64 * full;
    std::memcpy(tail, msg + 64 * full, rem);
    tail[rem] = 0x80;
    uint64_t tail_len = (rem + 9 <= 64) ? 64 : 128;
    uint64_t bits = len * 8;
    for (int k = 0; k < 8; ++k) tail[tail_len - 1 - k] = (uint8_t)(bits >> (8 * k));
    sha1_compress(H, tail);
    if (tail_len == 128) sha1_compress(H, tail + 64);
    for (int k = 0; k < 5; ++k) {
        out[4 * k] = (uint8_t)(H[k] >> 24);
        out[4 * k + 1] = (uint8_t)(H[k] >> 16);
        out[4 * k + 2] = (uint8_t)(H[k] >> 8);
        out[4 * k + 3] = (uint8_t)H[k];
    }
}

// ----------------------------------------------------------------------------
// Stream dedup (P:215 duplicate check, P:217 reorder).
// A context carries the global digest table across calls so that a stream can
// be fed item by item or in arbitrary groups.
// ----------------------------------------------------------------------------
struct oracle_ctx {
    oracle_params prm;
    std::unordered_map<std::string, uint64_t> table;  // digest -> first id
    uint64_t chunks = 0, dup_chunks = 0, dup_bytes = 0, bytes = 0, items = 0;
};

oracle_ctx* oracle_ctx_new(const oracle_params* prm) {
    oracle_ctx* c = new oracle_ctx();
    c->prm = *prm;
    return c;
}

void oracle_ctx_free(oracle_ctx* c) { delete c; }

// Process one item with sequence number `seq`.  Output arrays must hold at
// least oracle_max_chunks(len) entries.  Returns the number of chunks.
uint64_t oracle_ctx_item(oracle_ctx* c, uint64_t seq, const uint8_t* p, uint64_t n,
                         uint32_t* chunk_start, uint8_t* digest, uint8_t* is_dup,
                         uint64_t* first_id, uint64_t cap) {
    uint64_t k = oracle_chunk_item(p, n, &c->prm, chunk_start, cap);
    if (k > cap) return k;  // caller under-allocated; nothing else written
    for (uint64_t j = 0; j < k; ++j) {
        uint64_t s = chunk_start[j];
        uint64_t e = (j + 1 < k) ? chunk_start[j + 1] : n;
        uint8_t* d = digest + 20 * j;
        oracle_sha1(p + s, e - s, d);
        std::string key((const char*)d, 20);
        uint64_t id = (seq << 32) | j;
        auto it = c->table.find(key);
        if (it != c->table.end()) {
            is_dup[j] = 1;
            first_id[j] = it->second;
            c->dup_chunks++;
            c->dup_bytes += e - s;
        } else {
            c->table.emplace(key, id);
            is_dup[j] = 0;
            first_id[j] = id;
        }
    }
    c->chunks += k;
    c->bytes += n;
    c->items += 1;
    return k;
}

void oracle_ctx_counts(const oracle_ctx* c, uint64_t out[5]) {
    out[0] = c->items;
    out[1] = c->bytes;
    out[2] = c->chunks;
    out[3] = c->dup_chunks;
    out[4] = c->dup_bytes;
}

uint64_t oracle_max_chunks(uint64_t n, uint32_t min_chunk) {
    if (n == 0) return 0;
    uint32_t m = min_chunk ? min_chunk : 1;
    return n / m + 1;
}

// ----------------------------------------------------------------------------
// Threaded variant: steps 2-3 (chunking + SHA-1) of the
// items of one buffer spread over T host threads -- items are independent --
// then step 4 (the dedup table) sequentially in stream order, with exactly
// the functions above.  Used for the CPU baseline on all host cores and to
// run the oracle over the full-size configurations in the tests.
// ----------------------------------------------------------------------------
struct oracle_batch {
    std::vector<uint64_t> item_first;  // [n_items + 1] chunk offsets
    std::vector<uint32_t> chunk_start;
    std::vector<uint8_t> digest;
    std::vector<uint8_t> is_dup;
    std::vector<uint64_t> first_id;
    double s_chunk_sha = 0, s_dedup = 0;  // wall seconds of the two phases
};

// buf[item_off[k] .. item_off[k+1]) is item k (seq = seq0 + k).  Returns a
// result handle (free with oracle_batch_free); the dedup state continues the
// stream of ctx.
oracle_batch* oracle_ctx_items_parallel(oracle_ctx* c, uint64_t seq0, const uint8_t* buf,
                                        const uint64_t* item_off, uint64_t n_items,
                                        uint32_t threads) {
    auto* r = new oracle_batch();
    const auto t0 = std::chrono::steady_clock::now();
    std::vector<std::vector<uint32_t>> starts(n_items);
    std::vector<std::vector<uint8_t>> digs(n_items);
    std::atomic<uint64_t> next{0};
    auto work = [&]() {
        for (uint64_t k; (k = next.fetch_add(1)) < n_items;) {
            const uint8_t* p = buf + item_off[k];
            const uint64_t n = item_off[k + 1] - item_off[k];
            std::vector<uint32_t>& s = starts[k];
            s.resize(oracle_max_chunks(n, c->prm.min_chunk));
            s.resize(oracle_chunk_item(p, n, &c->prm, s.data(), s.size()));
            digs[k].resize(20 * s.size());
            for (uint64_t j = 0; j < s.size(); ++j) {
                const uint64_t e = j + 1 < s.size() ? s[j + 1] : n;
                oracle_sha1(p + s[j], e - s[j], digs[k].data() + 20 * j);
            }
        }
    };
    if (threads < 1) threads = 1;
    std::vector<std::thread> pool;
    for (uint32_t t = 1; t < threads; ++t) pool.emplace_back(work);
    work();
    for (auto& t : pool) t.join();
    const auto t1 = std::chrono::steady_clock::now();
    r->item_first.resize(n_items + 1, 0);
    for (uint64_t k = 0; k < n_items; ++k)
        r->item_first[k + 1] = r->item_first[k] + starts[k].size();
    const uint64_t total = r->item_first[n_items];
    r->chunk_start.resize(total);
    r->digest.resize(20 * total);
    r->is_dup.resize(total);
    r->first_id.resize(total);
    for (uint64_t k = 0; k < n_items; ++k) {  // step 4, sequential, stream order
        const uint64_t f = r->item_first[k], n = item_off[k + 1] - item_off[k];
        const std::vector<uint32_t>& s = starts[k];
        for (uint64_t j = 0; j < s.size(); ++j) {
            const uint64_t e = j + 1 < s.size() ? s[j + 1] : n;
            const uint8_t* d = digs[k].data() + 20 * j;
            r->chunk_start[f + j] = s[j];
            std::memcpy(r->digest.data() + 20 * (f + j), d, 20);
            std::string key((const char*)d, 20);
            const uint64_t id = ((seq0 + k) << 32) | j;
            auto it = c->table.find(key);
            if (it != c->table.end()) {
                r->is_dup[f + j] = 1;
                r->first_id[f + j] = it->second;
                c->dup_chunks++;
                c->dup_bytes += e - s[j];
            } else {
                c->table.emplace(key, id);
                r->is_dup[f + j] = 0;
                r->first_id[f + j] = id;
            }
        }
        c->chunks += s.size();
        c->bytes += n;
        c->items += 1;
    }
    const auto t2 = std::chrono::steady_clock::now();
    r->s_chunk_sha = std::chrono::duration<double>(t1 - t0).count();
    r->s_dedup = std::chrono::duration<double>(t2 - t1).count();
    return r;
}

uint64_t oracle_batch_chunks(const oracle_batch* r) { return r->chunk_start.size(); }

void oracle_batch_times(const oracle_batch* r, double out[2]) {
    out[0] = r->s_chunk_sha;
    out[1] = r->s_dedup;
}

// Copies the results out: item_first[n_items + 1], then per chunk.
void oracle_batch_fetch(const oracle_batch* r, uint64_t* item_first, uint32_t* chunk_start,
                        uint8_t* digest, uint8_t* is_dup, uint64_t* first_id) {
    std::memcpy(item_first, r->item_first.data(), 8 * r->item_first.size());
    const uint64_t n = r->chunk_start.size();
    std::memcpy(chunk_start, r->chunk_start.data(), 4 * n);
    std::memcpy(digest, r->digest.data(), 20 * n);
    std::memcpy(is_dup, r->is_dup.data(), n);
    std::memcpy(first_id, r->first_id.data(), 8 * n);
}

void oracle_batch_free(oracle_batch* r) { delete r; }

}  // extern "C"
