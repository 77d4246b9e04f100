// rabin.cu -- rows A2 (Rabin candidate scan) and A3 (cut selection +
// compaction) of the hot path.  PAPER.md P:197 (Rabin fingerprint
// fragmentation of fixed batches, "saved all the indexes where the algorithm
// would fragment the data"), P:199 / Fig. 2 (startPos).
//
// The paper ran this on the CPU; here it is two sm_100a kernels:
//
//  rabin_scan_kernel   every lane owns a contiguous segment of the batch,
//                      re-derives the 32-byte window hash over the 32 bytes
//                      before its segment (warm-up), then rolls byte by byte
//                      with the post-shift recurrence
//                        h' = ((h << 8) | in) ^ R[h >> 24] ^ W256[out]
//                      and emits one candidate bit per byte.  Both tables are
//                      replicated per lane in shared memory ([x][lane] layout,
//                      bank = lane, conflict-free), addressed with one PRMT.
//  select_*_kernel     greedy cut selection.  With min chunk = window = 32 the
//                      only state crossing a position is "positions still
//                      blocked" in [0, 31]; a warp simulates all 32 entry
//                      states of an 8192-position tile (lane s = state s) and
//                      stores the tile's 32-entry transfer function (agg); one
//                      CTA composes the functions in tile order with warp
//                      shuffles (prefix over an associative operator) giving
//                      every tile its real entry state and cut offset; a
//                      replay pass writes the cut positions.  Item starts are
//                      forced cuts and reset the state.
#include <cuda_runtime.h>
#include <stdint.h>

#include "internal.h"

namespace dd {

namespace {

constexpr int kScanThreads = 512;
constexpr int kTabBytes = 256 * 256;  // [x][R|W][lane] u32 = 64 KiB

// Rolls the 32 bytes of cur[0..7] (stream bytes, little-endian words) into h,
// removing the 32 bytes of old[0..7]; returns the 32 candidate bits.
__device__ __forceinline__ uint32_t roll32(uint32_t& h, const uint32_t cur[8],
                                           const uint32_t old[8], const uint8_t* tab,
                                           uint32_t laneoff, uint32_t mask, uint32_t value) {
    uint32_t bits = 0;
#pragma unroll
    for (int w = 0; w < 8; ++w) {
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            // R[x] at x*256 + lane*4, W256[o] at o*256 + 128 + lane*4.
            uint32_t aR = __byte_perm(h, laneoff, 0x6534);
            uint32_t aW = __byte_perm(old[w], laneoff, 0x6504 | (k << 4));
            uint32_t hs = __byte_perm(cur[w], h, 0x6540 | k);  // (h << 8) | in
            uint32_t r = *reinterpret_cast<const uint32_t*>(tab + aR);
            uint32_t o = *reinterpret_cast<const uint32_t*>(tab + 128 + aW);
            h = hs ^ r ^ o;
            bits |= ((h & mask) == value ? 1u : 0u) << (4 * w + k);
        }
    }
    return bits;
}

__device__ __forceinline__ void load32(const uint8_t* p, uint32_t v[8]) {
    uint4 a = __ldg(reinterpret_cast<const uint4*>(p));
    uint4 b = __ldg(reinterpret_cast<const uint4*>(p + 16));
    v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w;
    v[4] = b.x; v[5] = b.y; v[6] = b.z; v[7] = b.w;
}

// Guarded version: 16-byte vectors at or beyond lim16 (nbytes rounded up to
// 16) read as zero.
__device__ __forceinline__ void load32_guard(const uint8_t* base, uint64_t off, uint64_t lim16,
                                             uint32_t v[8]) {
    uint4 a = make_uint4(0, 0, 0, 0), b = make_uint4(0, 0, 0, 0);
    if (off < lim16) a = __ldg(reinterpret_cast<const uint4*>(base + off));
    if (off + 16 < lim16) b = __ldg(reinterpret_cast<const uint4*>(base + off + 16));
    v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w;
    v[4] = b.x; v[5] = b.y; v[6] = b.z; v[7] = b.w;
}

__global__ void __launch_bounds__(kScanThreads, 2)
rabin_scan_kernel(const BatchDesc* __restrict__ desc, const uint32_t* __restrict__ gtab,
                  uint32_t mask, uint32_t value, uint32_t* __restrict__ bitmap) {
    const uint8_t* __restrict__ bytes = desc->bytes;
    const uint64_t nbytes = desc->nbytes;
    if (nbytes == 0) return;
    // Segment per lane: long enough that the 32-byte warm-up is cheap, short
    // enough that the grid's lanes cover the batch in one pass.
    const uint64_t threads = (uint64_t)gridDim.x * blockDim.x;
    uint64_t seg = (nbytes + threads - 1) / threads;
    seg = ((seg + 31) / 32) * 32;
    if (seg < 256) seg = 256;
    const uint64_t n_lanes = (nbytes + seg - 1) / seg;
    extern __shared__ __align__(16) uint8_t tab[];
    {
        uint32_t* t32 = reinterpret_cast<uint32_t*>(tab);
        for (int idx = threadIdx.x; idx < kTabBytes / 4; idx += blockDim.x) {
            int x = idx >> 6, half = (idx >> 5) & 1;
            t32[idx] = gtab[half * 256 + x];
        }
    }
    __syncthreads();
    const uint32_t laneoff = (threadIdx.x & 31) * 4;
    const uint64_t lim16 = (nbytes + 15) & ~uint64_t(15);
    for (uint64_t L = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; L < n_lanes;
         L += (uint64_t)gridDim.x * blockDim.x) {
        const uint64_t q = L * seg;
        const uint64_t end = min(q + seg, nbytes);
        uint32_t h = 0;
        uint32_t prev[8] = {0, 0, 0, 0, 0, 0, 0, 0};
        if (q >= 32) {  // warm-up: hash of the window ending at q-1
            uint32_t w[8];
            load32(bytes + q - 32, w);
            (void)roll32(h, w, prev, tab, laneoff, mask, value);
#pragma unroll
            for (int i = 0; i < 8; ++i) prev[i] = w[i];
        }
        uint32_t cur[8];
        if (q + 32 <= nbytes) load32(bytes + q, cur);
        else load32_guard(bytes, q, lim16, cur);
        for (uint64_t base = q; base < end; base += 32) {
            uint32_t nxt[8];
            const uint64_t nb = base + 32;
            if (nb < end) {  // prefetch the next 32 bytes
                if (nb + 32 <= nbytes) load32(bytes + nb, nxt);
                else load32_guard(bytes, nb, lim16, nxt);
            }
            uint32_t bits = roll32(h, cur, prev, tab, laneoff, mask, value);
            if (base + 32 > nbytes) bits &= (1u << (uint32_t)(nbytes - base)) - 1u;
            bitmap[base >> 5] = bits;
#pragma unroll
            for (int i = 0; i < 8; ++i) { prev[i] = cur[i]; cur[i] = nxt[i]; }
        }
    }
}

// ---------------------------------------------------------------------------
// Cut selection.
// ---------------------------------------------------------------------------
constexpr int kSelWarps = 4;
constexpr uint32_t kInf = 0xFFFFFFFFu;

struct SelWarpSmem {
    uint32_t cand[kSelTileWords];
    uint32_t forced[kSelTileWords];
    uint32_t csum[8];
    uint32_t fsum[8];
};

// First set bit at tile-relative position >= from, or kInf.
__device__ __forceinline__ uint32_t next_set(const uint32_t* words, const uint32_t* summary,
                                             uint32_t from) {
    if (from >= kSelTile) return kInf;
    uint32_t w = from >> 5;
    uint32_t b = words[w] & (0xFFFFFFFFu << (from & 31));
    if (b) return (w << 5) + (__ffs(b) - 1);
    uint32_t sw = w + 1;
    if (sw >= kSelTileWords) return kInf;
    uint32_t si = sw >> 5;
    uint32_t sb = summary[si] & (0xFFFFFFFFu << (sw & 31));
    while (!sb) {
        if (++si >= kSelTileWords / 32) return kInf;
        sb = summary[si];
    }
    uint32_t ww = (si << 5) + (__ffs(sb) - 1);
    return (ww << 5) + (__ffs(words[ww]) - 1);
}

// Greedy walk over one tile from entry state s: returns the cut count and the
// exit state; if out != nullptr also writes the cut positions.
__device__ __forceinline__ uint32_t walk_tile(const SelWarpSmem& sm, uint32_t s,
                                              uint32_t& exit_state, uint32_t* out,
                                              uint64_t out_base, uint64_t cap, uint64_t T0) {
    uint32_t E = s, cur = 0, cnt = 0;
    while (true) {
        uint32_t f = next_set(sm.forced, sm.fsum, cur);
        uint32_t c = next_set(sm.cand, sm.csum, max(E, cur));
        uint32_t e = min(f, c);
        if (e == kInf) break;
        if (out != nullptr && out_base + cnt < cap) out[out_base + cnt] = (uint32_t)(T0 + e);
        ++cnt;
        E = e + 32;
        cur = e + 1;
    }
    exit_state = E > kSelTile ? E - kSelTile : 0;
    return cnt;
}

constexpr uint32_t kM27 = (1u << 27) - 1;

// Candidate (e-space: cut after byte i <=> e = i + 1) and forced-cut bits of
// tile t into the warp's shared memory, with one-bit-per-word summaries.
__device__ __forceinline__ void build_tile(SelWarpSmem& sm, uint64_t t,
                                           const uint32_t* __restrict__ bitmap, uint64_t nbytes,
                                           const uint64_t* __restrict__ item_off,
                                           uint32_t n_items, int lane) {
    const uint64_t T0 = t * kSelTile;
    const uint64_t n_words = (nbytes + 31) / 32;
    uint32_t cw[8], fw[8];
    const uint64_t E0 = T0 + (uint64_t)lane * 256;  // this lane's e-range
#pragma unroll
    for (int j = 0; j < 8; ++j) {
        const uint64_t g = T0 / 32 + lane * 8 + j;
        const uint32_t curw = g < n_words ? bitmap[g] : 0u;
        const uint32_t prvw = (g >= 1 && g - 1 < n_words) ? bitmap[g - 1] : 0u;
        uint32_t ew = __funnelshift_l(prvw, curw, 1);
        const uint64_t e_lo = E0 + 32 * j;
        if (e_lo >= nbytes) ew = 0;
        else if (e_lo + 32 > nbytes) ew &= (1u << (uint32_t)(nbytes - e_lo)) - 1u;
        cw[j] = ew;
        fw[j] = 0;
    }
    // items: no candidate at e in [q, q+32) (window would leave the item),
    // forced cut at q for non-empty items
    if (E0 < nbytes && n_items > 0) {
        const uint64_t key = E0 >= 31 ? E0 - 31 : 0;  // first start > E0 - 32
        uint32_t lo = 0, hi = n_items;
        while (lo < hi) {
            const uint32_t mid = (lo + hi) >> 1;
            if (item_off[mid] < key) lo = mid + 1; else hi = mid;
        }
        for (uint32_t it = lo; it < n_items; ++it) {
            const uint64_t q = item_off[it];
            if (q >= E0 + 256) break;
            const bool nonempty = item_off[it + 1] > q;
#pragma unroll
            for (int j = 0; j < 8; ++j) {
                const int64_t a = (int64_t)q - (int64_t)(E0 + 32 * j);
                if (a < 32 && a > -32) {
                    const uint32_t lo_r = a > 0 ? (uint32_t)a : 0u;
                    const uint32_t hi_r = a < 0 ? (uint32_t)(a + 32) : 32u;
                    const uint32_t hm = hi_r >= 32 ? 0xFFFFFFFFu : ((1u << hi_r) - 1u);
                    cw[j] &= ~(hm & ~((1u << lo_r) - 1u));
                    if (nonempty && a >= 0) fw[j] |= 1u << (uint32_t)a;
                }
            }
        }
    }
    uint32_t cm = 0, fm = 0;
#pragma unroll
    for (int j = 0; j < 8; ++j) {
        sm.cand[lane * 8 + j] = cw[j];
        sm.forced[lane * 8 + j] = fw[j];
        cm |= (cw[j] ? 1u : 0u) << j;
        fm |= (fw[j] ? 1u : 0u) << j;
    }
    reinterpret_cast<uint8_t*>(sm.csum)[lane] = (uint8_t)cm;
    reinterpret_cast<uint8_t*>(sm.fsum)[lane] = (uint8_t)fm;
    __syncwarp();
}

// Phase 1: the 32-entry transfer function of every tile:
// agg[32 t + s] = exit_state(s) << 27 | cuts(s).
__global__ void __launch_bounds__(kSelWarps * 32)
select_agg_kernel(const BatchDesc* __restrict__ desc, const uint32_t* __restrict__ bitmap,
                  uint32_t* __restrict__ agg) {
    __shared__ SelWarpSmem smem[kSelWarps];
    const int wid = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint64_t nbytes = desc->nbytes;
    const uint64_t n_tiles = (nbytes + kSelTile - 1) / kSelTile;
    for (uint64_t t = (uint64_t)blockIdx.x * kSelWarps + wid; t < n_tiles;
         t += (uint64_t)gridDim.x * kSelWarps) {
        build_tile(smem[wid], t, bitmap, nbytes, desc->item_off, desc->n_items, lane);
        uint32_t ex;
        const uint32_t cnt = walk_tile(smem[wid], lane, ex, nullptr, 0, 0, 0);
        agg[32 * t + lane] = (ex << 27) | cnt;
        __syncwarp();
    }
}

// Phase 2 (one CTA of 32 warps): prefix composition of the tile functions.
// tile_entry[2t] = entry state of tile t, tile_entry[2t+1] = cuts before it.
__global__ void __launch_bounds__(1024)
select_scan_kernel(const BatchDesc* __restrict__ desc, const uint32_t* __restrict__ agg,
                   uint32_t* __restrict__ tile_entry, uint32_t* __restrict__ n_chunks) {
    __shared__ uint32_t fs[32][32], fc[32][32], es[32], ec[32];
    const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint64_t n_tiles = (desc->nbytes + kSelTile - 1) / kSelTile;
    const uint64_t per = (n_tiles + 31) / 32;
    const uint64_t t0 = w * per, t1 = min(t0 + per, n_tiles);
    uint32_t Gs = lane, Gc = 0;  // composition of tiles [t0, t): entry lane -> (state, cuts)
#pragma unroll 4
    for (uint64_t t = t0; t < t1; ++t) {
        const uint32_t a = agg[32 * t + lane];
        const uint32_t ns = __shfl_sync(0xFFFFFFFFu, a >> 27, Gs);
        const uint32_t nc = Gc + __shfl_sync(0xFFFFFFFFu, a & kM27, Gs);
        Gs = ns;
        Gc = nc;
    }
    fs[w][lane] = Gs;
    fc[w][lane] = Gc;
    __syncthreads();
    if (threadIdx.x == 0) {
        uint32_t s = 0, c = 0;  // the batch starts with a forced cut: entry state 0
        for (int r = 0; r < 32; ++r) {
            es[r] = s;
            ec[r] = c;
            c += fc[r][s];
            s = fs[r][s];
        }
        *n_chunks = c;
    }
    __syncthreads();
    const uint32_t e_s = es[w], e_c = ec[w];
    Gs = lane;
    Gc = 0;
#pragma unroll 4
    for (uint64_t t = t0; t < t1; ++t) {
        const uint32_t a = agg[32 * t + lane];
        const uint32_t st = __shfl_sync(0xFFFFFFFFu, Gs, e_s);
        const uint32_t ct = __shfl_sync(0xFFFFFFFFu, Gc, e_s);
        if (lane == 0) {
            tile_entry[2 * t] = st;
            tile_entry[2 * t + 1] = e_c + ct;
        }
        const uint32_t ns = __shfl_sync(0xFFFFFFFFu, a >> 27, Gs);
        const uint32_t nc = Gc + __shfl_sync(0xFFFFFFFFu, a & kM27, Gs);
        Gs = ns;
        Gc = nc;
    }
}

// Phase 3: replay every tile from its real entry state, writing cut_pos.
__global__ void __launch_bounds__(kSelWarps * 32)
select_emit_kernel(const BatchDesc* __restrict__ desc, const uint32_t* __restrict__ bitmap,
                   const uint32_t* __restrict__ tile_entry, uint32_t* __restrict__ cut_pos,
                   uint64_t cap) {
    __shared__ SelWarpSmem smem[kSelWarps];
    const int wid = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint64_t nbytes = desc->nbytes;
    const uint64_t n_tiles = (nbytes + kSelTile - 1) / kSelTile;
    for (uint64_t t = (uint64_t)blockIdx.x * kSelWarps + wid; t < n_tiles;
         t += (uint64_t)gridDim.x * kSelWarps) {
        build_tile(smem[wid], t, bitmap, nbytes, desc->item_off, desc->n_items, lane);
        const uint32_t st = tile_entry[2 * t], base = tile_entry[2 * t + 1];
        if (lane == (int)st) {
            uint32_t ex;
            walk_tile(smem[wid], st, ex, cut_pos, base, cap, t * kSelTile);
        }
        __syncwarp();
    }
}

__global__ void chunk_meta_kernel(const BatchDesc* __restrict__ desc,
                                  const uint32_t* __restrict__ cut_pos,
                                  const uint32_t* __restrict__ n_chunks_p, uint64_t cap,
                                  uint32_t* __restrict__ chunk_start,
                                  uint64_t* __restrict__ chunk_id,
                                  uint32_t* __restrict__ item_first_chunk) {
    const uint64_t n = min((uint64_t)*n_chunks_p, cap);
    const uint64_t* __restrict__ item_off = desc->item_off;
    const uint32_t n_items = desc->n_items;
    const uint64_t first_seq = desc->first_seq;
    for (uint64_t k = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; k < n;
         k += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t e = cut_pos[k];
        // item = last index in [0, n_items) with item_off[item] <= e
        uint32_t lo = 0, hi = n_items;
        while (lo < hi) {
            uint32_t mid = (lo + hi) >> 1;
            if (item_off[mid] <= e) lo = mid + 1; else hi = mid;
        }
        const uint32_t item = lo - 1;
        const uint32_t q = (uint32_t)item_off[item];
        uint64_t first;
        if (q == e) {
            first = k;
            item_first_chunk[item] = (uint32_t)k;
        } else {  // first chunk index with cut_pos >= q
            uint64_t a = 0, b = k;
            while (a < b) {
                uint64_t mid = (a + b) >> 1;
                if (cut_pos[mid] < q) a = mid + 1; else b = mid;
            }
            first = a;
        }
        chunk_start[k] = e - q;
        chunk_id[k] = ((first_seq + item) << 32) | (k - first);
    }
}

}  // namespace

void launch_rabin_scan(const BatchDesc* d, const uint32_t* d_tab, uint32_t mask, uint32_t value,
                       uint32_t* bitmap, int num_sms, cudaStream_t s) {
    static bool attr_set = false;
    if (!attr_set) {
        cudaFuncSetAttribute(rabin_scan_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             kTabBytes);
        attr_set = true;
    }
    rabin_scan_kernel<<<(unsigned)(num_sms * 2), kScanThreads, kTabBytes, s>>>(d, d_tab, mask,
                                                                               value, bitmap);
}

void launch_select(const BatchDesc* d, const uint32_t* bitmap, uint32_t* agg,
                   uint32_t* tile_entry, uint64_t max_tiles, uint32_t* cut_pos, uint64_t cap,
                   uint32_t* n_chunks, int num_sms, cudaStream_t s) {
    uint64_t blocks = (max_tiles + kSelWarps - 1) / kSelWarps;
    const uint64_t max_blocks = (uint64_t)num_sms * 8;
    if (blocks > max_blocks) blocks = max_blocks;
    if (blocks < 1) blocks = 1;
    select_agg_kernel<<<(unsigned)blocks, kSelWarps * 32, 0, s>>>(d, bitmap, agg);
    select_scan_kernel<<<1, 1024, 0, s>>>(d, agg, tile_entry, n_chunks);
    select_emit_kernel<<<(unsigned)blocks, kSelWarps * 32, 0, s>>>(d, bitmap, tile_entry, cut_pos,
                                                                   cap);
}

void launch_chunk_meta(const BatchDesc* d, const uint32_t* cut_pos, const uint32_t* n_chunks,
                       uint64_t cap, uint32_t* chunk_start, uint64_t* chunk_id,
                       uint32_t* item_first_chunk, uint32_t max_items, int num_sms,
                       cudaStream_t s) {
    if (max_items) cudaMemsetAsync(item_first_chunk, 0xFF, sizeof(uint32_t) * max_items, s);
    uint64_t blocks = (cap + 255) / 256;
    const uint64_t max_blocks = (uint64_t)num_sms * 4;
    if (blocks > max_blocks) blocks = max_blocks;
    if (blocks < 1) blocks = 1;
    chunk_meta_kernel<<<(unsigned)blocks, 256, 0, s>>>(d, cut_pos, n_chunks, cap, chunk_start,
                                                       chunk_id, item_first_chunk);
}

}  // namespace dd
