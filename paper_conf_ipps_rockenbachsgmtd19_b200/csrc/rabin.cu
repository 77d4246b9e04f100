// rabin.cu -- rows A2 (Rabin candidate scan) and A3 (cut selection +
// compaction) of the hot path.  PAPER.md P:197 (Rabin fingerprint
// fragmentation of fixed batches, "saved all the indexes where the algorithm
// would fragment the data"), P:199 / Fig. 2 (startPos).
//
// The paper ran this on the CPU; here it is a set of sm_100a kernels:
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
//                      states of an 8192-position tile (lane s = state s)
//                      giving the tile's 32-entry transfer function; a CTA of
//                      32 warps composes its 32 tiles into a group function;
//                      one CTA composes the group functions in order (a prefix
//                      over an associative operator, warp shuffles); a replay
//                      pass walks every tile from its real entry state and
//                      writes the cut positions.  Item starts are forced cuts
//                      and reset the state.
#include <cuda_runtime.h>
#include <stdint.h>

#include "internal.h"

namespace dd {

namespace {

constexpr int kScanThreads = 512;
constexpr int kTabBytes = 256 * 256;  // [x][R|W][lane] u32 = 64 KiB
constexpr uint32_t kFull = 0xFFFFFFFFu;

// Rolls the 32 bytes of cur[0..7] (stream bytes, little-endian words) into h,
// removing the 32 bytes of old[0..7]; returns the 32 candidate bits.
template <bool kZeroValue>
__device__ __forceinline__ uint32_t roll32(uint32_t& h, const uint32_t cur[8],
                                           const uint32_t old[8], const uint8_t* tab,
                                           uint32_t laneoff, uint32_t mask, uint32_t value) {
    uint32_t bits = 0;
#pragma unroll
    for (int w = 0; w < 8; ++w) {
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            // R[x] at x*256 + lane*4, W256[o] at o*256 + 128 + lane*4.
            const uint32_t aR = __byte_perm(h, laneoff, 0x6534);
            const uint32_t aW = __byte_perm(old[w], laneoff, 0x6504 | (k << 4));
            const uint32_t hs = __byte_perm(cur[w], h, 0x6540 | k);  // (h << 8) | in
            const uint32_t r = *reinterpret_cast<const uint32_t*>(tab + aR);
            const uint32_t o = *reinterpret_cast<const uint32_t*>(tab + 128 + aW);
            h = hs ^ r ^ o;
            const bool hit = kZeroValue ? (h & mask) == 0 : (h & mask) == value;
            if (hit) bits |= 1u << (4 * w + k);
        }
    }
    return bits;
}

__device__ __forceinline__ void load32(const uint8_t* p, uint32_t v[8]) {
    const uint4 a = __ldg(reinterpret_cast<const uint4*>(p));
    const uint4 b = __ldg(reinterpret_cast<const uint4*>(p + 16));
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

__device__ __forceinline__ void load32_any(const uint8_t* base, uint64_t off, uint64_t nbytes,
                                           uint64_t lim16, uint32_t v[8]) {
    if (off + 32 <= nbytes) load32(base + off, v);
    else load32_guard(base, off, lim16, v);
}

template <bool kZeroValue>
__global__ void __launch_bounds__(kScanThreads, 2)
rabin_scan_kernel(const BatchDesc* __restrict__ desc, const uint32_t* __restrict__ gtab,
                  uint32_t mask, uint32_t value, uint32_t* __restrict__ bitmap) {
    extern __shared__ __align__(16) uint8_t tab[];
    __shared__ uint32_t src[512];
    const uint8_t* __restrict__ bytes = desc->bytes;
    const uint64_t nbytes = desc->nbytes;
    if (threadIdx.x < 512) src[threadIdx.x] = gtab[threadIdx.x];
    __syncthreads();
    {   // replicate R / W256 per lane: word idx = x*64 + half*32 + lane
        uint32_t* t32 = reinterpret_cast<uint32_t*>(tab);
        for (int idx = threadIdx.x; idx < kTabBytes / 4; idx += blockDim.x)
            t32[idx] = src[((idx >> 5) & 1) * 256 + (idx >> 6)];
    }
    __syncthreads();
    if (nbytes == 0) return;
    // Segment per lane: long enough that the 32-byte warm-up is cheap, short
    // enough that the grid's lanes cover the batch in one pass.
    const uint64_t threads = (uint64_t)gridDim.x * blockDim.x;
    uint64_t seg = (nbytes + threads - 1) / threads;
    seg = ((seg + 31) / 32) * 32;
    if (seg < 256) seg = 256;
    const uint64_t n_lanes = (nbytes + seg - 1) / seg;
    const uint32_t laneoff = (threadIdx.x & 31) * 4;
    const uint64_t lim16 = (nbytes + 15) & ~uint64_t(15);
    for (uint64_t L = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; L < n_lanes;
         L += threads) {
        const uint64_t q = L * seg;
        const uint64_t end = min(q + seg, nbytes);
        uint32_t h = 0;
        uint32_t prev[8] = {0, 0, 0, 0, 0, 0, 0, 0};
        uint32_t cur[8];
        // issue the warm-up and the first step's loads together
        if (q >= 32) load32(bytes + q - 32, prev);
        load32_any(bytes, q, nbytes, lim16, cur);
        if (q >= 32) {  // warm-up: hash of the window ending at q-1
            const uint32_t zero[8] = {0, 0, 0, 0, 0, 0, 0, 0};
            (void)roll32<kZeroValue>(h, prev, zero, tab, laneoff, mask, value);
        }
        for (uint64_t base = q; base < end; base += 32) {
            uint32_t nxt[8];
            const uint64_t nb = base + 32;
            if (nb < end) load32_any(bytes, nb, nbytes, lim16, nxt);  // prefetch
            uint32_t bits = roll32<kZeroValue>(h, cur, prev, tab, laneoff, mask, value);
            if (base + 32 > nbytes) bits &= (1u << (uint32_t)(nbytes - base)) - 1u;
            bitmap[base >> 5] = bits;
#pragma unroll
            for (int i = 0; i < 8; ++i) {
                prev[i] = cur[i];
                cur[i] = nxt[i];
            }
        }
    }
}

// ---------------------------------------------------------------------------
// Cut selection.
// ---------------------------------------------------------------------------
constexpr uint32_t kInf = 0xFFFFFFFFu;
constexpr uint32_t kM27 = (1u << 27) - 1;
constexpr int kGroup = 32;        // tiles per CTA (one per warp)
constexpr int kItemCache = 2048;  // item offsets cached in shared memory

struct SelWarpSmem {
    uint32_t cand[kSelTileWords];
    uint32_t forced[kSelTileWords];
    uint32_t csum[8];
    uint32_t fsum[8];
};

struct SelSmem {
    SelWarpSmem w[kGroup];
    uint32_t fun[kGroup][32];  // tile transfer functions of the group
    uint32_t te_state[kGroup], te_cnt[kGroup];
    uint64_t items[kItemCache];
};

// First set bit at tile-relative position >= from, or kInf.
__device__ __forceinline__ uint32_t next_set(const uint32_t* words, const uint32_t* summary,
                                             uint32_t from) {
    if (from >= kSelTile) return kInf;
    const uint32_t w = from >> 5;
    const uint32_t b = words[w] & (0xFFFFFFFFu << (from & 31));
    if (b) return (w << 5) + (__ffs(b) - 1);
    const uint32_t sw = w + 1;
    if (sw >= kSelTileWords) return kInf;
    uint32_t si = sw >> 5;
    uint32_t sb = summary[si] & (0xFFFFFFFFu << (sw & 31));
    while (!sb) {
        if (++si >= kSelTileWords / 32) return kInf;
        sb = summary[si];
    }
    const uint32_t ww = (si << 5) + (__ffs(sb) - 1);
    return (ww << 5) + (__ffs(words[ww]) - 1);
}

// Greedy walk over one tile from entry state s: returns the cut count and the
// exit state; if out != nullptr also writes the cut positions.
__device__ __forceinline__ uint32_t walk_tile(const SelWarpSmem& sm, uint32_t s,
                                              uint32_t& exit_state, uint32_t* out,
                                              uint64_t out_base, uint64_t cap, uint64_t T0) {
    uint32_t E = s, cur = 0, cnt = 0;
    while (true) {
        const uint32_t f = next_set(sm.forced, sm.fsum, cur);
        const uint32_t c = next_set(sm.cand, sm.csum, max(E, cur));
        const uint32_t e = min(f, c);
        if (e == kInf) break;
        if (out != nullptr && out_base + cnt < cap) out[out_base + cnt] = (uint32_t)(T0 + e);
        ++cnt;
        E = e + 32;
        cur = e + 1;
    }
    exit_state = E > kSelTile ? E - kSelTile : 0;
    return cnt;
}

// Item offsets: cached in shared memory when they fit.
__device__ __forceinline__ const uint64_t* cache_items(SelSmem& sm, const BatchDesc* desc) {
    const uint32_t n = desc->n_items + 1;
    if (n > kItemCache) return desc->item_off;
    for (uint32_t i = threadIdx.x; i < n; i += blockDim.x) sm.items[i] = desc->item_off[i];
    return sm.items;
}

// Candidate (e-space: cut after byte i <=> e = i + 1) and forced-cut bits of
// tile t into the warp's shared memory, with one-bit-per-word summaries.
__device__ __forceinline__ void build_tile(SelWarpSmem& sm, uint64_t t,
                                           const uint32_t* __restrict__ bitmap, uint64_t nbytes,
                                           const uint64_t* item_off, uint32_t n_items, int lane) {
    const uint64_t T0 = t * kSelTile;
    const uint64_t n_words = (nbytes + 31) / 32;
    uint32_t cw[8], fw[8], raw[9];
    const uint64_t E0 = T0 + (uint64_t)lane * 256;  // this lane's e-range
    const uint64_t g0 = T0 / 32 + lane * 8;
#pragma unroll
    for (int j = 0; j < 9; ++j) {  // bitmap words g0-1 .. g0+7
        const uint64_t g = g0 + j - 1;
        raw[j] = (g0 + j >= 1 && g < n_words) ? bitmap[g] : 0u;
    }
#pragma unroll
    for (int j = 0; j < 8; ++j) {
        uint32_t ew = __funnelshift_l(raw[j], raw[j + 1], 1);
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

// Phase 1 (CTA = 32 warps = one group of 32 tiles): every warp derives its
// tile's 32-entry transfer function agg[32 t + s] = exit(s) << 27 | cuts(s);
// warp 0 composes the 32 functions into the group function gagg[32 g + s].
__global__ void __launch_bounds__(1024)
select_agg_kernel(const BatchDesc* __restrict__ desc, const uint32_t* __restrict__ bitmap,
                  uint32_t* __restrict__ agg, uint32_t* __restrict__ gagg) {
    extern __shared__ __align__(16) uint8_t smraw[];
    SelSmem& sm = *reinterpret_cast<SelSmem*>(smraw);
    const int wid = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint64_t nbytes = desc->nbytes;
    const uint64_t n_tiles = (nbytes + kSelTile - 1) / kSelTile;
    const uint64_t n_groups = (n_tiles + kGroup - 1) / kGroup;
    const uint64_t* items = cache_items(sm, desc);
    const uint32_t n_items = desc->n_items;
    __syncthreads();
    for (uint64_t g = blockIdx.x; g < n_groups; g += gridDim.x) {
        const uint64_t t = g * kGroup + wid;
        uint32_t f = (uint32_t)lane << 27;  // identity beyond the last tile
        if (t < n_tiles) {
            build_tile(sm.w[wid], t, bitmap, nbytes, items, n_items, lane);
            uint32_t ex;
            const uint32_t cnt = walk_tile(sm.w[wid], lane, ex, nullptr, 0, 0, 0);
            f = (ex << 27) | cnt;
            agg[32 * t + lane] = f;
        }
        sm.fun[wid][lane] = f;
        __syncthreads();
        if (wid == 0) {
            uint32_t Gs = lane, Gc = 0;
#pragma unroll 8
            for (int j = 0; j < kGroup; ++j) {
                const uint32_t a = sm.fun[j][lane];
                const uint32_t ns = __shfl_sync(kFull, a >> 27, Gs);
                const uint32_t nc = Gc + __shfl_sync(kFull, a & kM27, Gs);
                Gs = ns;
                Gc = nc;
            }
            gagg[32 * g + lane] = (Gs << 27) | Gc;
        }
        __syncthreads();
    }
}

// Phase 2 (one CTA of 32 warps): prefix composition of the group functions.
// gentry[2g] = entry state of group g, gentry[2g+1] = cuts before it.
__global__ void __launch_bounds__(1024)
select_scan_kernel(const BatchDesc* __restrict__ desc, const uint32_t* __restrict__ gagg,
                   uint32_t* __restrict__ gentry, uint32_t* __restrict__ n_chunks) {
    __shared__ uint32_t fs[32][32], fc[32][32], es[32], ec[32];
    const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint64_t n_tiles = (desc->nbytes + kSelTile - 1) / kSelTile;
    const uint64_t n_units = (n_tiles + kGroup - 1) / kGroup;
    const uint64_t per = (n_units + 31) / 32;
    const uint64_t t0 = w * per, t1 = min(t0 + per, n_units);
    uint32_t Gs = lane, Gc = 0;  // composition of units [t0, t): entry lane -> (state, cuts)
    for (uint64_t tb = t0; tb < t1; tb += 16) {
        uint32_t a[16];  // 16 independent loads in flight, then 16 compositions
#pragma unroll
        for (int j = 0; j < 16; ++j)
            a[j] = tb + j < t1 ? gagg[32 * (tb + j) + lane] : ((uint32_t)lane << 27);
#pragma unroll
        for (int j = 0; j < 16; ++j) {
            const uint32_t ns = __shfl_sync(kFull, a[j] >> 27, Gs);
            const uint32_t nc = Gc + __shfl_sync(kFull, a[j] & kM27, Gs);
            Gs = ns;
            Gc = nc;
        }
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
    for (uint64_t tb = t0; tb < t1; tb += 16) {
        uint32_t a[16];
#pragma unroll
        for (int j = 0; j < 16; ++j)
            a[j] = tb + j < t1 ? gagg[32 * (tb + j) + lane] : ((uint32_t)lane << 27);
#pragma unroll
        for (int j = 0; j < 16; ++j) {
            const uint32_t st = __shfl_sync(kFull, Gs, e_s);
            const uint32_t ct = __shfl_sync(kFull, Gc, e_s);
            if (lane == j && tb + j < t1) {  // spread the stores over lanes
                gentry[2 * (tb + j)] = st;
                gentry[2 * (tb + j) + 1] = e_c + ct;
            }
            const uint32_t ns = __shfl_sync(kFull, a[j] >> 27, Gs);
            const uint32_t nc = Gc + __shfl_sync(kFull, a[j] & kM27, Gs);
            Gs = ns;
            Gc = nc;
        }
    }
}

// Phase 3 (CTA = one group): entry states of the group's tiles from the group
// entry, then every warp replays its tile from its real entry state, writing
// cut_pos.
__global__ void __launch_bounds__(1024)
select_emit_kernel(const BatchDesc* __restrict__ desc, const uint32_t* __restrict__ bitmap,
                   const uint32_t* __restrict__ agg, const uint32_t* __restrict__ gentry,
                   uint32_t* __restrict__ cut_pos, uint64_t cap) {
    extern __shared__ __align__(16) uint8_t smraw[];
    SelSmem& sm = *reinterpret_cast<SelSmem*>(smraw);
    const int wid = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint64_t nbytes = desc->nbytes;
    const uint64_t n_tiles = (nbytes + kSelTile - 1) / kSelTile;
    const uint64_t n_groups = (n_tiles + kGroup - 1) / kGroup;
    const uint64_t* items = cache_items(sm, desc);
    const uint32_t n_items = desc->n_items;
    __syncthreads();
    for (uint64_t g = blockIdx.x; g < n_groups; g += gridDim.x) {
        const uint64_t t = g * kGroup + wid;
        sm.fun[wid][lane] = t < n_tiles ? agg[32 * t + lane] : ((uint32_t)lane << 27);
        __syncthreads();
        if (threadIdx.x == 0) {
            uint32_t s = gentry[2 * g], c = gentry[2 * g + 1];
            for (int j = 0; j < kGroup; ++j) {
                sm.te_state[j] = s;
                sm.te_cnt[j] = c;
                const uint32_t a = sm.fun[j][s];
                c += a & kM27;
                s = a >> 27;
            }
        }
        __syncthreads();
        if (t < n_tiles) {
            build_tile(sm.w[wid], t, bitmap, nbytes, items, n_items, lane);
            const uint32_t st = sm.te_state[wid];
            if (lane == (int)st) {
                uint32_t ex;
                walk_tile(sm.w[wid], st, ex, cut_pos, sm.te_cnt[wid], cap, t * kSelTile);
            }
        }
        __syncthreads();
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
            const uint32_t mid = (lo + hi) >> 1;
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
                const uint64_t mid = (a + b) >> 1;
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
        cudaFuncSetAttribute(rabin_scan_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             kTabBytes);
        cudaFuncSetAttribute(rabin_scan_kernel<false>,
                             cudaFuncAttributeMaxDynamicSharedMemorySize, kTabBytes);
        attr_set = true;
    }
    const unsigned grid = (unsigned)(num_sms * 2);
    if (value == 0)
        rabin_scan_kernel<true><<<grid, kScanThreads, kTabBytes, s>>>(d, d_tab, mask, value, bitmap);
    else
        rabin_scan_kernel<false><<<grid, kScanThreads, kTabBytes, s>>>(d, d_tab, mask, value,
                                                                       bitmap);
}

uint64_t select_groups(uint64_t max_tiles) { return (max_tiles + kGroup - 1) / kGroup; }

void launch_select(const BatchDesc* d, const uint32_t* bitmap, uint32_t* agg, uint32_t* gagg,
                   uint32_t* gentry, uint64_t max_tiles, uint32_t* cut_pos, uint64_t cap,
                   uint32_t* n_chunks, int num_sms, cudaStream_t s) {
    static bool attr_set = false;
    if (!attr_set) {
        cudaFuncSetAttribute(select_agg_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)sizeof(SelSmem));
        cudaFuncSetAttribute(select_emit_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)sizeof(SelSmem));
        attr_set = true;
    }
    uint64_t blocks = select_groups(max_tiles);
    const uint64_t max_blocks = (uint64_t)num_sms * 2;
    if (blocks > max_blocks) blocks = max_blocks;
    if (blocks < 1) blocks = 1;
    select_agg_kernel<<<(unsigned)blocks, 1024, sizeof(SelSmem), s>>>(d, bitmap, agg, gagg);
    select_scan_kernel<<<1, 1024, 0, s>>>(d, gagg, gentry, n_chunks);
    select_emit_kernel<<<(unsigned)blocks, 1024, sizeof(SelSmem), s>>>(d, bitmap, agg, gentry,
                                                                       cut_pos, cap);
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
