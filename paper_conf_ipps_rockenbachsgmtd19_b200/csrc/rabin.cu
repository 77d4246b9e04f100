// rabin.cu -- rows A2 (Rabin candidate scan) and A3 (cut selection +
// compaction) of the hot path.  PAPER.md P:197 (Rabin fingerprint
// fragmentation of fixed batches, "saved all the indexes where the algorithm
// would fragment the data"), P:199 / Fig. 2 (startPos).
//
// The paper ran this on the CPU; here it is three sm_100a kernels:
//
//  rabin_scan_agg_kernel  persistent, one CTA of 32 warps per SM.  A warp
//      takes an 8 KiB tile (dynamic counter); each lane rolls the 32-byte
//      window hash over its 256 bytes (after a 32-byte warm-up) with the
//      post-shift recurrence
//          h' = ((h << 8) | in) ^ R[h >> 24] ^ W256[out]
//      and records one candidate bit per byte.  R and W256 are replicated per
//      lane in shared memory ([x][lane] layout: bank = lane, conflict-free);
//      the table sits on a 64 KiB boundary of the shared window so that one
//      PRMT builds the whole LDS address.  Greedy cut selection is then a
//      32-state machine (with min chunk = window = 32 the only state crossing
//      a position is "positions still blocked", 0..31): the warp simulates all
//      32 entry states over its tile (lane s = state s) and stores the tile's
//      transfer function; the last warp to finish a group of 32 tiles composes
//      them into the group function (warp shuffles).
//  select_scan_kernel     one CTA composes the group functions in order (a
//      prefix over an associative operator) -> entry state and cut offset of
//      every group, and the batch's chunk count.
//  select_emit_kernel     one CTA per group derives its tiles' entry states
//      and every warp replays its tile from the real entry state, writing the
//      cut positions (the paper's startPos).
// Item starts are forced cuts and reset the state; a candidate is valid only
// if its 32-byte window lies inside one item.
#include <cuda_runtime.h>
#include <stdint.h>

#include "internal.h"

namespace dd {

namespace {

// 16 warps per SM: enough to saturate the roll (measured: 512 threads/SM
// reach ~97% of the 1024-thread throughput) while leaving half of the
// register file to the SHA-1 / table kernels of other in-flight batches.
constexpr int kScanThreads = 512;
#ifndef DEDUP_SCAN_PREFETCH
#define DEDUP_SCAN_PREFETCH 2
#endif
constexpr int kScanPrefetch = DEDUP_SCAN_PREFETCH;  // 32-byte steps loaded ahead (0..2)
constexpr int kScanWarps = kScanThreads / 32;
constexpr int kEmitThreads = kScanThreads;  // one warp per tile of a group
constexpr int kEmitWarps = kEmitThreads / 32;
constexpr int kTabBytes = 256 * 256;  // [x][R|W][lane] u32 = 64 KiB
constexpr uint32_t kLaneBytes = kSelTile / 32;  // 256 bytes per lane per tile
constexpr uint32_t kFull = 0xFFFFFFFFu;
constexpr uint32_t kInf = 0xFFFFFFFFu;
constexpr uint32_t kM27 = (1u << 27) - 1;
#ifndef DEDUP_SCAN_ILP
#define DEDUP_SCAN_ILP 2
#endif
constexpr int kScanIlp = DEDUP_SCAN_ILP;  // tiles rolled together per warp (1 or 2)
constexpr int kGroup = kScanWarps * kScanIlp;  // tiles per group = one CTA round
constexpr int kItemCache = 1024;  // item offsets cached in shared memory

constexpr uint32_t kListCap = 128;  // events per tile kept as a sorted list

struct SelWarpSmem {
    uint32_t cand[kSelTileWords];
    uint32_t forced[kSelTileWords];
    uint32_t csum[8];
    uint32_t fsum[8];
    uint32_t list[kListCap];
};

// scan: [pad to a 64 KiB shared-window boundary][table]; the per-warp walk
// buffers and the item cache (aux) live in the pad when it is large enough,
// else after the table.
// The aux data must fit the pad, so that a scan CTA needs only 128 KiB of
// dynamic shared memory and other batches' kernels can share the SM; the
// kernel traps if the runtime layout ever leaves a smaller pad.
constexpr int kScanAux = kScanWarps * (int)sizeof(SelWarpSmem) + kItemCache * 8;
constexpr int kScanSmem = 65536 + kTabBytes;
static_assert(kScanAux <= 65536 - 1024 - 8192, "scan aux data must fit the alignment pad");

struct EmitSmem {
    SelWarpSmem w[kEmitWarps];
    uint32_t fun[kGroup][32];
    uint32_t te_state[kGroup], te_cnt[kGroup];
    uint64_t items[kItemCache];
};

// Group buffers in the scan (double buffering across the group barrier).
constexpr int kFunBufs = 2;

__device__ __forceinline__ uint32_t lds(uint32_t addr) {
    uint32_t v;
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(addr));
    return v;
}

// Rolls the 32 bytes of cur[0..7] (stream bytes, little-endian words) into h,
// removing the 32 bytes of old[0..7]; returns the 32 candidate bits
// (bit b <=> the window ending at byte b of this step).
// laneR / laneW = table base (64 KiB aligned) | lane*4 (+128 for W256).
template <bool kZeroValue>
__device__ __forceinline__ uint32_t roll32(uint32_t& h, const uint32_t cur[8],
                                           const uint32_t old[8], uint32_t laneR, uint32_t laneW,
                                           uint32_t mask, uint32_t value) {
    uint32_t bits = 0;
#pragma unroll
    for (int w = 0; w < 8; ++w) {
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            // R[x] at base + x*256 + lane*4, W256[o] at base + o*256 + 128 + lane*4.
            const uint32_t aR = __byte_perm(h, laneR, 0x7634);
            const uint32_t aW = __byte_perm(old[w], laneW, 0x7604 | (k << 4));
            const uint32_t hs = __byte_perm(cur[w], h, 0x6540 | k);  // (h << 8) | in
            h = hs ^ lds(aR) ^ lds(aW);
            const uint32_t t = kZeroValue ? (h & mask) : ((h & mask) ^ value);
            asm("{\n\t.reg .pred p;\n\tsetp.eq.u32 p, %1, 0;\n\t@p or.b32 %0, %0, %2;\n\t}"
                : "+r"(bits)
                : "r"(t), "r"(1u << (4 * w + k)));
        }
    }
    return bits;
}

#ifndef DEDUP_SCAN_EXPERIMENT
#define DEDUP_SCAN_EXPERIMENT 0  // timing experiments only (results invalid): 4 = no
                                 // global loads in the scan, 8 = no per-tile epilogue
#endif

__device__ __forceinline__ void load32(const uint8_t* p, uint32_t v[8]) {
    if (DEDUP_SCAN_EXPERIMENT & 4) {
#pragma unroll
        for (int i = 0; i < 8; ++i) v[i] = (uint32_t)(uintptr_t)p * 2654435761u + i;
        return;
    }
    const uint4 a = __ldg(reinterpret_cast<const uint4*>(p));
    const uint4 b = __ldg(reinterpret_cast<const uint4*>(p + 16));
    v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w;
    v[4] = b.x; v[5] = b.y; v[6] = b.z; v[7] = b.w;
}

// 32 bytes at off; 16-byte vectors at or beyond lim16 (nbytes rounded up to
// 16) read as zero.
__device__ __forceinline__ void load32_any(const uint8_t* base, uint64_t off, uint64_t nbytes,
                                           uint64_t lim16, uint32_t v[8]) {
    if (off + 32 <= nbytes || (DEDUP_SCAN_EXPERIMENT & 4)) {
        load32(base + off, v);
        return;
    }
    uint4 a = make_uint4(0, 0, 0, 0), b = make_uint4(0, 0, 0, 0);
    if (off < lim16) a = __ldg(reinterpret_cast<const uint4*>(base + off));
    if (off + 16 < lim16) b = __ldg(reinterpret_cast<const uint4*>(base + off + 16));
    v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w;
    v[4] = b.x; v[5] = b.y; v[6] = b.z; v[7] = b.w;
}

// 16 bytes at off (16-byte aligned); vectors at or beyond lim16 read as zero.
__device__ __forceinline__ void load16_any(const uint8_t* base, uint64_t off, uint64_t lim16,
                                           uint32_t v[4]) {
    if (DEDUP_SCAN_EXPERIMENT & 4) {
#pragma unroll
        for (int i = 0; i < 4; ++i) v[i] = (uint32_t)off * 2654435761u + i;
        return;
    }
    uint4 a = make_uint4(0, 0, 0, 0);
    if (off < lim16) a = __ldg(reinterpret_cast<const uint4*>(base + off));
    v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w;
}

// 32 bytes at off with one 256-bit load (LDG.E.256, sm_100) when the address
// is 32-byte aligned (a32) and the whole vector lies below lim16, else as
// 16-byte vectors (at or beyond lim16: zero).  One request per lane-sector
// instead of two halves the L1 tag work of the lane-strided scan loads.
__device__ __forceinline__ void load32_v8(const uint8_t* base, uint32_t off, uint32_t lim16,
                                          bool a32, uint32_t v[8]) {
    if (DEDUP_SCAN_EXPERIMENT & 4) {
#pragma unroll
        for (int i = 0; i < 8; ++i) v[i] = off * 2654435761u + i;
        return;
    }
    if (a32 && off + 32 <= lim16) {
#ifndef DEDUP_SCAN_LDHINT
#define DEDUP_SCAN_LDHINT 0  // 1: L1::no_allocate, 2: L2::256B prefetch (timing knobs)
#endif
#if DEDUP_SCAN_LDHINT == 1
#define DEDUP_LDV8 "ld.global.nc.L1::no_allocate.v8.u32"
#elif DEDUP_SCAN_LDHINT == 2
#define DEDUP_LDV8 "ld.global.nc.L2::256B.v8.u32"
#else
#define DEDUP_LDV8 "ld.global.nc.v8.u32"
#endif
        asm(DEDUP_LDV8 " {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
            : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]),
              "=r"(v[6]), "=r"(v[7])
            : "l"(base + off));
        return;
    }
    uint4 a = make_uint4(0, 0, 0, 0), b = make_uint4(0, 0, 0, 0);
    if (off < lim16) a = __ldg(reinterpret_cast<const uint4*>(base + off));
    if (off + 16 < lim16) b = __ldg(reinterpret_cast<const uint4*>(base + off + 16));
    v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w;
    v[4] = b.x; v[5] = b.y; v[6] = b.z; v[7] = b.w;
}

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
__device__ __forceinline__ const uint64_t* cache_items(uint64_t* cache, const BatchDesc* desc) {
    const uint32_t n = desc->n_items + 1;
    if (n > kItemCache) return desc->item_off;
    for (uint32_t i = threadIdx.x; i < n; i += blockDim.x) cache[i] = desc->item_off[i];
    return cache;
}

// Events of a tile as a sorted compact list (bit 31 = forced cut), when there
// are at most kListCap of them; returns their number, or kInf if the list
// would overflow (dense candidates: the bitmap walker is used instead).
__device__ __forceinline__ uint32_t build_events(SelWarpSmem& sm, const uint32_t cw[8],
                                                 const uint32_t fw[8], int lane) {
    uint32_t cnt = 0;
#pragma unroll
    for (int j = 0; j < 8; ++j) cnt += __popc(cw[j] | fw[j]);
    uint32_t incl = cnt;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const uint32_t v = __shfl_up_sync(kFull, incl, d);
        if (lane >= d) incl += v;
    }
    const uint32_t total = __shfl_sync(kFull, incl, 31);
    if (total > kListCap) return kInf;
    uint32_t o = incl - cnt;
#pragma unroll
    for (int j = 0; j < 8; ++j) {
        uint32_t b = cw[j] | fw[j];
        while (b) {
            const uint32_t bit = __ffs(b) - 1;
            b &= b - 1;
            const uint32_t pos = (uint32_t)(lane * kLaneBytes + 32 * j) + bit;
            sm.list[o++] = pos | (((fw[j] >> bit) & 1u) << 31);
        }
    }
    __syncwarp();
    return total;
}

// Greedy walk over the tile's event list from entry state s (see walk_tile).
__device__ __forceinline__ uint32_t walk_events(const SelWarpSmem& sm, uint32_t n_ev, uint32_t s,
                                                uint32_t& exit_state, uint32_t* out,
                                                uint64_t out_base, uint64_t cap, uint64_t T0) {
    uint32_t E = s, cnt = 0;
    for (uint32_t i = 0; i < n_ev; ++i) {
        const uint32_t ev = sm.list[i];
        const uint32_t p = ev & 0x7FFFFFFFu;
        if ((ev >> 31) || p >= E) {
            if (out != nullptr && out_base + cnt < cap) out[out_base + cnt] = (uint32_t)(T0 + p);
            ++cnt;
            E = p + 32;
        }
    }
    exit_state = E > kSelTile ? E - kSelTile : 0;
    return cnt;
}

// First item index whose start is > T0 - 32 (lane 0 searches, all get it).
__device__ __forceinline__ uint32_t first_item(uint64_t T0, const uint64_t* item_off,
                                               uint32_t n_items, int lane) {
    uint32_t lo = 0;
    if (lane == 0 && n_items > 0) {
        const uint64_t key = T0 >= 31 ? T0 - 31 : 0;
        uint32_t hi = n_items;
        while (lo < hi) {
            const uint32_t mid = (lo + hi) >> 1;
            if (item_off[mid] < key) lo = mid + 1; else hi = mid;
        }
    }
    return __shfl_sync(kFull, lo, 0);
}

// Lane's 8 e-space candidate words (already in sm.cand) get the item rules:
// no candidate at e in [q, q+32) (the window would leave the item), a forced
// cut at q for every non-empty item; then the summaries and the event list.
// Returns the number of events (kInf: use the bitmap walker).
__device__ __forceinline__ uint32_t apply_items(SelWarpSmem& sm, uint64_t T0, uint64_t nbytes,
                                                const uint64_t* item_off, uint32_t n_items,
                                                int lane) {
    uint32_t cw[8], fw[8];
#pragma unroll
    for (int j = 0; j < 8; ++j) {
        cw[j] = sm.cand[lane * 8 + j];
        fw[j] = 0;
    }
    const uint64_t E0 = T0 + (uint64_t)lane * kLaneBytes;  // this lane's e-range
    const uint32_t lo = first_item(T0, item_off, n_items, lane);
    if (E0 < nbytes && n_items > 0) {
        for (uint32_t it = lo; it < n_items; ++it) {
            const uint64_t q = item_off[it];
            if (q >= E0 + kLaneBytes) break;
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
    const uint32_t n_ev = build_events(sm, cw, fw, lane);
    if (n_ev != kInf) return n_ev;
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
    return kInf;
}

// Walk from entry state s using the event list, or the bitmaps if dense.
__device__ __forceinline__ uint32_t walk_any(const SelWarpSmem& sm, uint32_t n_ev, uint32_t s,
                                             uint32_t& exit_state, uint32_t* out,
                                             uint64_t out_base, uint64_t cap, uint64_t T0) {
    if (n_ev != kInf) return walk_events(sm, n_ev, s, exit_state, out, out_base, cap, T0);
    return walk_tile(sm, s, exit_state, out, out_base, cap, T0);
}

// Scan + per-tile transfer functions + per-group composition.
// bitmap: e-space candidate words (bit e%32 of word e/32 <=> a window ends at
// byte e-1), before the item rules.  agg[32 t + s] = exit(s) << 27 | cuts(s).
// ctr[0] = tile counter, ctr[1 + g] = arrivals of group g (zeroed per batch).
template <bool kZeroValue>
__global__ void __launch_bounds__(kScanThreads, 2)  // <= 64 registers: half the RF
rabin_scan_agg_kernel(const BatchDesc* __restrict__ desc, const uint32_t* __restrict__ gtab,
                      uint32_t mask, uint32_t value, uint32_t* __restrict__ bitmap,
                      uint32_t* __restrict__ agg, uint32_t* __restrict__ gagg,
                      uint32_t* __restrict__ ctr) {
    extern __shared__ __align__(16) uint8_t smem[];
    __shared__ uint32_t src[512];
    const uint8_t* __restrict__ bytes = desc->bytes;
    const uint64_t nbytes = desc->nbytes;
    const int wid = threadIdx.x >> 5, lane = threadIdx.x & 31;
    // the table starts at the first 64 KiB boundary of the shared window
    const uint32_t win = (uint32_t)__cvta_generic_to_shared(smem);
    const uint32_t pad = (0x10000u - (win & 0xFFFFu)) & 0xFFFFu;
    const uint32_t base = win + pad;
    SelWarpSmem* wsm = reinterpret_cast<SelWarpSmem*>(
        smem);
    if (pad < (uint32_t)kScanAux) __trap();  // layout assumption (see kScanSmem)
    uint64_t* icache = reinterpret_cast<uint64_t*>(wsm + kScanWarps);
    SelWarpSmem& sm = wsm[wid];
    __shared__ uint32_t fun[kFunBufs][kGroup][32];  // tile functions of recent groups
    const uint64_t n_tiles = (nbytes + kSelTile - 1) / kSelTile;
    const uint64_t n_groups = (n_tiles + kGroup - 1) / kGroup;
    const uint64_t lim16 = (nbytes + 15) & ~uint64_t(15);
    // CTA b owns groups b, b + grid, ...; warp w owns tile w of each group
    const uint64_t stride = (uint64_t)gridDim.x * kGroup;
    const uint64_t lo = (uint64_t)blockIdx.x * kGroup, hi = n_groups * kGroup;
    // warm-up window and the first two 32-byte steps of a tile, loaded early
    uint32_t prev[8], cur[8], nxt[8];
    auto load_first = [&](uint64_t t) {
        const uint64_t q = t * kSelTile + (uint64_t)lane * kLaneBytes;
#pragma unroll
        for (int i = 0; i < 8; ++i) prev[i] = cur[i] = nxt[i] = 0;
        if (q >= 32) load32(bytes + q - 32, prev);
        if (q < nbytes) load32_any(bytes, q, nbytes, lim16, cur);
        if (kScanPrefetch == 2 && q + 32 < nbytes) load32_any(bytes, q + 32, nbytes, lim16, nxt);
    };
    if (lo + wid < n_tiles) load_first(lo + wid);  // in flight during the table build
    if (threadIdx.x < 512) src[threadIdx.x] = gtab[threadIdx.x];
    const uint64_t* items = cache_items(icache, desc);
    const uint32_t n_items = desc->n_items;
    __syncthreads();
    {   // replicate R / W256 per lane: word idx = x*64 + half*32 + lane
        uint32_t* t32 = reinterpret_cast<uint32_t*>(smem + pad);
        for (int idx = threadIdx.x; idx < kTabBytes / 4; idx += blockDim.x)
            t32[idx] = src[((idx >> 5) & 1) * 256 + (idx >> 6)];
    }
    __syncthreads();
    if (nbytes == 0) return;
    const uint32_t laneR = base | (lane * 4);
    const uint32_t laneW = laneR + 128;
    int par = 0;
    for (uint64_t t = lo + wid; t < hi; t += stride, par = (par + 1) % kFunBufs) {
      uint32_t f = (uint32_t)lane << 27;  // identity function beyond the last tile
      if (t < n_tiles) {
        const uint64_t T0 = t * kSelTile;
        const uint64_t q = T0 + (uint64_t)lane * kLaneBytes;
        // ---- scan: 8 steps of 32 bytes, bits written in e-space ----
        uint32_t h = 0, prev_bits = 0;
#if DEDUP_SCAN_EXPERIMENT & 2
        if (false) {  // timing experiment only: no warm-up
#else
        if (q >= 32) {  // warm-up: the window ending at q-1 -> bit for e = q
#endif
            const uint32_t zero[8] = {0, 0, 0, 0, 0, 0, 0, 0};
            prev_bits = roll32<kZeroValue>(h, prev, zero, laneR, laneW, mask, value);
        }
#pragma unroll
        for (int j = 0; j < 8; ++j) {
            const uint64_t b0 = q + 32 * j;
            uint32_t bits = 0, nx2[8] = {0, 0, 0, 0, 0, 0, 0, 0};
            if (kScanPrefetch == 2) {
                if (j < 6 && b0 + 64 < nbytes) load32_any(bytes, b0 + 64, nbytes, lim16, nx2);
            } else if (kScanPrefetch == 1) {
                if (j < 7 && b0 + 32 < nbytes) load32_any(bytes, b0 + 32, nbytes, lim16, nx2);
            } else if (j > 0 && b0 < nbytes) {
                load32_any(bytes, b0, nbytes, lim16, cur);
            }
            if (b0 < nbytes) {
                bits = roll32<kZeroValue>(h, cur, prev, laneR, laneW, mask, value);
                if (b0 + 32 > nbytes) bits &= (1u << (uint32_t)(nbytes - b0)) - 1u;
            }
            uint32_t ew = __funnelshift_l(prev_bits, bits, 1);  // e = i + 1
            if (b0 >= nbytes) ew = 0;
            else if (b0 + 32 > nbytes) ew &= (1u << (uint32_t)(nbytes - b0)) - 1u;
            sm.cand[lane * 8 + j] = ew;
            bitmap[T0 / 32 + lane * 8 + j] = ew;
            prev_bits = bits;
#pragma unroll
            for (int i = 0; i < 8; ++i) {
                prev[i] = cur[i];
                if (kScanPrefetch == 2) {
                    cur[i] = nxt[i];
                    nxt[i] = nx2[i];
                } else if (kScanPrefetch == 1) {
                    cur[i] = nx2[i];
                }
            }
        }
        // next tile's first loads fly during the transfer-function walk
        if (t + stride < n_tiles) load_first(t + stride);
        // ---- the tile's 32-entry transfer function ----
        const uint32_t n_ev = apply_items(sm, T0, nbytes, items, n_items, lane);
        uint32_t ex;
        const uint32_t cnt = walk_any(sm, n_ev, lane, ex, nullptr, 0, 0, 0);
        f = (ex << 27) | cnt;
        agg[32 * t + lane] = f;
      }
        // ---- the CTA composes its group of kGroup tiles (the barrier keeps
        // the warps of a CTA in step, measured faster than letting the last
        // arrival compose) ----
        fun[par][wid][lane] = f;
        __syncthreads();
        if (wid == 0) {
            uint32_t Gs = lane, Gc = 0;
#pragma unroll
            for (int j = 0; j < kGroup; ++j) {
                const uint32_t a = fun[par][j][lane];
                const uint32_t ns = __shfl_sync(kFull, a >> 27, Gs);
                const uint32_t nc = Gc + __shfl_sync(kFull, a & kM27, Gs);
                Gs = ns;
                Gc = nc;
            }
            gagg[32 * (t / kGroup) + lane] = (Gs << 27) | Gc;
        }
    }
    (void)ctr;
}

// Two independent rolling chains per lane (ILP 2): the LDS -> LOP3 -> PRMT
// dependency of one chain overlaps with the other's.
// Words [W0, W1) of the 32-byte step; bits accumulate into bitsA / bitsB.
#ifndef DEDUP_SCAN_FMA_AR
#define DEDUP_SCAN_FMA_AR 0
#endif
__device__ __forceinline__ uint32_t mad_hi_u32(uint32_t a, uint32_t b, uint32_t c) {
    uint32_t d;
    asm("mad.hi.u32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(c));
    return d;
}
__device__ __forceinline__ uint32_t mad_lo_u32(uint32_t a, uint32_t b, uint32_t c) {
    uint32_t d;
    asm("mad.lo.u32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(c));
    return d;
}
// LDS address of R[h >> 24] for this lane.  PRMT (ALU pipe), or with
// DEDUP_SCAN_FMA_AR two FMA-pipe ops (c256 = 256 at run time, so that ptxas
// keeps the IMADs): (h >> 24) = mad.hi(h, 256), then * 256 + laneR.
__device__ __forceinline__ uint32_t addr_r(uint32_t h, uint32_t laneR, uint32_t c256) {
    if (DEDUP_SCAN_FMA_AR) return mad_lo_u32(mad_hi_u32(h, c256, 0u), c256, laneR);
    return __byte_perm(h, laneR, 0x7634);
}

template <bool kZeroValue, int W0 = 0, int W1 = 8>
__device__ __forceinline__ void roll32x2(uint32_t& hA, const uint32_t curA[8],
                                         const uint32_t oldA[8], uint32_t& bitsA, uint32_t& hB,
                                         const uint32_t curB[8], const uint32_t oldB[8],
                                         uint32_t& bitsB, uint32_t laneR, uint32_t laneW,
                                         uint32_t mask, uint32_t value, uint32_t c256) {
    if (W0 == 0) bitsA = bitsB = 0;
#pragma unroll
    for (int w = W0; w < W1; ++w) {
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            const uint32_t aRA = addr_r(hA, laneR, c256);
            const uint32_t aRB = addr_r(hB, laneR, c256);
            const uint32_t aWA = __byte_perm(oldA[w], laneW, 0x7604 | (k << 4));
            const uint32_t aWB = __byte_perm(oldB[w], laneW, 0x7604 | (k << 4));
            const uint32_t hsA = __byte_perm(curA[w], hA, 0x6540 | k);
            const uint32_t hsB = __byte_perm(curB[w], hB, 0x6540 | k);
            hA = hsA ^ lds(aRA) ^ lds(aWA);
            hB = hsB ^ lds(aRB) ^ lds(aWB);
            const uint32_t tA = kZeroValue ? (hA & mask) : ((hA & mask) ^ value);
            const uint32_t tB = kZeroValue ? (hB & mask) : ((hB & mask) ^ value);
            asm("{\n\t.reg .pred p;\n\tsetp.eq.u32 p, %1, 0;\n\t@p or.b32 %0, %0, %2;\n\t}"
                : "+r"(bitsA)
                : "r"(tA), "r"(1u << (4 * w + k)));
            asm("{\n\t.reg .pred p;\n\tsetp.eq.u32 p, %1, 0;\n\t@p or.b32 %0, %0, %2;\n\t}"
                : "+r"(bitsB)
                : "r"(tB), "r"(1u << (4 * w + k)));
        }
    }
}

// L2 prefetch of tile t's bytes (and the 32 warm-up bytes before it) by the
// TMA unit: one bulk request per tile, no registers, issued a whole group
// ahead so that the per-step loads of the roll hit L2 instead of HBM.
__device__ __forceinline__ void prefetch_tile_l2(const uint8_t* bytes, uint64_t t,
                                                 uint64_t lim16) {
    uint64_t a = t * kSelTile;
    if (a >= lim16) return;
    a = a >= 32 ? a - 32 : 0;
    uint64_t n = kSelTile + 32;
    if (a + n > lim16) n = lim16 - a;
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(bytes + a), "r"((uint32_t)n)
                 : "memory");
}

// Measured (isolated chunk stage, 256 MiB): no prefetch 938 GB/s, register
// prefetch 949, L2 bulk prefetch 899, both 890 -- the scan is not load-latency
// bound at 16 warps x 2 chains per SM.
#ifndef DEDUP_SCAN_L2PF
#define DEDUP_SCAN_L2PF 0
#endif
#ifndef DEDUP_SCAN_REGPF
#define DEDUP_SCAN_REGPF 1
#endif
// 1: the next step's 32 bytes come with one 256-bit load at the end of a step
// (instead of two 128-bit loads at the halves); needs DEDUP_SCAN_REGPF.
#ifndef DEDUP_SCAN_V8
#define DEDUP_SCAN_V8 1
#endif

// ILP-2 scan: a CTA of kScanWarps warps takes groups of 2 x kScanWarps tiles;
// warp w rolls tiles w and w + kScanWarps of the group together.
template <bool kZeroValue>
__global__ void __launch_bounds__(kScanThreads, 2)
rabin_scan_agg2_kernel(const BatchDesc* __restrict__ desc, const uint32_t* __restrict__ gtab,
                       uint32_t mask, uint32_t value, uint32_t* __restrict__ bitmap,
                       uint32_t* __restrict__ agg, uint32_t* __restrict__ gagg,
                       uint32_t c256) {
    extern __shared__ __align__(16) uint8_t smem[];
    __shared__ uint32_t src[512];
    __shared__ uint32_t fun[kFunBufs][kGroup][32];
    const uint8_t* __restrict__ bytes = desc->bytes;
    const uint32_t nbytes = (uint32_t)desc->nbytes;  // <= 2^30 (check_cfg)
    const int wid = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint32_t win = (uint32_t)__cvta_generic_to_shared(smem);
    const uint32_t pad = (0x10000u - (win & 0xFFFFu)) & 0xFFFFu;
    const uint32_t base = win + pad;
    SelWarpSmem* wsm = reinterpret_cast<SelWarpSmem*>(smem);
    if (pad < (uint32_t)kScanAux) __trap();  // layout assumption (see kScanSmem)
    uint64_t* icache = reinterpret_cast<uint64_t*>(wsm + kScanWarps);
    SelWarpSmem& sm = wsm[wid];
    const uint32_t n_tiles = (nbytes + kSelTile - 1) / kSelTile;
    const uint32_t n_groups = (n_tiles + kGroup - 1) / kGroup;
    const uint32_t lim16 = (nbytes + 15) & ~15u;
    if (DEDUP_SCAN_L2PF && lane == 0 && blockIdx.x < n_groups) {  // first group, during the table build
        prefetch_tile_l2(bytes, (uint64_t)blockIdx.x * kGroup + wid, lim16);
        prefetch_tile_l2(bytes, (uint64_t)blockIdx.x * kGroup + wid + kScanWarps, lim16);
    }
    if (threadIdx.x < 512) src[threadIdx.x] = gtab[threadIdx.x];
    const uint64_t* items = cache_items(icache, desc);
    const uint32_t n_items = desc->n_items;
    __syncthreads();
    {
        uint32_t* t32 = reinterpret_cast<uint32_t*>(smem + pad);
        for (int idx = threadIdx.x; idx < kTabBytes / 4; idx += blockDim.x)
            t32[idx] = src[((idx >> 5) & 1) * 256 + (idx >> 6)];
    }
    __syncthreads();
    if (nbytes == 0) return;
    const uint32_t laneR = base | (lane * 4);
    const uint32_t laneW = laneR + 128;
    const bool a32 = (reinterpret_cast<uintptr_t>(bytes) & 31) == 0;
    int par = 0;
    for (uint32_t g = blockIdx.x; g < n_groups; g += gridDim.x, par ^= 1) {
        const uint32_t tA = g * kGroup + wid, tB = tA + kScanWarps;
        if (DEDUP_SCAN_L2PF && lane == 0 && g + gridDim.x < n_groups) {  // next group
            prefetch_tile_l2(bytes, tA + gridDim.x * kGroup, lim16);
            prefetch_tile_l2(bytes, tB + gridDim.x * kGroup, lim16);
        }
        const uint32_t qA = tA * kSelTile + lane * kLaneBytes;
        const uint32_t qB = tB * kSelTile + lane * kLaneBytes;
        uint32_t prevA[8], curA[8], prevB[8], curB[8];
#pragma unroll
        for (int i = 0; i < 8; ++i) prevA[i] = curA[i] = prevB[i] = curB[i] = 0;
        if (DEDUP_SCAN_V8) {
            if (qA >= 32 && qA < nbytes) load32_v8(bytes, qA - 32, lim16, a32, prevA);
            if (qB >= 32 && qB < nbytes) load32_v8(bytes, qB - 32, lim16, a32, prevB);
            if (qA < nbytes) load32_v8(bytes, qA, lim16, a32, curA);
            if (qB < nbytes) load32_v8(bytes, qB, lim16, a32, curB);
        } else {
            if (qA >= 32 && qA < nbytes) load32(bytes + qA - 32, prevA);
            if (qB >= 32 && qB < nbytes) load32(bytes + qB - 32, prevB);
            if (qA < nbytes) load32_any(bytes, qA, nbytes, lim16, curA);
            if (qB < nbytes) load32_any(bytes, qB, nbytes, lim16, curB);
        }
        uint32_t hA = 0, hB = 0, pbA = 0, pbB = 0;
        {   // warm-up of both chains: the windows ending at q-1
            const uint32_t zero[8] = {0, 0, 0, 0, 0, 0, 0, 0};
            uint32_t bA, bB;
            roll32x2<kZeroValue>(hA, prevA, zero, bA, hB, prevB, zero, bB, laneR, laneW, mask,
                                 value, c256);
            pbA = qA >= 32 ? bA : 0;
            pbB = qB >= 32 ? bB : 0;
            if (qA < 32) hA = 0;
            if (qB < 32) hB = 0;
        }
        // One 32-byte step of both chains: roll `in` against `old`, then the
        // bits in e-space.  With DEDUP_SCAN_REGPF the registers of `old` are
        // recycled: once a half (16 bytes) of `old` has been rolled out, the
        // same four registers receive the NEXT step's bytes of that half, so
        // the loads fly for a whole step with no extra registers; `in` and
        // `old` swap roles every step (the loop body holds two steps).
        auto step = [&](int j, uint32_t (&inA)[8], uint32_t (&oldA)[8], uint32_t (&inB)[8],
                        uint32_t (&oldB)[8]) {
            const uint32_t bA0 = qA + 32 * j, bB0 = qB + 32 * j;
#if !DEDUP_SCAN_REGPF
            if (j > 0) {
                if (bA0 < nbytes) load32_any(bytes, bA0, nbytes, lim16, inA);
                if (bB0 < nbytes) load32_any(bytes, bB0, nbytes, lim16, inB);
            }
#endif
            uint32_t bitsA, bitsB;
            roll32x2<kZeroValue, 0, 4>(hA, inA, oldA, bitsA, hB, inB, oldB, bitsB, laneR, laneW,
                                       mask, value, c256);
#if DEDUP_SCAN_REGPF && !DEDUP_SCAN_V8
            if (j < 7) {
                load16_any(bytes, bA0 + 32, lim16, oldA);
                load16_any(bytes, bB0 + 32, lim16, oldB);
            }
#endif
            roll32x2<kZeroValue, 4, 8>(hA, inA, oldA, bitsA, hB, inB, oldB, bitsB, laneR, laneW,
                                       mask, value, c256);
#if DEDUP_SCAN_REGPF && !DEDUP_SCAN_V8
            if (j < 7) {
                load16_any(bytes, bA0 + 48, lim16, oldA + 4);
                load16_any(bytes, bB0 + 48, lim16, oldB + 4);
            }
#endif
#if DEDUP_SCAN_REGPF && DEDUP_SCAN_V8
            if (j < 7) {
                load32_v8(bytes, bA0 + 32, lim16, a32, oldA);
                load32_v8(bytes, bB0 + 32, lim16, a32, oldB);
            }
#endif
            uint32_t ewA = __funnelshift_l(pbA, bitsA, 1), ewB = __funnelshift_l(pbB, bitsB, 1);
            if (bA0 >= nbytes) ewA = 0;
            else if (bA0 + 32 > nbytes) ewA &= (1u << (uint32_t)(nbytes - bA0)) - 1u;
            if (bB0 >= nbytes) ewB = 0;
            else if (bB0 + 32 > nbytes) ewB &= (1u << (uint32_t)(nbytes - bB0)) - 1u;
            if (bA0 + 32 > nbytes) bitsA &= bA0 < nbytes ? (1u << (uint32_t)(nbytes - bA0)) - 1u : 0u;
            if (bB0 + 32 > nbytes) bitsB &= bB0 < nbytes ? (1u << (uint32_t)(nbytes - bB0)) - 1u : 0u;
            sm.cand[lane * 8 + j] = ewA;
            if (tA < n_tiles) bitmap[tA * kSelTileWords + lane * 8 + j] = ewA;
            if (tB < n_tiles) bitmap[tB * kSelTileWords + lane * 8 + j] = ewB;
            pbA = bitsA;
            pbB = bitsB;
        };
#if DEDUP_SCAN_REGPF
#pragma unroll 1
        for (int j = 0; j < 8; j += 2) {
            step(j, curA, prevA, curB, prevB);      // prev now holds step j+1's bytes
            step(j + 1, prevA, curA, prevB, curB);  // cur now holds step j+2's bytes
        }
#else
#pragma unroll 1
        for (int j = 0; j < 8; ++j) {
            step(j, curA, prevA, curB, prevB);
#pragma unroll
            for (int i = 0; i < 8; ++i) {
                prevA[i] = curA[i];
                prevB[i] = curB[i];
            }
        }
#endif
        // transfer functions of tile A (candidate words already in smem), then B
        uint32_t fA = (uint32_t)lane << 27, fB = fA;
        if (tA < n_tiles && !(DEDUP_SCAN_EXPERIMENT & 8)) {
            const uint32_t n_ev = apply_items(sm, tA * kSelTile, nbytes, items, n_items, lane);
            uint32_t ex;
            const uint32_t cnt = walk_any(sm, n_ev, lane, ex, nullptr, 0, 0, 0);
            fA = (ex << 27) | cnt;
            agg[32 * tA + lane] = fA;
        }
        __syncwarp();
        if (tB < n_tiles && !(DEDUP_SCAN_EXPERIMENT & 8)) {
#pragma unroll
            for (int k = 0; k < 8; ++k)
                sm.cand[lane * 8 + k] = bitmap[tB * kSelTileWords + lane * 8 + k];
            const uint32_t n_ev = apply_items(sm, tB * kSelTile, nbytes, items, n_items, lane);
            uint32_t ex;
            const uint32_t cnt = walk_any(sm, n_ev, lane, ex, nullptr, 0, 0, 0);
            fB = (ex << 27) | cnt;
            agg[32 * tB + lane] = fB;
        }
        fun[par][wid][lane] = fA;
        fun[par][wid + kScanWarps][lane] = fB;
        __syncthreads();
        if (wid == 0) {
            uint32_t Gs = lane, Gc = 0;
#pragma unroll
            for (int j = 0; j < kGroup; ++j) {
                const uint32_t a = fun[par][j][lane];
                const uint32_t ns = __shfl_sync(kFull, a >> 27, Gs);
                const uint32_t nc = Gc + __shfl_sync(kFull, a & kM27, Gs);
                Gs = ns;
                Gc = nc;
            }
            gagg[32 * g + lane] = (Gs << 27) | Gc;
        }
    }
}

// Prefix composition of the group functions (one CTA of 32 warps).
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

// One CTA per group: entry states of the group's tiles from the group entry,
// then the warps replay the group's tiles from their real entry states,
// writing cut_pos.
__global__ void __launch_bounds__(kEmitThreads)
select_emit_kernel(const BatchDesc* __restrict__ desc, const uint32_t* __restrict__ bitmap,
                   const uint32_t* __restrict__ agg, const uint32_t* __restrict__ gentry,
                   uint32_t* __restrict__ cut_pos, uint64_t cap) {
    extern __shared__ __align__(16) uint8_t smraw[];
    EmitSmem& sm = *reinterpret_cast<EmitSmem*>(smraw);
    const int wid = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint64_t nbytes = desc->nbytes;
    const uint64_t n_tiles = (nbytes + kSelTile - 1) / kSelTile;
    const uint64_t n_groups = (n_tiles + kGroup - 1) / kGroup;
    const uint64_t* items = cache_items(sm.items, desc);
    const uint32_t n_items = desc->n_items;
    __syncthreads();
    for (uint64_t g = blockIdx.x; g < n_groups; g += gridDim.x) {
        for (int j = wid; j < kGroup; j += kEmitWarps) {
            const uint64_t t = g * kGroup + j;
            sm.fun[j][lane] = t < n_tiles ? agg[32 * t + lane] : ((uint32_t)lane << 27);
        }
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
        for (int j = wid; j < kGroup; j += kEmitWarps) {
            const uint64_t t = g * kGroup + j;
            if (t >= n_tiles) break;
            SelWarpSmem& w = sm.w[wid];
#pragma unroll
            for (int k = 0; k < 8; ++k)
                w.cand[lane * 8 + k] = bitmap[t * kSelTileWords + lane * 8 + k];
            const uint32_t n_ev = apply_items(w, t * kSelTile, nbytes, items, n_items, lane);
            const uint32_t st = sm.te_state[j];
            if (lane == (int)st) {
                uint32_t ex;
                walk_any(w, n_ev, st, ex, cut_pos, sm.te_cnt[j], cap, t * kSelTile);
            }
            __syncwarp();
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

uint64_t select_groups(uint64_t max_tiles) { return (max_tiles + kGroup - 1) / kGroup; }

namespace {
void chunk_set_attrs() {
    static bool attr_set = false;
    if (attr_set) return;
    for (const void* f : {(const void*)rabin_scan_agg2_kernel<true>,
                          (const void*)rabin_scan_agg2_kernel<false>,
                          (const void*)rabin_scan_agg_kernel<true>,
                          (const void*)rabin_scan_agg_kernel<false>})
        cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, kScanSmem);
    cudaFuncSetAttribute(select_emit_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         (int)sizeof(EmitSmem));
    attr_set = true;
}
}  // namespace

const char* chunk_unlaunchable() {
    chunk_set_attrs();
    const void* kT = kScanIlp == 2 ? (const void*)rabin_scan_agg2_kernel<true>
                                   : (const void*)rabin_scan_agg_kernel<true>;
    const void* kF = kScanIlp == 2 ? (const void*)rabin_scan_agg2_kernel<false>
                                   : (const void*)rabin_scan_agg_kernel<false>;
    if (!fits(kT, kScanThreads, kScanSmem) || !fits(kF, kScanThreads, kScanSmem))
        return "rabin_scan_agg_kernel";
    if (!fits((const void*)select_scan_kernel, 1024, 0)) return "select_scan_kernel";
    if (!fits((const void*)select_emit_kernel, kEmitThreads, sizeof(EmitSmem)))
        return "select_emit_kernel";
    if (!fits((const void*)chunk_meta_kernel, 256, 0)) return "chunk_meta_kernel";
    return nullptr;
}

void launch_chunk_select(const BatchDesc* d, const uint32_t* d_tab, uint32_t mask,
                         uint32_t value, uint32_t* bitmap, uint32_t* agg, uint32_t* gagg,
                         uint32_t* gentry, uint32_t* scan_ctr, uint64_t max_tiles,
                         uint32_t* cut_pos, uint64_t cap, uint32_t* n_chunks, int num_sms,
                         cudaStream_t s, cudaEvent_t after_scan) {
    chunk_set_attrs();
    auto kT = kScanIlp == 2 ? rabin_scan_agg2_kernel<true> : nullptr;
    auto kF = kScanIlp == 2 ? rabin_scan_agg2_kernel<false> : nullptr;
    const uint64_t groups = select_groups(max_tiles);
    const unsigned grid = (unsigned)num_sms;
    if (kScanIlp == 2) {
        (value == 0 ? kT : kF)<<<grid, kScanThreads, kScanSmem, s>>>(d, d_tab, mask, value,
                                                                     bitmap, agg, gagg, 256u);
    } else {
        cudaMemsetAsync(scan_ctr, 0, sizeof(uint32_t) * (groups + 2), s);
        if (value == 0)
            rabin_scan_agg_kernel<true><<<grid, kScanThreads, kScanSmem, s>>>(
                d, d_tab, mask, value, bitmap, agg, gagg, scan_ctr);
        else
            rabin_scan_agg_kernel<false><<<grid, kScanThreads, kScanSmem, s>>>(
                d, d_tab, mask, value, bitmap, agg, gagg, scan_ctr);
    }
    if (after_scan) cudaEventRecordWithFlags(after_scan, s, cudaEventRecordExternal);
    select_scan_kernel<<<1, 1024, 0, s>>>(d, gagg, gentry, n_chunks);
    uint64_t blocks = groups;
    if (blocks > (uint64_t)num_sms) blocks = (uint64_t)num_sms;
    if (blocks < 1) blocks = 1;
    select_emit_kernel<<<(unsigned)blocks, kEmitThreads, sizeof(EmitSmem), s>>>(
        d, bitmap, agg, gentry, cut_pos, cap);
}

void launch_chunk_meta(const BatchDesc* d, const uint32_t* cut_pos, const uint32_t* n_chunks,
                       uint64_t cap, uint32_t* chunk_start, uint64_t* chunk_id,
                       uint32_t* item_first_chunk, uint32_t max_items, int num_sms,
                       cudaStream_t s) {
    if (max_items) cudaMemsetAsync(item_first_chunk, 0xFF, sizeof(uint32_t) * max_items, s);
    uint64_t blocks = (cap + 255) / 256;
    const uint64_t max_blocks = (uint64_t)num_sms;
    if (blocks > max_blocks) blocks = max_blocks;
    if (blocks < 1) blocks = 1;
    chunk_meta_kernel<<<(unsigned)blocks, 256, 0, s>>>(d, cut_pos, n_chunks, cap, chunk_start,
                                                       chunk_id, item_first_chunk);
}

}  // namespace dd
