// rabin.cu -- rows A2 (Rabin candidate scan) and A3 (cut selection +
// compaction) of the hot path.  PAPER.md P:197 (Rabin fingerprint
// fragmentation of fixed batches, "saved all the indexes where the algorithm
// would fragment the data"), P:199 / Fig. 2 (startPos).
//
// The paper ran this on the CPU; here it is four sm_100a kernels:
//
//  rabin_roll_kernel      persistent, two CTAs of 16 warps per SM.  A warp
//      task is 64 lanes-worth of contiguous ranges (two independent chains
//      per lane, ILP 2); each lane rolls the 32-byte window hash over its
//      range (after a 32-byte warm-up) with the post-shift recurrence
//          h' = ((h << 8) | in) ^ R[h >> 24] ^ W256[out]
//      and stores one candidate bit per byte (e-space bitmap words).  R and
//      W256 are replicated per lane in shared memory ([x][lane] layout: bank
//      = lane, conflict-free); one PRMT builds the LDS offset, the LDS
//      immediate adds the table base.
//  select_tiles_kernel    greedy cut selection is a 32-state machine (with
//      min chunk = window = 32 the only state crossing a position is
//      "positions still blocked", 0..31): per 8 KiB tile a warp applies the
//      item rules, simulates all 32 entry states (lane s = state s) and
//      stores the tile's transfer function and sorted event list (candidates
//      + forced cuts); it composes each group of 32 tiles (warp shuffles).
//  select_scan_kernel     one CTA composes the group functions in order (a
//      prefix over an associative operator) -> entry state and cut offset of
//      every group, and the batch's chunk count.
//  select_emit_ev_kernel  one warp per group derives its tiles' entry states;
//      lane j walks tile j's stored event list from its real entry state,
//      writing the cut positions (the paper's startPos).
// Measured (round 2, C3 bench at 300 steps): the roll and the selection were
// one kernel (selection as the scan CTA's per-group epilogue, 128 KiB of
// shared memory per CTA with the table on a 64 KiB boundary) -- 813 GB/s;
// split, the roll kernel is the hot loop alone -- 872 GB/s.  Measured and not
// kept: L1 / L2 prefetch of the step after next (838 / 841), the two chains
// rolled one after the other so that each chain's load flies during the
// other's half step (854).
// Item starts are forced cuts and reset the state; a candidate is valid only
// if its 32-byte window lies inside one item.
#include <cuda_runtime.h>

#include <mutex>
#include <stdint.h>

#include "internal.h"

namespace dd {

namespace {

constexpr int kTabBytes = 256 * 256;  // [x][R|W][lane] u32 = 64 KiB
constexpr uint32_t kLaneBytes = kSelTile / 32;  // 256 bytes of a tile per lane (selection)
constexpr uint32_t kFull = 0xFFFFFFFFu;
constexpr uint32_t kInf = 0xFFFFFFFFu;
constexpr uint32_t kM27 = (1u << 27) - 1;
constexpr int kGroup = 32;  // tiles per select group

constexpr uint32_t kListCap = 128;  // events per tile kept as a sorted list

struct SelWarpSmem {
    uint32_t cand[kSelTileWords];
    uint32_t forced[kSelTileWords];
    uint32_t csum[8];
    uint32_t fsum[8];
    uint32_t list[kListCap];
};

template <uint32_t kOff = 0>
__device__ __forceinline__ uint32_t lds(uint32_t addr) {
    uint32_t v;
    asm volatile("ld.shared.u32 %0, [%1+%2];" : "=r"(v) : "r"(addr), "n"(kOff));
    return v;
}

// One 256-bit load (LDG.E.256, sm_100) of 32 bytes at a 32-byte aligned p.
// One request per lane-sector instead of two halves the L1 tag work of the
// lane-strided scan loads; L1::no_allocate keeps the streamed bytes out of
// the L1 that the table lookups share.
// (measured: the no-allocate hint +10 %.)
__device__ __forceinline__ void ldg_v8(const uint8_t* p, uint32_t v[8]) {
    asm("ld.global.nc.L1::no_allocate.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
        : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]),
          "=r"(v[7])
        : "l"(p));
}

// 32 bytes at off: ldg_v8 when 32-byte aligned (a32) and the vector lies below
// lim16, else as 16-byte vectors (at or beyond lim16: zero).
__device__ __forceinline__ void load32_v8(const uint8_t* base, uint32_t off, uint32_t lim16,
                                          bool a32, uint32_t v[8]) {
    if (a32 && off + 32 <= lim16) {
        ldg_v8(base + off, v);
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
// Returns the number of events (kInf: use the bitmap walker).  first_rule:
// the first item whose start gets the rules (1 for a carry-over piece that
// continues the stream: its start is not a cut and its windows reach back
// into the previous piece).
__device__ __forceinline__ uint32_t apply_items(SelWarpSmem& sm, uint64_t T0, uint64_t nbytes,
                                                const uint64_t* item_off, uint32_t n_items,
                                                int lane, uint32_t first_rule = 0,
                                                uint32_t first = kInf) {
    uint32_t cw[8], fw[8];
#pragma unroll
    for (int j = 0; j < 8; ++j) {
        cw[j] = sm.cand[lane * 8 + j];
        fw[j] = 0;
    }
    const uint64_t E0 = T0 + (uint64_t)lane * kLaneBytes;  // this lane's e-range
    if (first == kInf) first = first_item(T0, item_off, n_items, lane);
    const uint32_t lo = max(first, first_rule);
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

// Per-tile event slot for the emit kernel: word 0 = number of events (kInf:
// more than kEvSlot, the emit kernel rebuilds the tile), words 1.. = events.
constexpr uint32_t kEvSlot = 15;
constexpr uint32_t kEvWords = kEvSlot + 1;
__device__ __forceinline__ void store_events(const SelWarpSmem& sm, uint32_t n_ev,
                                             uint32_t* __restrict__ slot, int lane) {
    const uint32_t n = n_ev <= kEvSlot ? n_ev : kInf;
    if (lane == 0) slot[0] = n;
    if (n != kInf && (uint32_t)lane < n) slot[1 + lane] = sm.list[lane];
}

// Walk from entry state s using the event list, or the bitmaps if dense.
__device__ __forceinline__ uint32_t walk_any(const SelWarpSmem& sm, uint32_t n_ev, uint32_t s,
                                             uint32_t& exit_state, uint32_t* out,
                                             uint64_t out_base, uint64_t cap, uint64_t T0) {
    if (n_ev != kInf) return walk_events(sm, n_ev, s, exit_state, out, out_base, cap, T0);
    return walk_tile(sm, s, exit_state, out, out_base, cap, T0);
}

// Two independent rolling chains per lane (ILP 2): the LDS -> LOP3 -> PRMT
// dependency of one chain overlaps with the other's.
// Words [W0, W1) of the 32-byte step; bits accumulate into bitsA / bitsB.
template <bool kZeroValue, int W0 = 0, int W1 = 8, uint32_t kOff = 0>
__device__ __forceinline__ void roll32x2(uint32_t& hA, const uint32_t curA[8],
                                         const uint32_t oldA[8], uint32_t& bitsA, uint32_t& hB,
                                         const uint32_t curB[8], const uint32_t oldB[8],
                                         uint32_t& bitsB, uint32_t laneR, uint32_t laneW,
                                         uint32_t mask, uint32_t value) {
    if (W0 == 0) bitsA = bitsB = 0;
#pragma unroll
    for (int w = W0; w < W1; ++w) {
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            const uint32_t aRA = __byte_perm(hA, laneR, 0x7634);
            const uint32_t aRB = __byte_perm(hB, laneR, 0x7634);
            const uint32_t aWA = __byte_perm(oldA[w], laneW, 0x7604 | (k << 4));
            const uint32_t aWB = __byte_perm(oldB[w], laneW, 0x7604 | (k << 4));
            const uint32_t hsA = __byte_perm(curA[w], hA, 0x6540 | k);
            const uint32_t hsB = __byte_perm(curB[w], hB, 0x6540 | k);
            hA = hsA ^ lds<kOff>(aRA) ^ lds<kOff>(aWA);
            hB = hsB ^ lds<kOff>(aRB) ^ lds<kOff>(aWB);
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

// ---- decoupled scan: roll kernel (candidate bitmap) + per-tile selection ----
//
// rabin_roll_kernel: a warp task is 64 x lane_bytes of the batch (two chains
// of 32 lanes x lane_bytes: chain B follows chain A); every lane rolls its
// lane_bytes after a 32-byte warm-up and stores one e-space candidate word
// per 32-byte step.  lane_bytes (a power of two, 256 .. kSelTile) is chosen
// per launch (launch_chunk_select).  No item knowledge, no selection, no
// barrier: the hot loop is the whole kernel.  The 64 KiB table is the only
// shared memory (no static shared memory: the dynamic window starts right
// after the 1 KiB the driver reserves), so two CTAs fit per SM.
constexpr int kRollWarps = 16;
constexpr int kRollThreads = kRollWarps * 32;
constexpr uint32_t kRollWin = 1024;  // shared-window offset of the dynamic smem (1 KiB reserved)

template <bool kZeroValue>
__global__ void __launch_bounds__(kRollThreads, 2)  // <= 64 registers
rabin_roll_kernel(const BatchDesc* __restrict__ desc, const uint32_t* __restrict__ gtab,
                  uint32_t mask, uint32_t value, uint32_t* __restrict__ bitmap,
                  uint32_t lane_bytes) {
    extern __shared__ __align__(16) uint8_t smem[];
    // layout assumption: no static shared memory, so the table (the dynamic
    // window) starts at kRollWin; the LDS immediate adds it to the PRMT-built
    // offset x * 256 + lane * 4 (+ 128 for W)
    if ((uint32_t)__cvta_generic_to_shared(smem) != kRollWin) __trap();
    {
        uint32_t* t32 = reinterpret_cast<uint32_t*>(smem);
        for (int idx = threadIdx.x; idx < kTabBytes / 4; idx += blockDim.x)
            t32[idx] = __ldg(gtab + ((idx >> 5) & 1) * 256 + (idx >> 6));
    }
    __syncthreads();
    const uint8_t* __restrict__ bytes = desc->bytes;
    const uint32_t nbytes = (uint32_t)desc->nbytes;  // <= 2^30 (check_cfg)
    if (nbytes == 0) return;
    const int wid = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint32_t cover = ((nbytes + kSelTile - 1) / kSelTile) * kSelTile;  // bitmap e-range
    const uint32_t chain_bytes = 32 * lane_bytes, task_bytes = 2 * chain_bytes;
    const int steps = (int)(lane_bytes >> 5);
    const uint32_t n_tasks = (cover + task_bytes - 1) / task_bytes;
    const uint32_t lim16 = (nbytes + 15) & ~15u;
    const bool cont = (desc->carry & kCarryCont) != 0;
    const uint32_t laneR = lane * 4;
    const uint32_t laneW = laneR + 128;
    const bool a32 = (reinterpret_cast<uintptr_t>(bytes) & 31) == 0;
    auto fetch = [&](uint32_t offA, uint32_t offB, bool okA, bool okB, uint32_t (&vA)[8],
                     uint32_t (&vB)[8]) {
        if (okA) load32_v8(bytes, offA, lim16, a32, vA);
        if (okB) load32_v8(bytes, offB, lim16, a32, vB);
    };
    for (uint32_t task = blockIdx.x * kRollWarps + wid; task < n_tasks;
         task += gridDim.x * kRollWarps) {
        const uint32_t qA = task * task_bytes + lane * lane_bytes;
        const uint32_t qB = qA + chain_bytes;
        const bool actA = qA < cover, actB = qB < cover;
        uint32_t prevA[8], curA[8], prevB[8], curB[8];
#pragma unroll
        for (int i = 0; i < 8; ++i) prevA[i] = curA[i] = prevB[i] = curB[i] = 0;
        // the whole task inside the batch and 32-byte aligned loads: no guards
        const bool full = a32 && (task + 1) * task_bytes <= nbytes;
        fetch(qA - 32, qB - 32, qA >= 32 && qA < nbytes, qB < nbytes, prevA, prevB);
        fetch(qA, qB, qA < nbytes, qB < nbytes, curA, curB);
        const bool contA = cont && qA == 0;  // carry-over: the stream's 32 bytes before
        if (contA) {
            const uint32_t* hw32 = reinterpret_cast<const uint32_t*>(desc->carry_in->hist);
#pragma unroll
            for (int i = 0; i < 8; ++i) prevA[i] = hw32[i];
        }
        uint32_t hA = 0, hB = 0, pbA = 0, pbB = 0;
        {   // warm-up of both chains: the windows ending at q-1
            const uint32_t zero[8] = {0, 0, 0, 0, 0, 0, 0, 0};
            uint32_t bA, bB;
            roll32x2<kZeroValue, 0, 8, kRollWin>(hA, prevA, zero, bA, hB, prevB, zero, bB, laneR,
                                                 laneW, mask, value);
            pbA = (qA >= 32 || contA) ? bA : 0;
            pbB = bB;  // qB >= 32 always
            if (qA < 32 && !contA) hA = 0;
        }
        // one 32-byte step of both chains (`in` and `old` swap roles every
        // step, as in the fused scan)
        auto step = [&](int j, uint32_t (&inA)[8], uint32_t (&oldA)[8], uint32_t (&inB)[8],
                        uint32_t (&oldB)[8]) {
            const uint32_t bA0 = qA + 32 * j, bB0 = qB + 32 * j;
            uint32_t bitsA, bitsB;
            roll32x2<kZeroValue, 0, 4, kRollWin>(hA, inA, oldA, bitsA, hB, inB, oldB, bitsB, laneR,
                                                 laneW, mask, value);
            roll32x2<kZeroValue, 4, 8, kRollWin>(hA, inA, oldA, bitsA, hB, inB, oldB, bitsB, laneR,
                                                 laneW, mask, value);
            if (j < steps - 1) {  // the next step's bytes into the freed `old`
                if (full) {
                    DD_CHECK(bB0 + 64 <= nbytes && bA0 + 64 <= nbytes);
                    ldg_v8(bytes + bA0 + 32, oldA);
                    ldg_v8(bytes + bB0 + 32, oldB);
                } else {
#pragma unroll
                    for (int i = 0; i < 8; ++i) oldA[i] = oldB[i] = 0;
                    fetch(bA0 + 32, bB0 + 32, bA0 + 32 < nbytes, bB0 + 32 < nbytes, oldA, oldB);
                }
            }
            uint32_t ewA = __funnelshift_l(pbA, bitsA, 1), ewB = __funnelshift_l(pbB, bitsB, 1);
            if (!full) {  // the batch's ragged end
                if (bA0 >= nbytes) ewA = 0;
                else if (bA0 + 32 > nbytes) ewA &= (1u << (nbytes - bA0)) - 1u;
                if (bB0 >= nbytes) ewB = 0;
                else if (bB0 + 32 > nbytes) ewB &= (1u << (nbytes - bB0)) - 1u;
                if (bA0 + 32 > nbytes) bitsA &= bA0 < nbytes ? (1u << (nbytes - bA0)) - 1u : 0u;
                if (bB0 + 32 > nbytes) bitsB &= bB0 < nbytes ? (1u << (nbytes - bB0)) - 1u : 0u;
            }
            DD_CHECK(!(full || actA) || bA0 < cover);
            DD_CHECK(!(full || actB) || bB0 < cover);
            if (full || actA) bitmap[(bA0 >> 5)] = ewA;
            if (full || actB) bitmap[(bB0 >> 5)] = ewB;
            pbA = bitsA;
            pbB = bitsB;
        };
#pragma unroll 1
        for (int j = 0; j < steps; j += 2) {
            step(j, curA, prevA, curB, prevB);
            step(j + 1, prevA, curA, prevB, curB);
        }
    }
}

// Per-tile selection from the candidate bitmap: a CTA of kSelWarps warps
// takes a group of 32 tiles, warp w its tiles w, w + kSelWarps, ...; per tile
// a warp applies the item rules, stores the tile's event list for the emit
// kernel and the tile's transfer function; warp 0 then composes the group's
// function.  A warp's tiles increase, so its first-item index advances
// incrementally (one binary search per warp and group); the next tile's
// candidate words are loaded while the current one is processed.
constexpr int kSelWarps = 8;
struct SelCtaSmem {
    SelWarpSmem w[kSelWarps];
    uint32_t fun[kGroup][33];
};

__global__ void __launch_bounds__(kSelWarps * 32)
select_tiles_kernel(const BatchDesc* __restrict__ desc, const uint32_t* __restrict__ bitmap,
                    uint32_t* __restrict__ agg, uint32_t* __restrict__ gagg,
                    uint32_t* __restrict__ evbuf) {
    extern __shared__ __align__(16) uint8_t smraw[];
    SelCtaSmem& cs = *reinterpret_cast<SelCtaSmem*>(smraw);
    const int wid = threadIdx.x >> 5, lane = threadIdx.x & 31;
    SelWarpSmem& sm = cs.w[wid];
    const uint64_t nbytes = desc->nbytes;
    const uint32_t n_tiles = (uint32_t)((nbytes + kSelTile - 1) / kSelTile);
    const uint32_t n_groups = (n_tiles + kGroup - 1) / kGroup;
    const uint64_t* items = desc->item_off;
    const uint32_t n_items = desc->n_items;
    const uint32_t first_rule = (desc->carry & kCarryCont) ? 1u : 0u;
    for (uint32_t g = blockIdx.x; g < n_groups; g += gridDim.x) {
        const uint32_t t0 = g * kGroup + wid;
        uint4 na = make_uint4(0, 0, 0, 0), nb = na;
        if (t0 < n_tiles) {
            const uint4* src = reinterpret_cast<const uint4*>(bitmap + (size_t)t0 * kSelTileWords);
            na = src[2 * lane];
            nb = src[2 * lane + 1];
        }
        uint32_t first = first_item((uint64_t)t0 * kSelTile, items, n_items, lane);
        for (int j = wid; j < kGroup; j += kSelWarps) {
            const uint32_t t = g * kGroup + j;
            uint32_t f = (uint32_t)lane << 27;
            if (t < n_tiles) {
                uint4* dst = reinterpret_cast<uint4*>(sm.cand);
                dst[2 * lane] = na;
                dst[2 * lane + 1] = nb;
                const uint32_t tn = t + kSelWarps;
                if (tn < n_tiles && j + kSelWarps < kGroup) {  // the next tile's words
                    const uint4* src =
                        reinterpret_cast<const uint4*>(bitmap + (size_t)tn * kSelTileWords);
                    na = src[2 * lane];
                    nb = src[2 * lane + 1];
                }
                // first item whose start is > T0 - 32 (first_item), advanced from
                // the previous tile of this warp
                const uint64_t T0 = (uint64_t)t * kSelTile;
                const uint64_t key = T0 >= 31 ? T0 - 31 : 0;
                if (lane == 0)
                    while (first < n_items && items[first] < key) ++first;
                first = __shfl_sync(kFull, first, 0);
                __syncwarp();
                DD_CHECK(first <= n_items && (first == n_items || items[first] >= key) &&
                         (first == 0 || items[first - 1] < key));
                const uint32_t n_ev =
                    apply_items(sm, T0, nbytes, items, n_items, lane, first_rule, first);
                store_events(sm, n_ev, evbuf + (size_t)t * kEvWords, lane);
                uint32_t ex;
                const uint32_t cnt = walk_any(sm, n_ev, lane, ex, nullptr, 0, 0, 0);
                f = (ex << 27) | cnt;
                agg[32 * t + lane] = f;
                __syncwarp();
            }
            cs.fun[j][lane] = f;
        }
        __syncthreads();
        if (wid == 0) {
            uint32_t Gs = lane, Gc = 0;
#pragma unroll 8
            for (int j = 0; j < kGroup; ++j) {
                const uint32_t a = cs.fun[j][lane];
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
        // the batch starts with a forced cut (entry state 0), or continues a
        // carry-over stream from the previous piece's exit state
        uint32_t s = (desc->carry & kCarryCont) ? desc->carry_in->exit_state : 0u, c = 0;
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

// Cut emission from the scan's per-tile event lists: one warp per group.
// Lane 0 derives the group's tile entry states from the group entry (gentry)
// and the tiles' transfer functions; lane j then walks tile j's stored event
// list (<= kEvSlot events: the common case, ~2 per 8 KiB tile) from its real
// entry state and writes its cut positions.  Tiles with more events (dense
// candidates) are rebuilt cooperatively from the bitmap as in the scan.
constexpr int kEmitEvWarps = 4;
struct EmitEvSmem {
    uint32_t fun[kEmitEvWarps][kGroup][33];
    uint32_t te_state[kEmitEvWarps][kGroup], te_cnt[kEmitEvWarps][kGroup];
    SelWarpSmem w[kEmitEvWarps];
};

__global__ void __launch_bounds__(kEmitEvWarps * 32)
select_emit_ev_kernel(const BatchDesc* __restrict__ desc, const uint32_t* __restrict__ bitmap,
                      const uint32_t* __restrict__ agg, const uint32_t* __restrict__ gentry,
                      const uint32_t* __restrict__ evbuf, uint32_t* __restrict__ cut_pos,
                      uint64_t cap) {
    extern __shared__ __align__(16) uint8_t smraw[];
    EmitEvSmem& sm = *reinterpret_cast<EmitEvSmem*>(smraw);
    const int wid = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint64_t nbytes = desc->nbytes;
    const uint32_t n_tiles = (uint32_t)((nbytes + kSelTile - 1) / kSelTile);
    const uint32_t n_groups = (n_tiles + kGroup - 1) / kGroup;
    const uint64_t* items = desc->item_off;
    const uint32_t n_items = desc->n_items;
    for (uint32_t g = blockIdx.x * kEmitEvWarps + wid; g < n_groups;
         g += gridDim.x * kEmitEvWarps) {
#pragma unroll 4
        for (int j = 0; j < kGroup; ++j) {
            const uint32_t t = g * kGroup + j;
            sm.fun[wid][j][lane] = t < n_tiles ? agg[32 * t + lane] : ((uint32_t)lane << 27);
        }
        // this lane's event slot (64 B) flies during the entry-state chain
        const uint32_t t = g * kGroup + lane;
        uint32_t ev[kEvWords];
        {
            const uint4* sl = reinterpret_cast<const uint4*>(evbuf + (size_t)t * kEvWords);
#pragma unroll
            for (int i = 0; i < (int)kEvWords / 4; ++i) {
                const uint4 v = t < n_tiles ? sl[i] : make_uint4(0, 0, 0, 0);
                ev[4 * i] = v.x; ev[4 * i + 1] = v.y; ev[4 * i + 2] = v.z; ev[4 * i + 3] = v.w;
            }
        }
        __syncwarp();
        if (lane == 0) {
            uint32_t st = gentry[2 * g], c = gentry[2 * g + 1];
            for (int j = 0; j < kGroup; ++j) {
                sm.te_state[wid][j] = st;
                sm.te_cnt[wid][j] = c;
                const uint32_t a = sm.fun[wid][j][st];
                c += a & kM27;
                st = a >> 27;
            }
        }
        __syncwarp();
        const bool dense = t < n_tiles && ev[0] > kEvSlot;
        if (t < n_tiles && !dense) {
            uint32_t E = sm.te_state[wid][lane];
            uint64_t o = sm.te_cnt[wid][lane];
            const uint32_t T0 = t * kSelTile;
#pragma unroll
            for (uint32_t i = 0; i < kEvSlot; ++i) {
                if (i < ev[0]) {
                    const uint32_t e = ev[1 + i], p = e & 0x7FFFFFFFu;
                    if ((e >> 31) || p >= E) {
                        if (o < cap) cut_pos[o] = T0 + p;
                        ++o;
                        E = p + 32;
                    }
                }
            }
        }
        uint32_t dm = __ballot_sync(kFull, dense);
        while (dm) {  // dense tiles: rebuild the candidate words and walk the bitmap
            const int j = __ffs(dm) - 1;
            dm &= dm - 1;
            const uint32_t td = g * kGroup + j;
            SelWarpSmem& w = sm.w[wid];
#pragma unroll
            for (int k = 0; k < 8; ++k)
                w.cand[lane * 8 + k] = bitmap[(size_t)td * kSelTileWords + lane * 8 + k];
            const uint32_t n_ev = apply_items(w, (uint64_t)td * kSelTile, nbytes, items,
                                              n_items, lane,
                                              (desc->carry & kCarryCont) ? 1u : 0u);
            const uint32_t st = sm.te_state[wid][j];
            if (lane == (int)st) {
                uint32_t ex;
                walk_any(w, n_ev, st, ex, cut_pos, sm.te_cnt[wid][j], cap,
                         (uint64_t)td * kSelTile);
            }
            __syncwarp();
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
uint64_t event_words(uint64_t max_tiles) { return max_tiles * kEvWords; }

namespace {
// Function attributes are per device: set once for every device this process
// launches the chunker on (the multi-GPU engine drives several from worker
// threads).
void chunk_set_attrs() {
    static std::mutex mu;
    static uint64_t done_mask = 0;
    int dev = 0;
    cudaGetDevice(&dev);
    const uint64_t bit = 1ull << (dev & 63);
    std::lock_guard<std::mutex> lock(mu);
    if (done_mask & bit) return;
    cudaFuncSetAttribute(select_emit_ev_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         (int)sizeof(EmitEvSmem));
    for (const void* f : {(const void*)rabin_roll_kernel<true>, (const void*)rabin_roll_kernel<false>})
        cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, kTabBytes);
    cudaFuncSetAttribute(select_tiles_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         (int)sizeof(SelCtaSmem));
    done_mask |= bit;
}
}  // namespace

void chunk_set_carveout(int pct) {
    for (const void* f : {(const void*)rabin_roll_kernel<true>, (const void*)rabin_roll_kernel<false>,
                          (const void*)select_tiles_kernel, (const void*)select_scan_kernel,
                          (const void*)select_emit_ev_kernel, (const void*)chunk_meta_kernel})
        cudaFuncSetAttribute(f, cudaFuncAttributePreferredSharedMemoryCarveout, pct);
}

const char* chunk_unlaunchable() {
    chunk_set_attrs();
    for (const void* f : {(const void*)rabin_roll_kernel<true>, (const void*)rabin_roll_kernel<false>})
        if (!fits(f, kRollThreads, kTabBytes)) return "rabin_roll_kernel";
    // the roll kernel addresses its table at window offset kRollWin (the shared
    // memory the driver reserves per block; the kernel traps if it differs)
    int dev = 0, reserved = -1;
    cudaGetDevice(&dev);
    if (cudaDeviceGetAttribute(&reserved, cudaDevAttrReservedSharedMemoryPerBlock, dev) !=
            cudaSuccess ||
        reserved != (int)kRollWin)
        return "rabin_roll_kernel (reserved shared memory per block != 1 KiB)";
    if (!fits((const void*)select_tiles_kernel, kSelWarps * 32, sizeof(SelCtaSmem)))
        return "select_tiles_kernel";
    if (!fits((const void*)select_scan_kernel, 1024, 0)) return "select_scan_kernel";
    if (!fits((const void*)select_emit_ev_kernel, kEmitEvWarps * 32, sizeof(EmitEvSmem)))
        return "select_emit_ev_kernel";
    if (!fits((const void*)chunk_meta_kernel, 256, 0)) return "chunk_meta_kernel";
    return nullptr;
}

void launch_chunk_select(const BatchDesc* d, const uint32_t* d_tab, uint32_t mask,
                         uint32_t value, uint32_t* bitmap, uint32_t* agg, uint32_t* gagg,
                         uint32_t* gentry, uint32_t* evbuf, uint64_t max_tiles,
                         uint32_t* cut_pos, uint64_t cap, uint32_t* n_chunks, int num_sms,
                         cudaStream_t s, cudaEvent_t after_scan, uint32_t max_chunk,
                         uint32_t* mc_ws, uint32_t max_items, uint32_t min_chunk,
                         cudaEvent_t before_select) {
    chunk_set_attrs();
    const uint64_t groups = select_groups(max_tiles);
    {
        // 2 KiB per lane when one task per warp covers the batch on <= 2 CTAs
        // per SM (the pipeline's 64 MiB batches: 32 CTAs, 1.5 % warm-up);
        // bigger launches take 512 B lanes, several tasks per warp, for balance.
        // Measured (C3, 300-step bench / isolated chunk stage over 672 MiB):
        // 512 B 837 / 1562, 1 KiB 867 / 1468, 2 KiB 876 / 1305 GB/s.
        const uint64_t span = max_tiles * kSelTile, cap = (uint64_t)num_sms * 2;
        uint32_t lane_bytes = 2048;
        if ((span + 64 * 2048 - 1) / (64 * 2048) > cap * kRollWarps) lane_bytes = 512;
        const uint64_t tasks = (span + 64 * lane_bytes - 1) / (64 * lane_bytes);
        uint64_t grid = (tasks + kRollWarps - 1) / kRollWarps;
        if (grid > cap) grid = cap;
        if (grid < 1) grid = 1;
        auto k = value == 0 ? rabin_roll_kernel<true> : rabin_roll_kernel<false>;
        k<<<(unsigned)grid, kRollThreads, kTabBytes, s>>>(d, d_tab, mask, value, bitmap,
                                                          lane_bytes);
        uint64_t sb = groups;  // one CTA per group of 32 tiles
        if (sb > (uint64_t)num_sms * 8) sb = (uint64_t)num_sms * 8;
        if (sb < 1) sb = 1;
        select_tiles_kernel<<<(unsigned)sb, kSelWarps * 32, sizeof(SelCtaSmem), s>>>(
            d, bitmap, agg, gagg, evbuf);
    }
    if (after_scan) cudaEventRecordWithFlags(after_scan, s, cudaEventRecordExternal);
    // NEXT-2 max_chunk: the state machine's cuts go to a scratch list first
    uint32_t* final_cut = cut_pos;
    uint32_t* final_n = n_chunks;
    const bool walk = max_chunk != 0 || min_chunk != 32;
    if (walk) {
        n_chunks = mc_ws;
        cut_pos = mc_ws + 1;
    }
    // carry-over: the entry state is the previous piece's exit state
    if (before_select) cudaStreamWaitEvent(s, before_select, cudaEventWaitExternal);
    select_scan_kernel<<<1, 1024, 0, s>>>(d, gagg, gentry, n_chunks);
    uint64_t blocks = (groups + kEmitEvWarps - 1) / kEmitEvWarps;
    if (blocks > (uint64_t)num_sms * 4) blocks = (uint64_t)num_sms * 4;
    if (blocks < 1) blocks = 1;
    select_emit_ev_kernel<<<(unsigned)blocks, kEmitEvWarps * 32, sizeof(EmitEvSmem), s>>>(
        d, bitmap, agg, gentry, evbuf, cut_pos, cap);
    if (walk) {
        uint32_t* item_cnt = mc_ws + 1 + cap;
        uint32_t* item_flag = item_cnt + (uint64_t)max_items + 1;
        launch_select_walk(d, bitmap, max_chunk, min_chunk, item_cnt, item_flag, max_items,
                           cut_pos, n_chunks, final_cut, cap, final_n, num_sms, s);
    }
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
