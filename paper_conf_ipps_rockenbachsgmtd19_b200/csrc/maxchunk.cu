// maxchunk.cu -- row NEXT-2, the max_chunk and min_chunk >
// window chunker variants.  max_chunk:
// cut selection with a maximum chunk length M (PARSEC-style forced cut; the
// oracle's oracle_chunk_item with max_chunk != 0).  After a cut at c the
// next cut is the first Rabin candidate e in [c + 32, min(c + M, r)) of the
// item [q, r), else the forced cut c + M if c + M < r, else the item ends.
//
// The 32-state tile machine of rabin.cu cannot carry "distance since the
// last cut" (up to M states), so with max_chunk the selection is a walk per
// item over the candidate bitmap the scan kernel already wrote (bit e of the
// e-space bitmap <=> the window ending at byte e - 1 hits): one warp per
// item finds each next cut with one coalesced 32-word (1024-position) read
// and a ballot, so the cost is O(chunks + candidate-free words) per item.
// Two passes (count, then write at the item's prefix offset) keep cut_pos
// in batch order.  Items are independent, so the grid covers items.
//
// The walk is a serial chain per item, so it runs only where it can change
// the result: the 32-state machine's cuts (no forced cuts) are computed
// first, and an item whose chunks are all <= M is exactly right already --
// the max rule never fires in it.  Only items holding a chunk > M are
// walked, and only from the start of their first such chunk (the chain
// before it is the machine's); the others copy their cuts.
//
// min_chunk > 32 (the hash restarts at a cut; the next cut is the first
// candidate >= c + min_chunk): the 32-state machine does not apply at all,
// every item is walked with that lower bound.
#include <cuda_runtime.h>
#include <stdint.h>

#include "internal.h"

namespace dd {

namespace {

constexpr uint32_t kFull = 0xFFFFFFFFu;
constexpr uint64_t kNone = ~0ull;
constexpr int kWalkWarps = 8;

// First candidate e in [lo, hi) of the e-space bitmap, or kNone (warp-wide).
__device__ __forceinline__ uint64_t first_candidate(const uint32_t* __restrict__ bitmap,
                                                    uint64_t lo, uint64_t hi, int lane) {
    for (uint64_t w0 = lo >> 5; (w0 << 5) < hi; w0 += 32) {
        const uint64_t w = w0 + lane;
        uint32_t bits = 0;
        if ((w << 5) < hi) {
            bits = bitmap[w];
            if (w == (lo >> 5)) bits &= kFull << (lo & 31);
            if (((w + 1) << 5) > hi) {
                const uint32_t keep = (uint32_t)(hi - (w << 5));  // 1..31
                bits &= (1u << keep) - 1u;
            }
        }
        const uint32_t m = __ballot_sync(kFull, bits != 0);
        if (m) {
            const int src = __ffs(m) - 1;
            const uint32_t b = __shfl_sync(kFull, bits, src);
            return ((w0 + (uint64_t)src) << 5) + (uint64_t)(__ffs(b) - 1);
        }
    }
    return kNone;
}

// First index k with fsm_cut[k] >= x (fsm_cut sorted, n entries).
__device__ __forceinline__ uint32_t lower_cut(const uint32_t* __restrict__ fsm_cut, uint32_t n,
                                              uint64_t x) {
    uint32_t lo = 0, hi = n;
    while (lo < hi) {
        const uint32_t mid = (lo + hi) >> 1;
        if ((uint64_t)fsm_cut[mid] < x) lo = mid + 1;
        else hi = mid;
    }
    return lo;
}

// item_flag[it] = 1 iff item it holds a state-machine chunk longer than M.
__global__ void flag_long_kernel(const BatchDesc* __restrict__ desc,
                                 const uint32_t* __restrict__ fsm_cut,
                                 const uint32_t* __restrict__ fsm_n, uint64_t cap,
                                 uint32_t max_chunk, uint32_t* __restrict__ item_flag) {
    const uint32_t n = (uint32_t)min((uint64_t)*fsm_n, cap);
    const uint64_t nbytes = desc->nbytes;
    const uint32_t n_items = desc->n_items;
    const uint64_t* __restrict__ item_off = desc->item_off;
    for (uint32_t k = blockIdx.x * blockDim.x + threadIdx.x; k < n; k += gridDim.x * blockDim.x) {
        const uint64_t a = fsm_cut[k];
        const uint64_t b = k + 1 < n ? (uint64_t)fsm_cut[k + 1] : nbytes;
        if (b - a <= max_chunk) continue;
        uint32_t lo = 0, hi = n_items;  // last item with item_off <= a (non-empty)
        while (hi - lo > 1) {
            const uint32_t mid = (lo + hi) >> 1;
            if (item_off[mid] <= a) lo = mid;
            else hi = mid;
        }
        while (lo + 1 < n_items && item_off[lo + 1] <= a) ++lo;  // skip empty items
        item_flag[lo] = 1;
    }
}

// Pass 1 (write == false): item_cnt[it] = chunks of item it.
// Pass 2 (write == true): cut_pos[item_cnt[it] + k] = k-th chunk start of it
// (item_cnt holds the exclusive prefix by then).
template <bool kWrite>
__global__ void __launch_bounds__(kWalkWarps * 32)
select_walk_kernel(const BatchDesc* __restrict__ desc, const uint32_t* __restrict__ bitmap,
                   uint32_t max_chunk, uint32_t min_chunk, uint32_t* __restrict__ item_cnt,
                   uint32_t* __restrict__ cut_pos, uint64_t cap,
                   const uint32_t* __restrict__ fsm_cut, const uint32_t* __restrict__ fsm_n,
                   const uint32_t* __restrict__ item_flag) {
    const int lane = threadIdx.x & 31;
    const uint32_t n_items = desc->n_items;
    const uint64_t* __restrict__ item_off = desc->item_off;
    const uint64_t M = max_chunk ? max_chunk : ~0ull >> 1;  // 0: no forced cut
    const uint64_t m = min_chunk;
    const uint32_t nf = (uint32_t)min((uint64_t)*fsm_n, cap);
    for (uint32_t it = blockIdx.x * kWalkWarps + (threadIdx.x >> 5); it < n_items;
         it += gridDim.x * kWalkWarps) {
        const uint64_t q = item_off[it], r = item_off[it + 1];
        const uint64_t base = kWrite ? item_cnt[it] : 0;
        if (!item_flag[it]) {  // the state machine's cuts are exact here: copy them
            const uint32_t k0 = lower_cut(fsm_cut, nf, q), k1 = lower_cut(fsm_cut, nf, r);
            if (kWrite) {
                for (uint32_t k = k0 + lane; k < k1; k += 32)
                    if (base + (k - k0) < cap) cut_pos[base + (k - k0)] = fsm_cut[k];
            } else if (lane == 0) {
                item_cnt[it] = k1 - k0;
            }
            continue;
        }
        uint64_t count = 0;
        uint64_t c = q;
        if (m == 32) {
            // the chain is the state machine's up to the first chunk longer
            // than M: copy those cuts and walk from that chunk's start on
            const uint32_t k0 = lower_cut(fsm_cut, nf, q), k1 = lower_cut(fsm_cut, nf, r);
            const uint64_t nbytes = desc->nbytes;
            uint32_t kf = k1;
            for (uint32_t kb = k0; kb < k1; kb += 32) {
                const uint32_t k = kb + lane;
                bool lng = false;
                if (k < k1) {
                    const uint64_t e = k + 1 < nf ? (uint64_t)fsm_cut[k + 1] : nbytes;
                    lng = e - fsm_cut[k] > M;
                }
                const uint32_t bl = __ballot_sync(kFull, lng);
                if (bl) {
                    kf = kb + (uint32_t)(__ffs(bl) - 1);
                    break;
                }
            }
            if (kWrite)
                for (uint32_t k = k0 + lane; k < kf; k += 32)
                    if (base + (k - k0) < cap) cut_pos[base + (k - k0)] = fsm_cut[k];
            count = kf - k0;
            c = kf < k1 ? (uint64_t)fsm_cut[kf] : r;
        }
        while (c < r) {
            if (kWrite && lane == 0 && base + count < cap) cut_pos[base + count] = (uint32_t)c;
            ++count;
            const uint64_t lim = c + M < r ? c + M : r;
            const uint64_t e = c + m < lim ? first_candidate(bitmap, c + m, lim, lane) : kNone;
            if (e != kNone) c = e;
            else if (c + M < r) c = c + M;
            else break;
        }
        if (!kWrite && lane == 0) item_cnt[it] = (uint32_t)count;
    }
}

// Exclusive prefix of item_cnt[0..n_items) in place; total -> *n_chunks.
__global__ void __launch_bounds__(1024)
item_scan_kernel(const BatchDesc* __restrict__ desc, uint32_t* __restrict__ item_cnt,
                 uint32_t* __restrict__ n_chunks) {
    __shared__ uint32_t s_warp[32];
    __shared__ uint32_t s_carry;
    const uint32_t n = desc->n_items;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    if (threadIdx.x == 0) s_carry = 0;
    __syncthreads();
    for (uint32_t b = 0; b < n; b += 1024) {
        const uint32_t i = b + threadIdx.x;
        const uint32_t v = i < n ? item_cnt[i] : 0u;
        uint32_t x = v;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const uint32_t y = __shfl_up_sync(kFull, x, d);
            if (lane >= d) x += y;
        }
        if (lane == 31) s_warp[wid] = x;
        __syncthreads();
        if (wid == 0) {
            uint32_t t = s_warp[lane];
#pragma unroll
            for (int d = 1; d < 32; d <<= 1) {
                const uint32_t y = __shfl_up_sync(kFull, t, d);
                if (lane >= d) t += y;
            }
            s_warp[lane] = t;  // inclusive over warps
        }
        __syncthreads();
        const uint32_t carry = s_carry;
        const uint32_t excl = carry + (wid ? s_warp[wid - 1] : 0u) + x - v;
        if (i < n) item_cnt[i] = excl;
        __syncthreads();
        if (threadIdx.x == 1023) s_carry = carry + s_warp[31];
        __syncthreads();
    }
    if (threadIdx.x == 0) *n_chunks = s_carry;
}

}  // namespace

void launch_select_walk(const BatchDesc* d, const uint32_t* bitmap, uint32_t max_chunk,
                        uint32_t min_chunk, uint32_t* item_cnt, uint32_t* item_flag,
                        uint32_t max_items, const uint32_t* fsm_cut, const uint32_t* fsm_n,
                        uint32_t* cut_pos, uint64_t cap, uint32_t* n_chunks, int num_sms,
                        cudaStream_t s) {
    if (min_chunk != 32) {
        // the state machine assumes min chunk = window = 32: walk every item
        cudaMemsetAsync(item_flag, 1, sizeof(uint32_t) * ((uint64_t)max_items + 1), s);
    } else {
        cudaMemsetAsync(item_flag, 0, sizeof(uint32_t) * ((uint64_t)max_items + 1), s);
        uint64_t fb = (cap + 255) / 256;
        if (fb > (uint64_t)num_sms * 4) fb = (uint64_t)num_sms * 4;
        if (fb < 1) fb = 1;
        flag_long_kernel<<<(unsigned)fb, 256, 0, s>>>(d, fsm_cut, fsm_n, cap, max_chunk,
                                                      item_flag);
    }
    uint64_t blocks = ((uint64_t)max_items + kWalkWarps - 1) / kWalkWarps;
    if (blocks > (uint64_t)num_sms * 8) blocks = (uint64_t)num_sms * 8;
    if (blocks < 1) blocks = 1;
    select_walk_kernel<false><<<(unsigned)blocks, kWalkWarps * 32, 0, s>>>(
        d, bitmap, max_chunk, min_chunk, item_cnt, cut_pos, cap, fsm_cut, fsm_n, item_flag);
    item_scan_kernel<<<1, 1024, 0, s>>>(d, item_cnt, n_chunks);
    select_walk_kernel<true><<<(unsigned)blocks, kWalkWarps * 32, 0, s>>>(
        d, bitmap, max_chunk, min_chunk, item_cnt, cut_pos, cap, fsm_cut, fsm_n, item_flag);
}

}  // namespace dd
