// lzss.cu -- row NEXT-1 of SURVEY.md section 8(f): the LZSS FindMatch step of
// the paper's GPU Dedup (stage 4, "compress every not
// duplicated blocks on GPU ... reuses data already on GPU"; P:223-225 and
// Listing 3, "running all the FindMatch operations in a single
// kernel function, considering the startPos").
//
// What it computes (Listing 3, readings L1-L6 in DESIGN.md): for every byte
// i of a batch, inside its own block [bs, be) (the chunker's startPos), the
// longest match block[c .. c+L) == block[i .. i+L) with
//     max(i - W, bs) <= c < i,   c + L <= i,   i + L <= be,   L <= MAX_CODED,
// the earliest such c among the longest (the listing's strict `>`), reported
// as length L (0: no byte matches) and offset (c - bs) mod W.
//
// Kept from the paper: one launch over a whole batch, blocks located through
// the startPos array, a block never matches into another block.  Changed for
// sm_100a: the paper's thread per byte scans all W window positions (W byte
// compares per byte, ~4096).  Here a CTA takes a tile of kFmTile positions,
// stages the bytes of the tile and of its window in shared memory and
// bucket-sorts the window positions by byte value (a stable counting sort:
// per-warp histograms built with __match_any_sync, one prefix, an ordered
// scatter).  A position then visits only the window positions that hold its
// own first byte, in increasing order (a binary search finds the first one
// inside its window), rejects a candidate with one compare at the current
// best length, and stops as soon as no later candidate can be longer
// (c >= i - best) -- the same earliest-longest answer with ~W/256 candidates
// per position on high-entropy data instead of W.
#include <cuda_runtime.h>
#include <stdint.h>

#include "internal.h"

namespace dd {

namespace {

constexpr int kFmThreads = 256;
constexpr int kFmWarps = kFmThreads / 32;
constexpr uint32_t kFmTile = 2048;       // positions per tile
// a tile whose most frequent first byte occurs more often than this among
// its candidate positions also builds the 2-byte-keyed list (low entropy)
constexpr uint32_t kWalkMax = 64;
constexpr uint32_t kFull = 0xFFFFFFFFu;

// Dynamic shared memory of a CTA for window W and max length MC (the kernel
// computes the same offsets): region bytes [W + tile + MC + pad], two u32
// candidate lists [W + tile] each, u32 per-warp histograms [warps][256], u32
// bucket starts [257], u32 block starts [tile + 2].
uint32_t fm_smem_bytes(uint32_t W, uint32_t MC) {
    const uint32_t data_bytes = (W + kFmTile + MC + 32 + 15) & ~15u;
    const uint32_t hist_off = (data_bytes + 8 * (W + kFmTile) + 15) & ~15u;
    const uint32_t bstart_off = hist_off + 4 * kFmWarps * 256;
    const uint32_t blk_off = (bstart_off + 4 * 257 + 15) & ~15u;
    return blk_off + 4 * (kFmTile + 2);
}

// Stable counting sort by an 8-bit key of the sequence x in [0, ncand):
// get(x, key, val); dst[rank] = val in (key, x) order.  Warp w owns a
// contiguous segment (per-warp histograms built with __match_any_sync, one
// prefix over (key, warp), an ordered scatter).  bstart (optional) receives
// the 257 key bucket starts.  Called by all threads of the CTA.
template <class Get>
__device__ __forceinline__ void sort_pass(uint32_t ncand, Get get, uint32_t* dst, uint32_t* hist,
                                          uint32_t* bstart, uint32_t* s_scan, int tid, int lane,
                                          int wid) {
    for (int b = tid; b < kFmWarps * 256; b += kFmThreads) hist[b] = 0;
    __syncthreads();
    const uint32_t seg = ((ncand + kFmWarps - 1) / kFmWarps + 31) & ~31u;
    const uint32_t s_lo = wid * seg, s_hi = min(s_lo + seg, ncand);
    uint32_t* wh = hist + wid * 256;
    for (uint32_t x = s_lo; x < s_hi; x += 32) {  // warp-uniform bounds
        const uint32_t q = x + lane;
        uint32_t key = 0x100u + lane, val = 0;
        if (q < s_hi) get(q, key, val);
        const uint32_t peers = __match_any_sync(kFull, key);
        if (q < s_hi && lane == __ffs(peers) - 1) wh[key] += __popc(peers);
        __syncwarp();
    }
    __syncthreads();
    {   // bucket b = tid: per-warp offsets in (key, warp) order
        uint32_t tot = 0;
#pragma unroll
        for (int w = 0; w < kFmWarps; ++w) tot += hist[w * 256 + tid];
        uint32_t incl = tot;  // block-wide inclusive scan over the 256 buckets
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const uint32_t y = __shfl_up_sync(kFull, incl, d);
            if (lane >= d) incl += y;
        }
        if (lane == 31) s_scan[wid] = incl;
        __syncthreads();
        uint32_t before = 0;
        for (int w = 0; w < wid; ++w) before += s_scan[w];
        uint32_t o = before + incl - tot;
        if (bstart) {
            bstart[tid] = o;
            if (tid == kFmThreads - 1) bstart[256] = o + tot;
        }
#pragma unroll
        for (int w = 0; w < kFmWarps; ++w) {
            const uint32_t c = hist[w * 256 + tid];
            hist[w * 256 + tid] = o;
            o += c;
        }
    }
    __syncthreads();
    for (uint32_t x = s_lo; x < s_hi; x += 32) {
        const uint32_t q = x + lane;
        uint32_t key = 0x100u + lane, val = 0;
        if (q < s_hi) get(q, key, val);
        const uint32_t peers = __match_any_sync(kFull, key);
        if (q < s_hi) dst[wh[key] + __popc(peers & ((1u << lane) - 1u))] = val;
        __syncwarp();
        if (q < s_hi && lane == __ffs(peers) - 1) wh[key] += __popc(peers);
        __syncwarp();
    }
    __syncthreads();
}

__global__ void __launch_bounds__(kFmThreads, 4)
findmatch_kernel(const uint8_t* __restrict__ bytes, uint32_t nbytes,
                 const uint32_t* __restrict__ cut_pos, const uint32_t* __restrict__ n_chunks_p,
                 uint64_t cap, const uint8_t* __restrict__ skip, uint32_t W, uint32_t MC,
                 uint8_t* __restrict__ out_len, uint16_t* __restrict__ out_off) {
    extern __shared__ __align__(16) uint8_t smem[];
    const uint32_t data_bytes = (W + kFmTile + MC + 32 + 15) & ~15u;
    const uint32_t list_off = data_bytes;
    const uint32_t list2_off = list_off + 4 * (W + kFmTile);
    const uint32_t hist_off = (list_off + 8 * (W + kFmTile) + 15) & ~15u;
    const uint32_t bstart_off = hist_off + 4 * kFmWarps * 256;
    const uint32_t blk_off = (bstart_off + 4 * 257 + 15) & ~15u;
    uint8_t* data = smem;
    uint32_t* list = reinterpret_cast<uint32_t*>(smem + list_off);
    uint32_t* list2 = reinterpret_cast<uint32_t*>(smem + list2_off);
    uint32_t* hist = reinterpret_cast<uint32_t*>(smem + hist_off);
    uint32_t* bstart = reinterpret_cast<uint32_t*>(smem + bstart_off);
    uint32_t* blk = reinterpret_cast<uint32_t*>(smem + blk_off);
    __shared__ uint32_t s_kb0, s_nblk, s_keyed, s_scan[kFmWarps];
    const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
    const uint32_t n = (uint32_t)min((uint64_t)*n_chunks_p, cap);
    const uint32_t n_tiles = (nbytes + kFmTile - 1) / kFmTile;

    for (uint32_t tile = blockIdx.x; tile < n_tiles; tile += gridDim.x) {
        const uint32_t t0 = tile * kFmTile;
        const uint32_t R1 = min(t0 + kFmTile, nbytes);  // positions of the tile: [t0, R1)
        // ---- blocks overlapping the tile (Listing 3 lines 4-10 for all of
        // its positions): kb0 = last start <= t0 ----
        if (tid == 0) {
            uint32_t lo = 0, hi = n;  // first start > t0
            while (lo < hi) {
                const uint32_t mid = (lo + hi) >> 1;
                if (cut_pos[mid] <= t0) lo = mid + 1;
                else hi = mid;
            }
            s_kb0 = lo;  // kb0 + 1 (0: no start <= t0, virtual start 0)
        }
        __syncthreads();
        const uint32_t kb1 = s_kb0;  // index of the first start > t0
        const uint32_t bs0 = kb1 > 0 ? cut_pos[kb1 - 1] : 0u;
        // blk[0] = bs0, blk[1..m] = starts in (t0, R1), blk[m + 1] = the end of
        // the last of these blocks
        uint32_t cnt = 0;
        for (uint32_t r = 0; r < (kFmTile + kFmThreads) / kFmThreads; ++r) {
            const uint32_t j = r * kFmThreads + tid;
            const uint32_t k = kb1 + j;
            const bool in = j < kFmTile && k < n && cut_pos[k] < R1;
            if (in) blk[1 + j] = cut_pos[k];
            cnt += __syncthreads_count(in);
        }
        const uint32_t m = cnt;  // starts inside (t0, R1)
        if (tid == 0) {
            blk[0] = bs0;
            const uint32_t k = kb1 + m;
            blk[m + 1] = k < n ? cut_pos[k] : nbytes;
            s_nblk = m + 1;
        }
        // ---- stage the bytes [A0, R1 + MC) in shared memory ----
        const uint32_t R0 = max(t0 >= W ? t0 - W : 0u, bs0);  // first candidate
        const uint32_t A0 = R0 & ~15u;
        const uint32_t Aend = min(R1 + MC, nbytes);
        const uint32_t nvec = (Aend - A0 + 15) / 16;
        for (uint32_t v = tid; v < nvec; v += kFmThreads)
            reinterpret_cast<uint4*>(data)[v] =
                __ldg(reinterpret_cast<const uint4*>(bytes + A0) + v);
        __syncthreads();
        // ---- candidate positions [R0, R1 - 1) in two stable orders:
        //   list  by (byte0, position):  r | byte1 << 16 | byte2 << 24
        //   list2 by (byte0, byte1, position) inside byte0's range: byte1 << 16 | r
        // (LSD: by byte1 into `list` as scratch, then by byte0 into list2;
        // then `list` by byte0).  r = region index of the position. ----
        const uint32_t ncand = R1 - 1 > R0 ? R1 - 1 - R0 : 0u;
        const uint32_t rb = R0 - A0;
        // byte histogram of the candidates: long runs of one first byte
        // (low-entropy data) make the one-list walk long, so such tiles also
        // build the 2-byte-keyed list
        for (int b = tid; b < 256; b += kFmThreads) hist[b] = 0;
        __syncthreads();
        for (uint32_t q = tid; q < ncand; q += kFmThreads) atomicAdd(&hist[data[rb + q]], 1u);
        __syncthreads();
        {
            uint32_t v = hist[tid];  // kFmThreads == 256 buckets
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) v = max(v, __shfl_xor_sync(kFull, v, o));
            if (lane == 0) s_scan[wid] = v;
            __syncthreads();
            if (tid == 0) {
                uint32_t m = 0;
                for (int w = 0; w < kFmWarps; ++w) m = max(m, s_scan[w]);
                s_keyed = m > kWalkMax ? 1u : 0u;
            }
            __syncthreads();
        }
        const bool keyed = s_keyed != 0;
        if (keyed) {
            sort_pass(ncand, [&](uint32_t q, uint32_t& key, uint32_t& val) {
                const uint32_t r = rb + q;
                key = data[r + 1];
                val = (key << 16) | r;
            }, list, hist, nullptr, s_scan, tid, lane, wid);
            sort_pass(ncand, [&](uint32_t x, uint32_t& key, uint32_t& val) {
                val = list[x];
                key = data[val & 0xFFFFu];
            }, list2, hist, nullptr, s_scan, tid, lane, wid);
        }
        sort_pass(ncand, [&](uint32_t q, uint32_t& key, uint32_t& val) {
            const uint32_t r = rb + q;
            key = data[r];
            val = r | ((uint32_t)data[r + 1] << 16) | ((uint32_t)data[r + 2] << 24);
        }, list, hist, bstart, s_scan, tid, lane, wid);
        // ---- search: one position per thread per step ----
        const uint32_t nb = s_nblk;
        for (uint32_t i = t0 + tid; i < R1; i += kFmThreads) {
            // block of i: last j with blk[j] <= i (Listing 3 lines 4-10)
            uint32_t lo = 0, hi = nb;  // blk[0] <= i always
            while (hi - lo > 1) {
                const uint32_t mid = (lo + hi) >> 1;
                if (blk[mid] <= i) lo = mid;
                else hi = mid;
            }
            const uint32_t bs = blk[lo], be = blk[lo + 1];
            uint32_t best = 0, bestc = 0;
            const bool skipped = skip != nullptr && kb1 + lo >= 1 && skip[kb1 + lo - 1];
            if (!skipped && i > bs && !keyed) {
                // short first-byte runs: walk the first byte's positions in
                // order; an entry carries its candidate's bytes 1, 2, so most
                // candidates are rejected without touching the region bytes
                const uint32_t wlo = max(i >= W ? i - W : 0u, bs);  // window start
                const uint32_t lim = min(MC, be - i);
                const uint32_t ri = i - A0;
                const uint32_t b0 = data[ri];
                uint32_t e = bstart[b0], eh = bstart[b0 + 1];
                const uint32_t key = wlo - A0;
                while (e < eh) {
                    const uint32_t mid = (e + eh) >> 1;
                    if ((list[mid] & 0xFFFFu) < key) e = mid + 1;
                    else eh = mid;
                }
                eh = bstart[b0 + 1];
                const uint32_t key1 = data[ri + 1], key12 = key1 | ((uint32_t)data[ri + 2] << 8);
                uint32_t kb = 0;  // data[ri + best] once best >= 3
                for (; e < eh; ++e) {
                    const uint32_t E = list[e];
                    const uint32_t rc = E & 0xFFFFu;       // region index of c
                    if (rc + best >= ri) break;            // i - c <= best: no longer match
                    // bytes valid below: best < lim <= be - i and best < i - c
                    if (best == 1 && ((E >> 16) & 0xFFu) != key1) continue;
                    if (best == 2 && (E >> 16) != key12) continue;
                    if (best >= 3 && data[rc + best] != kb) continue;
                    const uint32_t capj = min(lim, ri - rc);
                    uint32_t j = 1;
                    if (capj > 1 && ((E >> 16) & 0xFFu) == key1) {
                        j = 2;
                        if (capj > 2 && (E >> 24) == (key12 >> 8)) {
                            j = 3;
                            while (j < capj && data[rc + j] == data[ri + j]) ++j;
                        }
                    }
                    if (j > best) {
                        best = j;
                        bestc = rc;
                        if (best >= lim) break;            // cannot be beaten
                        if (best >= 3) kb = data[ri + best];
                    }
                }
            }
            if (!skipped && i > bs && keyed) {
                const uint32_t wlo = max(i >= W ? i - W : 0u, bs);  // window start
                const uint32_t lim = min(MC, be - i);
                const uint32_t ri = i - A0;
                const uint32_t b0 = data[ri], b1 = data[ri + 1];
                const uint32_t lo0 = bstart[b0], hi0 = bstart[b0 + 1];
                const uint32_t key = wlo - A0;
                // L >= 1: the first position >= wlo holding byte0 (list)
                uint32_t e = lo0, eh = hi0;
                while (e < eh) {
                    const uint32_t mid = (e + eh) >> 1;
                    if ((list[mid] & 0xFFFFu) < key) e = mid + 1;
                    else eh = mid;
                }
                if (e < hi0 && (list[e] & 0xFFFFu) < ri) {
                    best = 1;
                    bestc = list[e] & 0xFFFFu;
                }
                // L >= 2: positions >= wlo holding byte0 byte1, in order (list2)
                if (best == 1 && lim >= 2) {
                    const uint32_t k2 = (b1 << 16) | key;
                    e = lo0;
                    eh = hi0;
                    while (e < eh) {
                        const uint32_t mid = (e + eh) >> 1;
                        if (list2[mid] < k2) e = mid + 1;
                        else eh = mid;
                    }
                    uint32_t kb = 0;  // data[ri + best] once best >= 2
                    for (; e < hi0; ++e) {
                        const uint32_t E = list2[e];
                        if ((E >> 16) != b1) break;            // past byte1's run
                        const uint32_t rc = E & 0xFFFFu;       // region index of c
                        if (rc + best >= ri) break;            // i - c <= best: no longer match
                        // bytes valid below: best < lim <= be - i and best < i - c
                        if (best >= 2 && data[rc + best] != kb) continue;
                        const uint32_t capj = min(lim, ri - rc);
                        uint32_t j = 2;                        // bytes 0, 1 match by key
                        while (j < capj && data[rc + j] == data[ri + j]) ++j;
                        if (j > best) {
                            best = j;
                            bestc = rc;
                            if (best >= lim) break;            // cannot be beaten
                            kb = data[ri + best];
                        }
                    }
                }
            }
            out_len[i] = (uint8_t)best;
            out_off[i] = best ? (uint16_t)((bestc + A0 - bs) % W) : (uint16_t)0;
        }
        __syncthreads();
    }
}

}  // namespace

uint32_t findmatch_smem(uint32_t window, uint32_t max_coded) {
    return fm_smem_bytes(window, max_coded);
}

const char* findmatch_unlaunchable(uint32_t window, uint32_t max_coded) {
    const uint32_t sm = findmatch_smem(window, max_coded);
    if (cudaFuncSetAttribute(findmatch_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)sm) != cudaSuccess ||
        !fits((const void*)findmatch_kernel, kFmThreads, sm))
        return "findmatch_kernel";
    return nullptr;
}

void launch_findmatch(const uint8_t* bytes, uint32_t nbytes, const uint32_t* cut_pos,
                      const uint32_t* n_chunks, uint64_t cap, const uint8_t* skip,
                      uint32_t window, uint32_t max_coded, uint8_t* out_len, uint16_t* out_off,
                      int num_sms, cudaStream_t s) {
    if (nbytes == 0) return;
    const uint32_t sm = findmatch_smem(window, max_coded);
    int per_sm = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, findmatch_kernel, kFmThreads, sm);
    if (per_sm < 1) per_sm = 1;
    const uint32_t n_tiles = (nbytes + kFmTile - 1) / kFmTile;
    uint32_t grid = (uint32_t)num_sms * (uint32_t)per_sm;
    if (grid > n_tiles) grid = n_tiles;
    findmatch_kernel<<<grid, kFmThreads, sm, s>>>(bytes, nbytes, cut_pos, n_chunks, cap, skip,
                                                  window, max_coded, out_len, out_off);
}

}  // namespace dd
