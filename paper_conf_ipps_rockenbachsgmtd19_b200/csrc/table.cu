// table.cu -- rows A5 (route by digest owner), A7 (global digest table:
// insert + lookup), A8 (reply scatter) and A9 (results into pinned host
// memory).  PAPER.md P:215: "it checks if blocks in the batch are
// duplicated"; results are reordered by sequence on the host.
//
// The table is a GPU-resident open-addressing hash table of 32-byte slots
// (one L2 sector each): 20-byte digest key, a state word claimed by atomic
// CAS (0 empty -> 1 writing -> 2 published), and ~min_id updated with
// atomicMax, so the recorded first occurrence is the minimum (seq, index)
// id -- the sequential stream-order answer -- independent of thread timing
// (reading O12).  Linear probing from 64 digest bits that are
// independent of the owner-routing prefix.
#include <cuda_runtime.h>
#include <stdint.h>

#include <cstdlib>

#include "internal.h"

namespace dd {

namespace {

__device__ __forceinline__ uint32_t ld_acquire(const uint32_t* p) {
    uint32_t v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ void load_key(const uint8_t* digest, const uint64_t* id,
                                         const void* rec, uint64_t r, uint32_t key[5],
                                         uint64_t& myid) {
    if (rec != nullptr) {
        const uint32_t* p = reinterpret_cast<const uint32_t*>(
            static_cast<const uint8_t*>(rec) + 32 * r);
#pragma unroll
        for (int i = 0; i < 5; ++i) key[i] = p[i];
        myid = *reinterpret_cast<const uint64_t*>(p + 6);
    } else {
        const uint32_t* p = reinterpret_cast<const uint32_t*>(digest + 20 * r);
#pragma unroll
        for (int i = 0; i < 5; ++i) key[i] = p[i];
        myid = id != nullptr ? id[r] : r;  // no ids: the record index (local combine)
    }
}

__device__ __forceinline__ uint64_t record_count(const uint32_t* d_n, uint64_t n_host,
                                                 uint64_t cap) {
    return d_n != nullptr ? min((uint64_t)*d_n, cap) : n_host;
}

__global__ void table_prepare_kernel(const BatchDesc* __restrict__ desc) {
    if (!desc->fresh) return;
    const TableView t = desc->table;
    uint4* p = reinterpret_cast<uint4*>(t.slots);
    const uint64_t n = 2 * (t.mask + 1);  // two uint4 per 32-byte slot
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n;
         i += (uint64_t)gridDim.x * blockDim.x)
        p[i] = make_uint4(0, 0, 0, 0);
    if (blockIdx.x == 0 && threadIdx.x < 4) t.status[threadIdx.x] = 0;
}

__global__ void table_insert_kernel(const TableView* __restrict__ tv,
                                    const uint8_t* __restrict__ digest,
                                    const uint64_t* __restrict__ id, const void* rec,
                                    const uint32_t* d_n, uint64_t n_host, uint64_t cap,
                                    uint32_t* __restrict__ slot_idx) {
    const TableView t = *tv;
    const uint64_t n = record_count(d_n, n_host, cap);
    for (uint64_t r = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; r < n;
         r += (uint64_t)gridDim.x * blockDim.x) {
        uint32_t key[5];
        uint64_t myid;
        load_key(digest, id, rec, r, key, myid);
        // bytes 4..11 of the digest; bytes 0..3 pick the owner GPU
        uint64_t idx = (((uint64_t)key[2] << 32) | key[1]) & t.mask;
        uint32_t found = 0xFFFFFFFFu;
        for (uint64_t probe = 0; probe <= t.mask; ++probe) {
            TableSlot* s = t.slots + idx;
            uint32_t st = ld_acquire(&s->state);
            if (st == 0) {
                const uint32_t old = atomicCAS(&s->state, 0u, 1u);
                if (old == 0) {
#pragma unroll
                    for (int i = 0; i < 5; ++i) s->key[i] = key[i];
                    __threadfence();
                    atomicExch(&s->state, 2u);
                    atomicAdd(&t.status[1], 1u);
                    atomicMax(reinterpret_cast<unsigned long long*>(&s->inv_min),
                              (unsigned long long)~myid);
                    found = (uint32_t)idx;
                    break;
                }
                st = old;
            }
            while (st == 1) st = ld_acquire(&s->state);
            bool eq = true;
#pragma unroll
            for (int i = 0; i < 5; ++i) eq = eq && (ld_acquire(&s->key[i]) == key[i]);
            if (eq) {
                atomicMax(reinterpret_cast<unsigned long long*>(&s->inv_min),
                          (unsigned long long)~myid);
                found = (uint32_t)idx;
                break;
            }
            idx = (idx + 1) & t.mask;
        }
        if (found == 0xFFFFFFFFu) atomicExch(&t.status[0], 1u);
        slot_idx[r] = found;
    }
}

__global__ void table_lookup_kernel(const TableView* __restrict__ tv,
                                    const uint64_t* __restrict__ id,
                                    const void* rec, const uint32_t* d_n, uint64_t n_host,
                                    uint64_t cap, const uint32_t* __restrict__ slot_idx,
                                    uint64_t* __restrict__ first_id, uint8_t* __restrict__ is_dup,
                                    uint32_t* __restrict__ status_out,
                                    const uint32_t* __restrict__ cut_pos,
                                    const BatchDesc* __restrict__ desc) {
    const TableView t = *tv;
    const uint64_t n = record_count(d_n, n_host, cap);
    if (status_out != nullptr && blockIdx.x == 0 && threadIdx.x < 2)
        status_out[threadIdx.x] = t.status[threadIdx.x];  // overflow flag, used slots
    // batch statistics (status_out[2..4], zeroed by the caller): duplicate
    // chunks, duplicate bytes, 64-byte SHA-1 blocks
    uint32_t s_dup = 0, s_dup_bytes = 0, s_blocks = 0;
    const uint64_t nbytes = cut_pos != nullptr ? desc->nbytes : 0;
    for (uint64_t r = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; r < n;
         r += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t si = slot_idx[r];
        const uint64_t f = si == 0xFFFFFFFFu ? ~0ull : ~t.slots[si].inv_min;
        first_id[r] = f;
        if (is_dup != nullptr) {
            uint64_t myid = rec != nullptr
                                ? *reinterpret_cast<const uint64_t*>(
                                      static_cast<const uint8_t*>(rec) + 32 * r + 24)
                                : id[r];
            const bool dup = f != myid;
            is_dup[r] = dup ? 1 : 0;
            if (cut_pos != nullptr) {
                const uint64_t e = r + 1 < n ? (uint64_t)cut_pos[r + 1] : nbytes;
                const uint32_t len = (uint32_t)(e - cut_pos[r]);
                s_blocks += (len + 9 + 63) / 64;
                if (dup) {
                    ++s_dup;
                    s_dup_bytes += len;
                }
            }
        }
    }
    if (cut_pos != nullptr) {
        s_dup = __reduce_add_sync(0xFFFFFFFFu, s_dup);
        s_dup_bytes = __reduce_add_sync(0xFFFFFFFFu, s_dup_bytes);
        s_blocks = __reduce_add_sync(0xFFFFFFFFu, s_blocks);
        if ((threadIdx.x & 31) == 0 && (s_dup | s_dup_bytes | s_blocks)) {
            atomicAdd(&status_out[2], s_dup);
            atomicAdd(&status_out[3], s_dup_bytes);
            atomicAdd(&status_out[4], s_blocks);
        }
    }
}

__device__ __forceinline__ uint32_t owner_of(const uint8_t* digest, uint64_t r, uint32_t G) {
    const uint32_t w = *reinterpret_cast<const uint32_t*>(digest + 20 * r);
    const uint32_t be = __byte_perm(w, 0, 0x0123);  // BE32(digest[0..3])
    return (uint32_t)(((uint64_t)be * G) >> 32);
}

// ---- transport 3 (p2p): the exchange fused into the table kernels ----
// One process, G ranks with peer access (NVLink) or sharing a GPU: a rank
// inserts its routed records directly into the owner ranks' shards and later
// reads the first ids back from them (remote atomics / loads on peer memory),
// instead of copying records to the owners and replies back.  System-scope
// atomics and fences: the shards are touched by the SMs of several GPUs.
__device__ __forceinline__ uint32_t ld_acquire_sys(const uint32_t* p) {
    uint32_t v;
    asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ uint32_t owner_of_key(uint32_t k0, uint32_t G) {
    const uint32_t be = __byte_perm(k0, 0, 0x0123);  // BE32(digest[0..3])
    return (uint32_t)(((uint64_t)be * G) >> 32);
}

__global__ void p2p_insert_kernel(const TableView* __restrict__ views, uint32_t G,
                                  const uint8_t* __restrict__ send,
                                  const uint32_t* __restrict__ send_off, uint64_t cap,
                                  uint32_t* __restrict__ slot_idx) {
    const uint64_t n = min((uint64_t)send_off[G], cap);
    for (uint64_t r = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; r < n;
         r += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t* rec = reinterpret_cast<const uint32_t*>(send + 32 * r);  // dedup_record
        uint32_t key[5];
#pragma unroll
        for (int i = 0; i < 5; ++i) key[i] = rec[i];
        const uint64_t myid = *reinterpret_cast<const uint64_t*>(rec + 6);
        DD_CHECK(owner_of_key(key[0], G) < G);
        const TableView t = views[owner_of_key(key[0], G)];
        uint64_t idx = (((uint64_t)key[2] << 32) | key[1]) & t.mask;
        uint32_t found = 0xFFFFFFFFu;
        for (uint64_t probe = 0; probe <= t.mask; ++probe) {
            TableSlot* sl = t.slots + idx;
            uint32_t st = ld_acquire_sys(&sl->state);
            if (st == 0) {
                const uint32_t old = atomicCAS_system(&sl->state, 0u, 1u);
                if (old == 0) {
#pragma unroll
                    for (int i = 0; i < 5; ++i) sl->key[i] = key[i];
                    __threadfence_system();
                    atomicExch_system(&sl->state, 2u);
                    atomicAdd_system(&t.status[1], 1u);
                    atomicMax_system(reinterpret_cast<unsigned long long*>(&sl->inv_min),
                                     (unsigned long long)~myid);
                    found = (uint32_t)idx;
                    break;
                }
                st = old;
            }
            while (st == 1) st = ld_acquire_sys(&sl->state);
            bool eq = true;
#pragma unroll
            for (int i = 0; i < 5; ++i) eq = eq && (ld_acquire_sys(&sl->key[i]) == key[i]);
            if (eq) {
                atomicMax_system(reinterpret_cast<unsigned long long*>(&sl->inv_min),
                                 (unsigned long long)~myid);
                found = (uint32_t)idx;
                break;
            }
            idx = (idx + 1) & t.mask;
        }
        if (found == 0xFFFFFFFFu) atomicExch_system(&t.status[0], 1u);
        slot_idx[r] = found;
    }
}

// After every rank's inserts of the wave: the first id of each routed record
// read from its owner's shard (~0 if the shard overflowed).
__global__ void p2p_lookup_kernel(const TableView* __restrict__ views, uint32_t G,
                                  const uint8_t* __restrict__ send,
                                  const uint32_t* __restrict__ send_off, uint64_t cap,
                                  const uint32_t* __restrict__ slot_idx,
                                  uint64_t* __restrict__ reply_back) {
    const uint64_t n = min((uint64_t)send_off[G], cap);
    for (uint64_t r = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; r < n;
         r += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t si = slot_idx[r];
        const TableView t =
            views[owner_of_key(*reinterpret_cast<const uint32_t*>(send + 32 * r), G)];
        DD_CHECK(si == 0xFFFFFFFFu || si <= t.mask);
        reply_back[r] = si == 0xFFFFFFFFu ? ~0ull : ~t.slots[si].inv_min;
    }
}

// rep (optional, local combine): only records with rep[r] == r are routed.
__device__ __forceinline__ bool routed(const uint32_t* rep, uint64_t r) {
    return rep == nullptr || rep[r] == (uint32_t)r;
}

__global__ void route_count_kernel(const uint8_t* __restrict__ digest, const uint32_t* d_n,
                                   uint64_t cap, uint32_t G, const uint32_t* __restrict__ rep,
                                   uint32_t* counts) {
    __shared__ uint32_t h[64];
    for (int i = threadIdx.x; i < 64; i += blockDim.x) h[i] = 0;
    __syncthreads();
    const uint64_t n = min((uint64_t)*d_n, cap);
    for (uint64_t r = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; r < n;
         r += (uint64_t)gridDim.x * blockDim.x)
        if (routed(rep, r)) atomicAdd(&h[owner_of(digest, r, G)], 1u);
    __syncthreads();
    for (uint32_t i = threadIdx.x; i < G; i += blockDim.x)
        if (h[i]) atomicAdd(&counts[i], h[i]);
}

__global__ void route_scan_kernel(uint32_t G, uint32_t* counts, uint32_t* send_off) {
    if (threadIdx.x == 0 && blockIdx.x == 0) {
        uint32_t acc = 0;
        for (uint32_t i = 0; i < G; ++i) {
            const uint32_t c = counts[i];
            send_off[i] = acc;
            counts[64 + i] = acc;  // scatter cursor
            acc += c;
        }
        send_off[G] = acc;
    }
}

__global__ void route_scatter_kernel(const uint8_t* __restrict__ digest,
                                     const uint64_t* __restrict__ id, const uint32_t* d_n,
                                     uint64_t cap, uint32_t G, const uint32_t* __restrict__ rep,
                                     uint32_t* counts, uint8_t* send,
                                     uint32_t* __restrict__ send_pos) {
    const uint64_t n = min((uint64_t)*d_n, cap);
    for (uint64_t r = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; r < n;
         r += (uint64_t)gridDim.x * blockDim.x) {
        if (!routed(rep, r)) continue;
        const uint32_t o = owner_of(digest, r, G);
        const uint32_t pos = atomicAdd(&counts[64 + o], 1u);
        uint32_t* dst = reinterpret_cast<uint32_t*>(send + 32 * (uint64_t)pos);
        const uint32_t* src = reinterpret_cast<const uint32_t*>(digest + 20 * r);
#pragma unroll
        for (int i = 0; i < 5; ++i) dst[i] = src[i];
        dst[5] = 0;
        *reinterpret_cast<uint64_t*>(dst + 6) = id[r];
        send_pos[r] = pos;
    }
}

__global__ void scatter_kernel(const uint64_t* __restrict__ reply,
                               const uint32_t* __restrict__ send_pos,
                               const uint32_t* __restrict__ rep,
                               const uint64_t* __restrict__ id, const uint32_t* d_n, uint64_t cap,
                               uint64_t* __restrict__ first_id, uint8_t* __restrict__ is_dup,
                               uint32_t* overflow) {
    const uint64_t n = min((uint64_t)*d_n, cap);
    bool bad = false;
    for (uint64_t r = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; r < n;
         r += (uint64_t)gridDim.x * blockDim.x) {
        // with local combine a chunk takes the reply of its representative
        const uint64_t f = reply[send_pos[rep != nullptr ? rep[r] : (uint32_t)r]];
        first_id[r] = f;
        if (is_dup != nullptr) is_dup[r] = (f != id[r]) ? 1 : 0;
        bad |= f == ~0ull;  // the owner's shard overflowed (table_lookup_kernel)
    }
    if (overflow != nullptr && bad) atomicExch(overflow, 1u);
}

// Copy exchange (the in-process transport of the multi-GPU engine, mg.cpp):
// rank `me` pulls its rows from every rank s.  Source s's rows for `me` are
// rows [src_off[s][me], src_off[s][me + 1]) of src[s] (row_bytes each, a
// multiple of 8); they land at dst_off[s] (if given) or at the prefix of
// the counts over s, which is then written to out_off[0..G] (out_off[G] =
// total rows).  One CTA group per source; peer pointers are device memory
// of this GPU or of a peer GPU with peer access enabled (NVLink).
__global__ void gather_rows_kernel(const uint8_t* const* __restrict__ src,
                                   const uint32_t* const* __restrict__ src_off, uint32_t me,
                                   uint32_t G, uint32_t row_bytes, uint8_t* __restrict__ dst,
                                   const uint32_t* __restrict__ dst_off,
                                   uint32_t* __restrict__ out_off) {
    const uint32_t s = blockIdx.y;
    uint64_t base = 0;
    if (dst_off != nullptr) {
        base = dst_off[s];
    } else {
        for (uint32_t q = 0; q < s; ++q) base += src_off[q][me + 1] - src_off[q][me];
        if (blockIdx.x == 0 && threadIdx.x == 0) {
            out_off[s] = (uint32_t)base;
            if (s == G - 1) out_off[G] = (uint32_t)(base + src_off[s][me + 1] - src_off[s][me]);
        }
    }
    const uint32_t b = src_off[s][me], e = src_off[s][me + 1];
    const uint64_t words = (uint64_t)(e - b) * (row_bytes / 8);
    const uint64_t* __restrict__ sp =
        reinterpret_cast<const uint64_t*>(src[s] + (uint64_t)b * row_bytes);
    uint64_t* __restrict__ dp = reinterpret_cast<uint64_t*>(dst + base * row_bytes);
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < words;
         i += (uint64_t)gridDim.x * blockDim.x)
        dp[i] = sp[i];
}

// counts: cnt[2 s], cnt[2 s + 1] = rank s's send_off[me], send_off[me + 1]
__global__ void gather_counts_kernel(const uint32_t* const* __restrict__ src_off, uint32_t me,
                                     uint32_t G, uint32_t* __restrict__ cnt) {
    for (uint32_t s = threadIdx.x; s < G; s += blockDim.x) {
        cnt[2 * s] = src_off[s][me];
        cnt[2 * s + 1] = src_off[s][me + 1];
    }
}

// Local combine (row A5): after the insert of records 0..n-1 with ids = the
// record index into the ctx's local table, rep[r] = the smallest index with
// the same digest; then the slots this batch used are cleared again (O(n),
// no full-table memset per wave).
__global__ void combine_rep_kernel(TableView t, const uint32_t* d_n, uint64_t cap,
                                   const uint32_t* __restrict__ slot_idx,
                                   uint32_t* __restrict__ rep) {
    const uint64_t n = min((uint64_t)*d_n, cap);
    for (uint64_t r = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; r < n;
         r += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t si = slot_idx[r];
        rep[r] = si == 0xFFFFFFFFu ? (uint32_t)r : (uint32_t)~t.slots[si].inv_min;
    }
}

__global__ void table_clear_used_kernel(TableView t, const uint32_t* d_n, uint64_t cap,
                                        const uint32_t* __restrict__ slot_idx) {
    const uint64_t n = min((uint64_t)*d_n, cap);
    for (uint64_t r = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; r < n;
         r += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t si = slot_idx[r];
        if (si != 0xFFFFFFFFu) {
            uint4* p = reinterpret_cast<uint4*>(t.slots + si);
            p[0] = make_uint4(0, 0, 0, 0);
            p[1] = make_uint4(0, 0, 0, 0);
        }
    }
    if (blockIdx.x == 0 && threadIdx.x < 4) t.status[threadIdx.x] = 0;
}

__global__ void pack_kernel(const BatchDesc* __restrict__ desc,
                            const uint32_t* __restrict__ n_chunks_p, uint64_t cap,
                            const uint32_t* __restrict__ chunk_start,
                            const uint64_t* __restrict__ first_id,
                            const uint8_t* __restrict__ digest, const uint8_t* __restrict__ is_dup,
                            const uint32_t* __restrict__ item_first_chunk,
                            const uint32_t* __restrict__ table_status, HostResultLayout h,
                            const uint32_t* __restrict__ extra) {
    const uint64_t n = min((uint64_t)*n_chunks_p, cap);
    const uint32_t n_items = desc->n_items;
    const uint64_t tid = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    if (tid == 0) {
        h.header[0] = (uint32_t)*n_chunks_p;
        h.header[1] = table_status[0];  // overflow flag (copied by the lookup)
        h.header[2] = table_status[1];  // used table slots
        h.header[3] = table_status[2];  // duplicate chunks
        h.header[4] = table_status[3];  // duplicate bytes
        h.header[5] = table_status[4];  // SHA-1 blocks
        for (int i = 0; i < 3; ++i) h.header[6 + i] = extra != nullptr ? extra[i] : 0u;
    }
    for (uint64_t r = tid; r < n; r += stride) {
        h.chunk_start[r] = chunk_start[r];
        h.first_id[r] = first_id[r];
        h.is_dup[r] = is_dup[r];
    }
    const uint32_t* dw = reinterpret_cast<const uint32_t*>(digest);
    uint32_t* hw = reinterpret_cast<uint32_t*>(h.digest);
    for (uint64_t r = tid; r < 5 * n; r += stride) hw[r] = dw[r];
    for (uint64_t r = tid; r < n_items; r += stride) h.item_first_chunk[r] = item_first_chunk[r];
}

unsigned grid_for(uint64_t n, int threads, int num_sms, int per_sm) {
    uint64_t b = (n + threads - 1) / threads;
    const uint64_t mx = (uint64_t)num_sms * per_sm;
    if (b > mx) b = mx;
    if (b == 0) b = 1;
    return (unsigned)b;
}

}  // namespace

void launch_table_prepare(const BatchDesc* d, uint64_t max_slots, int num_sms, cudaStream_t s) {
    // small grids (grid-stride loops) so that the kernels of other in-flight
    // batches keep their SMs
    table_prepare_kernel<<<grid_for(2 * max_slots, 256, 32, 1), 256, 0, s>>>(d);
}

void launch_table_insert(const TableView* t, const uint8_t* digest, const uint64_t* id,
                         const void* rec, const uint32_t* d_n, uint64_t n_host, uint64_t cap,
                         uint32_t* slot_idx, int num_sms, cudaStream_t s) {
    const uint64_t n = d_n != nullptr ? cap : n_host;
    if (n == 0) return;
    table_insert_kernel<<<grid_for(n, 256, num_sms, 1), 256, 0, s>>>(t, digest, id, rec, d_n,
                                                                       n_host, cap, slot_idx);
}

void launch_table_lookup(const TableView* t, const uint64_t* id, const void* rec,
                         const uint32_t* d_n, uint64_t n_host, uint64_t cap,
                         const uint32_t* slot_idx, uint64_t* first_id, uint8_t* is_dup,
                         uint32_t* status_out, const uint32_t* cut_pos,
                         const BatchDesc* desc, int num_sms, cudaStream_t s) {
    const uint64_t n = d_n != nullptr ? cap : n_host;
    table_lookup_kernel<<<grid_for(n, 256, num_sms, 1), 256, 0, s>>>(
        t, id, rec, d_n, n_host, cap, slot_idx, first_id, is_dup, status_out, cut_pos, desc);
}

// One shared-memory / L1 split for every kernel of the batch pipeline, so
// that co-resident CTAs of different kernels never force an SM to
// reconfigure (the driver's per-kernel default picks max L1 for the kernels
// without shared memory and a large carve-out for the roll kernel).
// Measured (C3 bench, 300 / 20 steps, interleaved reps): no preference
// 899-903 / 840-860 GB/s; 44-52 % 923-925 / 865-884; 58 % 913-916 / 861-876;
// 72 % 907; 86-100 % 688-693 (too little L1 for SHA-1's 16-byte loads);
// 36-40 % 890-901; 0 % (max L1) 768-773 at 20 steps.  DEDUP_CARVEOUT=<pct>
// overrides (A/B runs); -1 keeps the driver's choice.
void set_pipeline_carveout() {
    int pct = 48;
    if (const char* cv = std::getenv("DEDUP_CARVEOUT")) pct = std::atoi(cv);
    if (pct < 0) return;
    sha1_set_carveout(pct);
    chunk_set_carveout(pct);
    table_set_carveout(pct);
}

void table_set_carveout(int pct) {
    for (const void* f :
         {(const void*)table_prepare_kernel, (const void*)table_insert_kernel,
          (const void*)table_lookup_kernel, (const void*)pack_kernel, (const void*)scatter_kernel,
          (const void*)route_count_kernel, (const void*)route_scan_kernel,
          (const void*)route_scatter_kernel, (const void*)combine_rep_kernel,
          (const void*)gather_rows_kernel, (const void*)gather_counts_kernel,
          (const void*)p2p_insert_kernel, (const void*)p2p_lookup_kernel})
        cudaFuncSetAttribute(f, cudaFuncAttributePreferredSharedMemoryCarveout, pct);
}

void launch_p2p_insert(const TableView* views, uint32_t G, const void* send,
                       const uint32_t* send_off, uint64_t cap, uint32_t* slot_idx, int num_sms,
                       cudaStream_t s) {
    if (cap == 0) return;
    p2p_insert_kernel<<<grid_for(cap, 256, num_sms, 1), 256, 0, s>>>(
        views, G, static_cast<const uint8_t*>(send), send_off, cap, slot_idx);
}

void launch_p2p_lookup(const TableView* views, uint32_t G, const void* send,
                       const uint32_t* send_off, uint64_t cap, const uint32_t* slot_idx,
                       uint64_t* reply_back, int num_sms, cudaStream_t s) {
    if (cap == 0) return;
    p2p_lookup_kernel<<<grid_for(cap, 256, num_sms, 1), 256, 0, s>>>(
        views, G, static_cast<const uint8_t*>(send), send_off, cap, slot_idx, reply_back);
}

void launch_route(const uint8_t* digest, const uint64_t* id, const uint32_t* d_n, uint64_t cap,
                  const uint32_t* rep, uint32_t num_owners, void* send, uint32_t* send_off,
                  uint32_t* send_pos, uint32_t* scratch_counts, int num_sms, cudaStream_t s) {
    cudaMemsetAsync(scratch_counts, 0, sizeof(uint32_t) * 128, s);
    const unsigned g = grid_for(cap, 256, num_sms, 4);
    if (cap)
        route_count_kernel<<<g, 256, 0, s>>>(digest, d_n, cap, num_owners, rep, scratch_counts);
    route_scan_kernel<<<1, 32, 0, s>>>(num_owners, scratch_counts, send_off);
    if (cap)
        route_scatter_kernel<<<g, 256, 0, s>>>(digest, id, d_n, cap, num_owners, rep,
                                               scratch_counts, static_cast<uint8_t*>(send),
                                               send_pos);
}

void launch_scatter(const uint64_t* reply, const uint32_t* send_pos, const uint32_t* rep,
                    const uint64_t* id, const uint32_t* d_n, uint64_t cap, uint64_t* first_id,
                    uint8_t* is_dup, int num_sms, cudaStream_t s, uint32_t* overflow) {
    if (cap == 0) return;
    scatter_kernel<<<grid_for(cap, 256, num_sms, 8), 256, 0, s>>>(reply, send_pos, rep, id, d_n,
                                                                  cap, first_id, is_dup, overflow);
}

void launch_gather_rows(const uint8_t* const* src, const uint32_t* const* src_off, uint32_t me,
                        uint32_t G, uint32_t row_bytes, uint8_t* dst, const uint32_t* dst_off,
                        uint32_t* out_off, uint64_t max_rows_per_src, int num_sms,
                        cudaStream_t s) {
    const uint64_t words = max_rows_per_src * (row_bytes / 8);
    uint64_t bx = (words + 255) / 256;
    const uint64_t mx = (uint64_t)num_sms * 4 / G + 1;
    if (bx > mx) bx = mx;
    if (bx < 1) bx = 1;
    gather_rows_kernel<<<dim3((unsigned)bx, G), 256, 0, s>>>(src, src_off, me, G, row_bytes, dst,
                                                             dst_off, out_off);
}

void launch_gather_counts(const uint32_t* const* src_off, uint32_t me, uint32_t G, uint32_t* cnt,
                          cudaStream_t s) {
    gather_counts_kernel<<<1, 64, 0, s>>>(src_off, me, G, cnt);
}

void launch_local_combine(TableView local, const uint8_t* digest, const uint32_t* d_n,
                          uint64_t cap, uint32_t* slot_idx, uint32_t* rep, int num_sms,
                          cudaStream_t s, const TableView* d_local) {
    if (cap == 0) return;
    const unsigned g = grid_for(cap, 256, num_sms, 4);
    table_insert_kernel<<<g, 256, 0, s>>>(d_local, digest, nullptr, nullptr, d_n, 0, cap,
                                          slot_idx);
    combine_rep_kernel<<<g, 256, 0, s>>>(local, d_n, cap, slot_idx, rep);
    table_clear_used_kernel<<<g, 256, 0, s>>>(local, d_n, cap, slot_idx);
}

void launch_pack(const BatchDesc* d, const uint32_t* n_chunks, uint64_t cap, uint32_t max_items,
                 const uint32_t* chunk_start, const uint64_t* first_id, const uint8_t* digest,
                 const uint8_t* is_dup, const uint32_t* item_first_chunk,
                 const uint32_t* table_status, HostResultLayout h, int num_sms,
                 cudaStream_t s, const uint32_t* extra) {
    pack_kernel<<<grid_for(cap / 4 + max_items + 1, 256, 64, 1), 256, 0, s>>>(
        d, n_chunks, cap, chunk_start, first_id, digest, is_dup, item_first_chunk, table_status,
        h, extra);
}

}  // namespace dd
