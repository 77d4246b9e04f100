// dist.cpp -- rows A5-A8 at G > 1 in C++: the multi-GPU wave pipeline of
// SURVEY 8(e) with NCCL called directly (one process per GPU).
//
// Waves: in wave w every rank submits one batch.  Its local rows run on one
// of `depth` slots (each a ctx of its own for the op workspace, a stream and
// device buffers): A2-A4 chunk + SHA-1, A5 local combine + route by digest
// owner.  Right behind its local rows each wave exchanges its per-owner
// record counts on the owner stream (NCCL grouped send/recv of two u32 per
// peer) into pinned memory.  When `depth` waves are in flight, the oldest
// completes on the owner stream: the host reads its counts (the only
// synchronisation: it sizes the payload; the event was recorded `depth`
// waves ago, so it does not wait for newer owner work), the 32-byte records go to their owners (A6), the owner inserts
// then looks up all of them in its table shard (A7, dedup_op_owner), the
// first-occurrence ids go back (A8), are scattered to chunk order, and the
// results are copied to pinned host memory.  Owner work stays in wave order
// on one stream, so results are the sequential stream-order answer
// (reading O12) for any GPU count.  Every rank must call submit/complete in
// the same wave order (NCCL matches the grouped calls in order).
//
// This is the same protocol as dist.WavePipeline (Python), without the
// per-call interpreter overhead.
#include <cuda_runtime.h>
#include <nccl.h>

#include <chrono>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <deque>
#include <string>
#include <vector>

#include "dedup.h"

namespace {

struct DSlot {
    // ctx: its op-descriptor ring is used only by the first (warm-up) wave and
    // the graph captures, so the descriptors the graphs copy from are never
    // reused; ctx2 runs every uncaptured op after that (chunk_meta each wave).
    dedup_ctx* ctx = nullptr;
    dedup_ctx* ctx2 = nullptr;
    cudaStream_t s = nullptr;
    cudaEvent_t e_local = nullptr, e_done = nullptr;
    cudaEvent_t e_cnt = nullptr;  // the wave's counts exchange landed in h_cnt
    cudaEvent_t e_prod = nullptr;  // the producer stream's bytes are ready
    uint64_t cap = 0;
    uint32_t max_items = 0;
    // device
    uint32_t *cut = nullptr, *n = nullptr, *chunk_start = nullptr, *item_first = nullptr,
             *send_off = nullptr, *send_pos = nullptr, *rep = nullptr, *cnt_recv = nullptr;
    uint64_t *chunk_id = nullptr, *first_id = nullptr, *item_off = nullptr, *reply = nullptr,
             *reply_back = nullptr;
    uint8_t *digest = nullptr, *is_dup = nullptr;
    dedup_record *send = nullptr, *recv = nullptr;
    // pinned host
    uint64_t* h_off = nullptr;
    uint32_t* h_send_off = nullptr;  // [G + 1] then n
    uint32_t* h_cnt = nullptr;       // [G] received counts
    uint32_t* h_item_first = nullptr;
    uint32_t* h_chunk_start = nullptr;
    uint8_t* h_digest = nullptr;
    uint64_t* h_first_id = nullptr;
    uint8_t* h_is_dup = nullptr;
    // wave
    uint64_t first_seq = 0;
    uint32_t n_items = 0;
    uint32_t n_chunks = 0;
    bool busy = false;
    bool warm = false;  // one uncaptured wave done (lazy allocations inside the ops)
    // The local rows as two CUDA graphs per batch geometry (bytes, nbytes,
    // n_items): chunk (A2-A3), then chunk_meta uncaptured (its first_seq
    // changes every wave), then SHA-1 + local combine + route (A4-A5).
    struct G {
        const uint8_t* bytes;
        uint64_t nbytes;
        uint32_t n_items;
        cudaGraphExec_t g1, g2;
    };
    std::vector<G> graphs;
};

constexpr size_t kMaxGraphs = 8;  // per slot

}  // namespace

struct dedup_dist {
    ncclComm_t comm = nullptr;
    ncclComm_t ccomm = nullptr;  // counts exchange (split of comm), on stream cs
    cudaStream_t cs = nullptr;
    int nranks = 1, rank = 0, device = 0;
    dedup_ctx* owner = nullptr;
    cudaStream_t os = nullptr;  // owner stream
    std::vector<DSlot> slots;
    // table resets deferred by dedup_dist_end_stream with waves in flight:
    // each is issued on the owner stream right before the owner work of
    // the wave it names (the first wave of the next stream)
    std::deque<uint64_t> resets;
    uint32_t depth = 1;
    uint64_t next_wave = 0, done_wave = 0;
    int last_done = -1;  // slot of the last completed wave (results readable)
    bool use_graphs = true;  // DEDUP_DIST_GRAPHS=0: plain op calls
    bool early_counts = true;  // DEDUP_DIST_EARLY_COUNTS=0: counts exchanged at completion
    // metadata of the last completed wave (its slot is reused right away)
    uint64_t res_first_seq = 0;
    uint32_t res_n_items = 0, res_n_chunks = 0;
    std::vector<uint64_t> res_item_off;
    std::string err = "no error";
    // DEDUP_DIST_HOST_TIMING=1: host seconds spent in submit (issue) and in
    // the completion's wait for the counts, printed to stderr at destroy
    bool host_timing = false;
    double t_submit = 0, t_wait = 0, t_complete = 0, t_local = 0;
    uint64_t n_submit = 0;
};

namespace {

dedup_status dfail(dedup_dist* d, dedup_status st, const std::string& m) {
    if (d) d->err = m;
    return st;
}

#define DCU(x)                                                                       \
    do {                                                                             \
        cudaError_t e_ = (x);                                                        \
        if (e_ != cudaSuccess) return dfail(d, DEDUP_ECUDA, cudaGetErrorString(e_)); \
    } while (0)
#define DNC(x)                                                                         \
    do {                                                                               \
        ncclResult_t r_ = (x);                                                         \
        if (r_ != ncclSuccess) return dfail(d, DEDUP_ECUDA, ncclGetErrorString(r_)); \
    } while (0)
#define DTRY(x)                                                                      \
    do {                                                                             \
        dedup_status s_ = (x);                                                       \
        if (s_ != DEDUP_OK) return dfail(d, s_, dedup_last_error(sl.ctx));           \
    } while (0)

template <class T>
dedup_status dmalloc(dedup_dist* d, T** p, uint64_t n) {
    DCU(cudaMalloc(reinterpret_cast<void**>(p), sizeof(T) * (n ? n : 1)));
    return DEDUP_OK;
}
template <class T>
dedup_status hmalloc(dedup_dist* d, T** p, uint64_t n) {
    DCU(cudaHostAlloc(reinterpret_cast<void**>(p), sizeof(T) * (n ? n : 1), 0));
    return DEDUP_OK;
}

dedup_status slot_alloc(dedup_dist* d, DSlot& sl, const dedup_config& base, uint64_t batch_bytes,
                        uint32_t batch_items) {
    dedup_config c = base;
    c.batch_bytes = batch_bytes;
    c.batch_items = batch_items;
    c.slots = 1;
    c.host_fed = 0;
    c.table_capacity = 1024;  // the slot's own table is not used
    if (c.sha_lane_bytes == 0) c.sha_lane_bytes = 8192;
    dedup_status st = dedup_init(&c, &sl.ctx);
    if (st == DEDUP_OK) st = dedup_init(&c, &sl.ctx2);
    if (st != DEDUP_OK) return dfail(d, st, "dedup_init of a wave slot failed");
    const uint32_t G = (uint32_t)d->nranks;
    sl.cap = batch_bytes / 32 + batch_items + 2;
    sl.max_items = batch_items;
    DCU(cudaStreamCreateWithFlags(&sl.s, cudaStreamNonBlocking));
    DCU(cudaEventCreateWithFlags(&sl.e_local, cudaEventDisableTiming));
    DCU(cudaEventCreateWithFlags(&sl.e_done, cudaEventDisableTiming));
    DCU(cudaEventCreateWithFlags(&sl.e_cnt, cudaEventDisableTiming));
    DCU(cudaEventCreateWithFlags(&sl.e_prod, cudaEventDisableTiming));
    const uint64_t cap = sl.cap;
    if (dmalloc(d, &sl.cut, cap) || dmalloc(d, &sl.n, 1) || dmalloc(d, &sl.chunk_start, cap) ||
        dmalloc(d, &sl.item_first, batch_items + 1) || dmalloc(d, &sl.send_off, G + 1) ||
        dmalloc(d, &sl.send_pos, cap) || dmalloc(d, &sl.rep, cap) ||
        dmalloc(d, &sl.cnt_recv, 2 * G) ||
        dmalloc(d, &sl.chunk_id, cap) || dmalloc(d, &sl.first_id, cap) ||
        dmalloc(d, &sl.item_off, batch_items + 1) || dmalloc(d, &sl.reply, cap * G) ||
        dmalloc(d, &sl.reply_back, cap) || dmalloc(d, &sl.digest, cap * 20) ||
        dmalloc(d, &sl.is_dup, cap) || dmalloc(d, &sl.send, cap) ||
        dmalloc(d, &sl.recv, cap * G) || hmalloc(d, &sl.h_off, batch_items + 1) ||
        hmalloc(d, &sl.h_send_off, G + 2) || hmalloc(d, &sl.h_cnt, 2 * G) ||
        hmalloc(d, &sl.h_item_first, batch_items + 1) || hmalloc(d, &sl.h_chunk_start, cap) ||
        hmalloc(d, &sl.h_digest, cap * 20) || hmalloc(d, &sl.h_first_id, cap) ||
        hmalloc(d, &sl.h_is_dup, cap))
        return dfail(d, DEDUP_ENOMEM, "wave slot allocation failed");
    return DEDUP_OK;
}

void slot_free(DSlot& sl) {
    for (void* p : {(void*)sl.cut, (void*)sl.n, (void*)sl.chunk_start, (void*)sl.item_first,
                    (void*)sl.send_off, (void*)sl.send_pos, (void*)sl.rep, (void*)sl.cnt_recv, (void*)sl.chunk_id, (void*)sl.first_id,
                    (void*)sl.item_off, (void*)sl.reply, (void*)sl.reply_back, (void*)sl.digest,
                    (void*)sl.is_dup, (void*)sl.send, (void*)sl.recv})
        if (p) cudaFree(p);
    for (void* p : {(void*)sl.h_off, (void*)sl.h_send_off, (void*)sl.h_cnt,
                    (void*)sl.h_item_first, (void*)sl.h_chunk_start, (void*)sl.h_digest,
                    (void*)sl.h_first_id, (void*)sl.h_is_dup})
        if (p) cudaFreeHost(p);
    if (sl.e_local) cudaEventDestroy(sl.e_local);
    if (sl.e_done) cudaEventDestroy(sl.e_done);
    if (sl.e_cnt) cudaEventDestroy(sl.e_cnt);
    if (sl.e_prod) cudaEventDestroy(sl.e_prod);
    if (sl.s) cudaStreamDestroy(sl.s);
    for (auto& g : sl.graphs) {
        if (g.g1) cudaGraphExecDestroy(g.g1);
        if (g.g2) cudaGraphExecDestroy(g.g2);
    }
    if (sl.ctx) dedup_destroy(sl.ctx);
    if (sl.ctx2) dedup_destroy(sl.ctx2);
    sl = DSlot{};
}

// Row A6's first half, issued at submit time on the owner stream right after
// the wave's local rows: per-owner record counts -> every peer (peer p gets
// this rank's (send_off[p], send_off[p + 1]) and returns its own pair), then
// to pinned host memory.  complete_oldest waits only for this event, so the
// host never blocks on the owner stream's newest work (the previous wave's
// exchange, insert and D2H).  Every rank issues the same NCCL sequence.
dedup_status exchange_counts(dedup_dist* d, DSlot& sl) {
    const uint32_t G = (uint32_t)d->nranks;
    // early: own communicator and stream, so the owner stream (and through
    // e_done the next wave's slot) never waits for the newest local rows
    cudaStream_t st = d->early_counts ? d->cs : d->os;
    ncclComm_t cm = d->early_counts ? d->ccomm : d->comm;
    DCU(cudaStreamWaitEvent(st, sl.e_local, 0));
    DNC(ncclGroupStart());
    for (uint32_t p = 0; p < G; ++p) {
        DNC(ncclSend(sl.send_off + p, 2, ncclUint32, (int)p, cm, st));
        DNC(ncclRecv(sl.cnt_recv + 2 * p, 2, ncclUint32, (int)p, cm, st));
    }
    DNC(ncclGroupEnd());
    DCU(cudaMemcpyAsync(sl.h_cnt, sl.cnt_recv, sizeof(uint32_t) * 2 * G,
                        cudaMemcpyDeviceToHost, st));
    DCU(cudaEventRecord(sl.e_cnt, st));
    return DEDUP_OK;
}

// Completes the oldest wave in flight (rows A6-A8 + D2H on the owner stream).
dedup_status complete_oldest(dedup_dist* d) {
    const int i = (int)(d->done_wave % d->depth);
    DSlot& sl = d->slots[i];
    const uint32_t G = (uint32_t)d->nranks;
    cudaStream_t os = d->os;
    // the counts were exchanged when the wave was submitted (exchange_counts);
    // waiting for them does not wait for the owner stream's newer work
    while (!d->resets.empty() && d->resets.front() <= d->done_wave) {
        const dedup_status st = dedup_op_table_reset(d->owner, os);
        if (st != DEDUP_OK) return dfail(d, st, dedup_last_error(d->owner));
        d->resets.pop_front();
    }
    if (!d->early_counts) {
        const dedup_status st = exchange_counts(d, sl);
        if (st != DEDUP_OK) return st;
    }
    const auto tw0 = std::chrono::steady_clock::now();
    DCU(cudaEventSynchronize(sl.e_cnt));  // sizes of the payload (host); local rows done too
    if (d->host_timing)
        d->t_wait += std::chrono::duration<double>(std::chrono::steady_clock::now() - tw0).count();
    DCU(cudaStreamWaitEvent(os, sl.e_cnt, 0));  // the records (send) come from the local rows
    const uint32_t* soff = sl.h_send_off;
    sl.n_chunks = sl.h_send_off[G + 1];
    uint64_t roff = 0;
    std::vector<uint64_t> recv_off(G + 1, 0);
    std::vector<uint64_t> rcnt(G, 0);
    for (uint32_t p = 0; p < G; ++p) {
        recv_off[p] = roff;
        rcnt[p] = (uint64_t)sl.h_cnt[2 * p + 1] - sl.h_cnt[2 * p];
        roff += rcnt[p];
    }
    recv_off[G] = roff;
    if (roff > sl.cap * G) return dfail(d, DEDUP_ECUDA, "received records exceed the slot");
    // row A6: records to their owners
    DNC(ncclGroupStart());
    for (uint32_t p = 0; p < G; ++p) {
        const uint64_t ns = soff[p + 1] - soff[p], nr = rcnt[p];
        if (ns) DNC(ncclSend(sl.send + soff[p], ns * sizeof(dedup_record), ncclUint8, (int)p,
                             d->comm, os));
        if (nr) DNC(ncclRecv(sl.recv + recv_off[p], nr * sizeof(dedup_record), ncclUint8, (int)p,
                             d->comm, os));
    }
    DNC(ncclGroupEnd());
    // row A7 on this rank's shard
    if (roff) {
        const dedup_status st = dedup_op_owner(d->owner, os, sl.recv, roff, sl.reply);
        if (st != DEDUP_OK) return dfail(d, st, dedup_last_error(d->owner));
    }
    // row A8: replies back to the senders, then scatter to chunk order
    DNC(ncclGroupStart());
    for (uint32_t p = 0; p < G; ++p) {
        const uint64_t ns = soff[p + 1] - soff[p], nr = rcnt[p];
        if (nr) DNC(ncclSend(sl.reply + recv_off[p], nr, ncclUint64, (int)p, d->comm, os));
        if (ns) DNC(ncclRecv(sl.reply_back + soff[p], ns, ncclUint64, (int)p, d->comm, os));
    }
    DNC(ncclGroupEnd());
    const uint32_t n = sl.n_chunks;
    if (n) {
        const dedup_status st = dedup_op_scatter(sl.ctx, os, sl.reply_back, sl.send_pos, sl.rep,
                                                 sl.chunk_id, sl.n, sl.cap, sl.first_id,
                                                 sl.is_dup);
        if (st != DEDUP_OK) return dfail(d, st, dedup_last_error(sl.ctx));
    }
    // results to pinned host memory (row A9)
    DCU(cudaMemcpyAsync(sl.h_item_first, sl.item_first, sizeof(uint32_t) * sl.n_items,
                        cudaMemcpyDeviceToHost, os));
    if (n) {
        DCU(cudaMemcpyAsync(sl.h_chunk_start, sl.chunk_start, sizeof(uint32_t) * n,
                            cudaMemcpyDeviceToHost, os));
        DCU(cudaMemcpyAsync(sl.h_digest, sl.digest, 20ull * n, cudaMemcpyDeviceToHost, os));
        DCU(cudaMemcpyAsync(sl.h_first_id, sl.first_id, sizeof(uint64_t) * n,
                            cudaMemcpyDeviceToHost, os));
        DCU(cudaMemcpyAsync(sl.h_is_dup, sl.is_dup, n, cudaMemcpyDeviceToHost, os));
    }
    DCU(cudaEventRecord(sl.e_done, os));  // results readable after it (dedup_dist_result)
    sl.busy = false;
    d->last_done = i;
    d->res_first_seq = sl.first_seq;
    d->res_n_items = sl.n_items;
    d->res_n_chunks = n;
    d->res_item_off.assign(sl.h_off, sl.h_off + sl.n_items + 1);
    ++d->done_wave;
    return DEDUP_OK;
}

}  // namespace

extern "C" {

dedup_status dedup_nccl_unique_id(uint8_t out[128]) {
    static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId is 128 bytes");
    if (out == nullptr) return DEDUP_EINVAL;
    ncclUniqueId id;
    if (ncclGetUniqueId(&id) != ncclSuccess) return DEDUP_ECUDA;
    std::memcpy(out, &id, 128);
    return DEDUP_OK;
}

dedup_status dedup_dist_create(const dedup_config* cfg, const uint8_t nccl_id[128], int nranks,
                               int rank, uint32_t depth, uint64_t batch_bytes,
                               uint32_t batch_items, dedup_dist** out) {
    if (out == nullptr) return DEDUP_EINVAL;
    *out = nullptr;
    if (cfg == nullptr || nccl_id == nullptr || nranks < 1 || rank < 0 || rank >= nranks ||
        depth < 1 || depth > 64 || batch_bytes < 1 || batch_bytes > (1ull << 30) ||
        batch_items < 1 || (uint32_t)nranks != cfg->num_owners || (uint32_t)rank != cfg->owner_rank)
        return DEDUP_EINVAL;
    auto* d = new dedup_dist();
    d->nranks = nranks;
    d->rank = rank;
    d->depth = depth;
    d->device = cfg->device;
    if (const char* e = std::getenv("DEDUP_DIST_GRAPHS")) d->use_graphs = std::atoi(e) != 0;
    if (const char* e = std::getenv("DEDUP_DIST_EARLY_COUNTS")) d->early_counts = std::atoi(e) != 0;
    if (const char* e = std::getenv("DEDUP_DIST_HOST_TIMING")) d->host_timing = std::atoi(e) != 0;
    auto bail = [&](dedup_status st) {
        dedup_dist_destroy(d);
        return st;
    };
    if (cudaSetDevice(cfg->device) != cudaSuccess) return bail(DEDUP_ECUDA);
    // the owner ctx: this rank's table shard; it receives up to G batches' records
    dedup_config oc = *cfg;
    oc.slots = 1;
    oc.host_fed = 0;
    const uint64_t ob = batch_bytes * (uint64_t)nranks;
    oc.batch_bytes = ob < (1ull << 30) ? ob : (1ull << 30);
    oc.batch_items = 1;
    if (dedup_init(&oc, &d->owner) != DEDUP_OK) return bail(DEDUP_ENOMEM);
    if (cudaStreamCreateWithFlags(&d->os, cudaStreamNonBlocking) != cudaSuccess)
        return bail(DEDUP_ECUDA);
    ncclUniqueId id;
    std::memcpy(&id, nccl_id, 128);
    if (ncclCommInitRank(&d->comm, nranks, id, rank) != ncclSuccess) return bail(DEDUP_ECUDA);
    if (d->early_counts) {
        if (cudaStreamCreateWithFlags(&d->cs, cudaStreamNonBlocking) != cudaSuccess)
            return bail(DEDUP_ECUDA);
        if (ncclCommSplit(d->comm, 0, rank, &d->ccomm, nullptr) != ncclSuccess)
            return bail(DEDUP_ECUDA);
    }
    d->slots.resize(depth);
    for (auto& sl : d->slots)
        if (slot_alloc(d, sl, *cfg, batch_bytes, batch_items) != DEDUP_OK)
            return bail(DEDUP_ENOMEM);
    *out = d;
    return DEDUP_OK;
}

void dedup_dist_destroy(dedup_dist* d) {
    if (d == nullptr) return;
    if (d->host_timing && d->n_submit)
        std::fprintf(stderr,
                     "dedup_dist host timing: %llu submits, %.1f us/submit total, of which "
                     "%.1f us completing the oldest wave (%.1f us waiting for its counts), "
                     "%.1f us issuing the local rows\n",
                     (unsigned long long)d->n_submit, 1e6 * d->t_submit / d->n_submit,
                     1e6 * d->t_complete / d->n_submit, 1e6 * d->t_wait / d->n_submit,
                     1e6 * d->t_local / d->n_submit);
    cudaSetDevice(d->device);
    for (auto& sl : d->slots) slot_free(sl);
    if (d->ccomm) ncclCommDestroy(d->ccomm);
    if (d->comm) ncclCommDestroy(d->comm);
    if (d->cs) cudaStreamDestroy(d->cs);
    if (d->os) cudaStreamDestroy(d->os);
    if (d->owner) dedup_destroy(d->owner);
    delete d;
}

const char* dedup_dist_last_error(const dedup_dist* d) {
    return d ? d->err.c_str() : "null dist";
}

dedup_status dedup_dist_submit(dedup_dist* d, const uint8_t* d_bytes, uint64_t nbytes,
                               const uint64_t* item_off, uint32_t n_items, uint64_t first_seq,
                               void* producer, uint32_t* completed) {
    if (d == nullptr || item_off == nullptr || completed == nullptr) return DEDUP_EINVAL;
    *completed = 0;
    struct Timer {
        dedup_dist* d;
        std::chrono::steady_clock::time_point t0 = std::chrono::steady_clock::now();
        ~Timer() {
            if (!d->host_timing) return;
            d->t_submit +=
                std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
            ++d->n_submit;
        }
    } timer{d};
    if (cudaSetDevice(d->device) != cudaSuccess) return DEDUP_ECUDA;
    if (d->next_wave - d->done_wave >= d->depth) {
        const auto tc0 = std::chrono::steady_clock::now();
        const dedup_status st = complete_oldest(d);
        if (d->host_timing)
            d->t_complete +=
                std::chrono::duration<double>(std::chrono::steady_clock::now() - tc0).count();
        if (st != DEDUP_OK) return st;
        *completed = 1;
    }
    DSlot& sl = d->slots[d->next_wave % d->depth];
    if (n_items > sl.max_items || item_off[n_items] != nbytes)
        return dfail(d, DEDUP_EINVAL, "bad batch");
    // the slot's previous wave may still be copying its results out
    DCU(cudaStreamWaitEvent(sl.s, sl.e_done, 0));
    const uint32_t G = (uint32_t)d->nranks;
    sl.first_seq = first_seq;
    sl.n_items = n_items;
    std::memcpy(sl.h_off, item_off, sizeof(uint64_t) * (n_items + 1));
    // (the wait takes the event's state now, so the slot's event is reusable)
    DCU(cudaEventRecord(sl.e_prod, static_cast<cudaStream_t>(producer)));
    DCU(cudaStreamWaitEvent(sl.s, sl.e_prod, 0));
    DCU(cudaMemcpyAsync(sl.item_off, sl.h_off, sizeof(uint64_t) * (n_items + 1),
                        cudaMemcpyHostToDevice, sl.s));
    // rows A2-A5 on the slot's stream
    auto part1 = [&](dedup_ctx* c) -> dedup_status {
        return dedup_op_chunk(c, sl.s, d_bytes, nbytes, sl.item_off, n_items, sl.cut, sl.cap,
                              sl.n);
    };
    auto part2 = [&](dedup_ctx* c) -> dedup_status {
        dedup_status st = dedup_op_sha1(c, sl.s, d_bytes, nbytes, sl.cut, sl.n, sl.cap,
                                        sl.digest);
        if (st == DEDUP_OK) st = dedup_op_local_combine(c, sl.s, sl.digest, sl.n, sl.cap, sl.rep);
        if (st == DEDUP_OK)
            st = dedup_op_route(c, sl.s, sl.digest, sl.chunk_id, sl.n, sl.cap, sl.rep, G,
                                sl.send, sl.send_off, sl.send_pos);
        return st;
    };
    auto meta = [&](dedup_ctx* c) -> dedup_status {
        return dedup_op_chunk_meta(c, sl.s, sl.item_off, n_items, sl.cut, sl.n, sl.cap,
                                   first_seq, sl.chunk_start, sl.chunk_id, sl.item_first);
    };
    const auto tl0 = std::chrono::steady_clock::now();
    DSlot::G* g = nullptr;
    for (auto& x : sl.graphs)
        if (x.bytes == d_bytes && x.nbytes == nbytes && x.n_items == n_items) g = &x;
    if (g == nullptr && sl.warm && d->use_graphs && sl.graphs.size() < kMaxGraphs) {
        // capture both parts once for this geometry (on ctx)
        DSlot::G ng{d_bytes, nbytes, n_items, nullptr, nullptr};
        for (int part = 0; part < 2; ++part) {
            cudaGraph_t graph = nullptr;
            DCU(cudaStreamBeginCapture(sl.s, cudaStreamCaptureModeRelaxed));
            const dedup_status st = part == 0 ? part1(sl.ctx) : part2(sl.ctx);
            const cudaError_t ce = cudaStreamEndCapture(sl.s, &graph);
            if (st != DEDUP_OK) return dfail(d, st, dedup_last_error(sl.ctx));
            if (ce != cudaSuccess) return dfail(d, DEDUP_ECUDA, cudaGetErrorString(ce));
            DCU(cudaGraphInstantiate(part == 0 ? &ng.g1 : &ng.g2, graph, 0));
            cudaGraphDestroy(graph);
        }
        sl.graphs.push_back(ng);
        g = &sl.graphs.back();
    }
    if (g != nullptr) {
        DCU(cudaGraphLaunch(g->g1, sl.s));
        DTRY(meta(sl.ctx2));
        DCU(cudaGraphLaunch(g->g2, sl.s));
    } else {
        dedup_ctx* c = sl.warm ? sl.ctx2 : sl.ctx;  // ctx's ring: warm-up and captures only
        DTRY(part1(c));
        DTRY(meta(c));
        DTRY(part2(c));
        sl.warm = true;
    }
    if (d->host_timing)
        d->t_local += std::chrono::duration<double>(std::chrono::steady_clock::now() - tl0).count();
    // the per-owner offsets and n to pinned host memory (read at completion)
    DCU(cudaMemcpyAsync(sl.h_send_off, sl.send_off, sizeof(uint32_t) * (G + 1),
                        cudaMemcpyDeviceToHost, sl.s));
    DCU(cudaMemcpyAsync(sl.h_send_off + G + 1, sl.n, sizeof(uint32_t), cudaMemcpyDeviceToHost,
                        sl.s));
    DCU(cudaEventRecord(sl.e_local, sl.s));
    if (d->early_counts) {
        const dedup_status st = exchange_counts(d, sl);
        if (st != DEDUP_OK) return st;
    }
    sl.busy = true;
    ++d->next_wave;
    return DEDUP_OK;
}

dedup_status dedup_dist_flush(dedup_dist* d, uint32_t* completed) {
    if (d == nullptr || completed == nullptr) return DEDUP_EINVAL;
    *completed = 0;
    if (d->done_wave == d->next_wave) return DEDUP_OK;
    if (cudaSetDevice(d->device) != cudaSuccess) return DEDUP_ECUDA;
    const dedup_status st = complete_oldest(d);
    if (st == DEDUP_OK) *completed = 1;
    return st;
}

dedup_status dedup_dist_end_stream(dedup_dist* d) {
    if (d == nullptr) return DEDUP_EINVAL;
    if (d->done_wave != d->next_wave) {
        // waves of this stream still in flight: their owner work is issued in
        // wave order on the owner stream, so the reset goes in right before
        // the next stream's first wave (no drain of the pipeline)
        d->resets.push_back(d->next_wave);
        return DEDUP_OK;
    }
    if (cudaSetDevice(d->device) != cudaSuccess) return DEDUP_ECUDA;
    d->resets.clear();  // every deferred reset is subsumed by this one
    const dedup_status st = dedup_op_table_reset(d->owner, d->os);
    return st == DEDUP_OK ? st : dfail(d, st, dedup_last_error(d->owner));
}

dedup_status dedup_dist_last_counts(const dedup_dist* d, uint32_t* n_items, uint32_t* n_chunks,
                                    uint64_t* nbytes) {
    if (d == nullptr || d->last_done < 0) return DEDUP_EINVAL;
    if (n_items) *n_items = d->res_n_items;
    if (n_chunks) *n_chunks = d->res_n_chunks;
    if (nbytes) *nbytes = d->res_item_off.empty() ? 0 : d->res_item_off.back();
    return DEDUP_OK;
}

dedup_status dedup_dist_result(const dedup_dist* d, dedup_wave_result* out) {
    if (d == nullptr || out == nullptr || d->last_done < 0) return DEDUP_EINVAL;
    const DSlot& sl = d->slots[d->last_done];
    if (cudaEventSynchronize(sl.e_done) != cudaSuccess) return DEDUP_ECUDA;
    out->first_seq = d->res_first_seq;
    out->n_items = d->res_n_items;
    out->n_chunks = d->res_n_chunks;
    out->item_off = d->res_item_off.data();
    out->item_first_chunk = sl.h_item_first;
    out->chunk_start = sl.h_chunk_start;
    out->digest = sl.h_digest;
    out->first_id = sl.h_first_id;
    out->is_dup = sl.h_is_dup;
    return DEDUP_OK;
}

}  // extern "C"
