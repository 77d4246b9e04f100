// mg.cpp -- the multi-GPU engine: rows A2-A9 on G GPUs with the digest
// exchange of rows A5-A8.
//
// The paper's GPU Dedup takes batches round-robin over the GPUs (P:185,
// P:214), one host thread per device, and its last stage
// "reorders the batches".  Here batch b goes to rank b % G in wave
// b / G; the duplicate check is global (reading O11), so every digest has an
// owner rank (its BE32 prefix p: owner = floor(p G / 2^32)) holding that
// shard of the table.  Per wave and rank:
//   local rows (slot stream, ONE CUDA graph per slot, parameters from a
//   device descriptor): A2-A3 chunking, chunk metadata, A4 SHA-1, A5 local
//   combine (one record per distinct digest of the batch) + route by owner;
//   completion (owner stream, in wave order): A6 records to their owners,
//   A7 insert-all-then-lookup in the owner's shard, A8 first ids back to
//   the senders and scattered to chunk order, A9 results packed into mapped
//   pinned host memory.
// Owner work runs in wave order on one stream per rank, every record of a
// wave is inserted before any is looked up, and ids are (seq << 32) | index,
// so the table's minimum id is the first occurrence in stream order for any
// G (reading O12) -- the sequential answer.
//
// Two transports for A6/A8, selected per engine:
//   * NCCL: grouped ncclSend/ncclRecv; the per-owner counts are exchanged
//     right behind a wave's local rows on a second communicator (stream cs)
//     so that the completion (which needs the sizes on the host) waits only
//     for them.  Ordering: every rank issues the same sequence of calls on
//     each communicator (counts of wave w on ccomm at submit, records and
//     replies of wave w on comm at completion, both in wave order); the only
//     cross-communicator dependency is records(w) after counts(w) on every
//     rank, which is acyclic.
//   * copy (in-process): each rank PULLS its rows from every rank's buffers
//     with one gather kernel (peer loads over NVLink, or the loopback when
//     ranks share a GPU); offsets stay in device memory, so the completion
//     needs no host synchronisation.  Host barriers of the rank threads order
//     the events: all ranks submitted the wave; all owners looked up; all
//     pulls done (before any buffer of the wave is reused).
//   * p2p (in-process, transport 3): the exchange fused into the table
//     kernels -- a rank inserts its routed records straight into the owners'
//     shards (system-scope atomics on peer memory over NVLink, or the
//     loopback) and, once every rank's inserts of the wave are done, reads
//     its first ids back from them: no record or reply copies, 2 kernels per
//     wave instead of 4.  Barriers as for copy (all submitted + resets
//     issued; all inserted; all looked up).
// Uses: dedup_init with num_devices >= 2 (one process, one worker thread per
// rank, results merged in seq order by dedup_drain) and dedup_dist_* (one
// process per GPU, NCCL, driven by the caller's thread).
#include <cuda_runtime.h>
#include <nccl.h>

#include <atomic>
#include <chrono>
#include <condition_variable>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <deque>
#include <memory>
#include <mutex>
#include <string>
#include <thread>
#include <vector>

#include "dedup.h"
#include "internal.h"
#include "mg.h"

namespace dd {
namespace mg {
namespace {

using Clock = std::chrono::steady_clock;

uint64_t next_pow2(uint64_t v) {
    uint64_t p = 1;
    while (p < v) p <<= 1;
    return p;
}

// Host barrier of the rank threads of one process (copy transport).  A wait
// returns false once the engine aborted (a rank failed), so no thread stays
// blocked on a peer that will never arrive.
struct Barrier {
    std::mutex m;
    std::condition_variable cv;
    uint32_t n = 1, count = 0;
    uint64_t gen = 0;
    bool wait(const std::atomic<bool>& abort) {
        std::unique_lock<std::mutex> lk(m);
        const uint64_t g = gen;
        if (++count == n) {
            count = 0;
            ++gen;
            cv.notify_all();
            return !abort.load();
        }
        while (gen == g) {
            if (abort.load()) return false;
            cv.wait_for(lk, std::chrono::milliseconds(2));
        }
        return !abort.load();
    }
    void wake() { cv.notify_all(); }
};

// One in-flight wave of one rank.
struct Slot {
    cudaStream_t s = nullptr;
    cudaEvent_t e_local = nullptr, e_cnt = nullptr, e_done = nullptr, e_prod = nullptr;
    cudaEvent_t e_rep = nullptr;  // NCCL: this wave's replies are in (owner stream)
    cudaEvent_t e_a0 = nullptr, e_a1 = nullptr;  // exchange + owner phase (timed)
    cudaGraphExec_t graph = nullptr;
    BatchDesc *d_desc = nullptr, *h_desc = nullptr;
    uint64_t *d_item_off = nullptr, *h_item_off = nullptr;
    uint8_t* d_in = nullptr;  // host-fed input
    uint8_t* h_bounce = nullptr;  // page-locked bounce buffer for pageable items (lazy)
    // chunking / SHA-1 workspace (as the single-GPU engine's)
    uint32_t *bitmap = nullptr, *agg = nullptr, *gagg = nullptr, *gentry = nullptr,
             *evbuf = nullptr, *counters = nullptr, *slot_idx = nullptr, *sha_ws = nullptr,
             *mc_ws = nullptr;
    uint64_t max_tiles = 0, item_cap = 0;
    // per-chunk arrays
    uint32_t *cut = nullptr, *small = nullptr, *chunk_start = nullptr, *item_first = nullptr,
             *send_off = nullptr, *send_pos = nullptr, *rep = nullptr, *cnt_recv = nullptr,
             *route_scratch = nullptr;
    uint64_t *chunk_id = nullptr, *first_id = nullptr, *reply_back = nullptr;
    uint8_t *digest = nullptr, *is_dup = nullptr;
    dedup_record* send = nullptr;
    // local-combine table (row A5)
    TableSlot* lt = nullptr;
    uint32_t* lt_status = nullptr;
    TableView* d_lt = nullptr;
    uint64_t lt_cap = 0;
    // pinned host
    uint32_t* h_cnt = nullptr;   // [2G] (NCCL) received [begin, end) per source
    uint32_t* h_self = nullptr;  // [G + 2]: own send offsets, then n_chunks
    uint8_t* h_res = nullptr;    // mapped results
    HostResultLayout hdev{}, hhost{};
    // copy transport: device arrays of the peers' send buffers / offsets
    const uint8_t** p_rec_src = nullptr;
    const uint32_t** p_rec_off = nullptr;
    // ---- the batch (written by the submitting thread before SUBMIT) ----
    uint64_t wave = ~0ull, first_seq = 0, nbytes = 0;
    uint32_t n_items = 0;
    const uint8_t* d_bytes = nullptr;  // device-resident input (nullptr: host-fed)
    struct Range {
        const uint8_t* src;
        uint64_t dst, len;
    };
    std::vector<Range> h2d;            // host-fed copies
    cudaEvent_t e_prod_foreign = nullptr;  // producer on another device (owned)
    std::vector<uint64_t> item_len;
    bool timed = false;
    // ---- completion / results ----
    std::atomic<uint64_t> done_wave{~0ull};  // set after e_done is recorded for `wave`
    bool busy = false, parsed = false;
    uint32_t next_item = 0, n_chunks = 0;
    std::vector<uint32_t> item_first_v, item_n;
};

struct Engine;

struct Rank {
    Engine* E = nullptr;
    uint32_t me = 0;  // global rank
    int dev = 0;
    int num_sms = 0;
    uint32_t* d_rtab = nullptr;
    std::vector<std::unique_ptr<Slot>> slots;
    cudaStream_t os = nullptr, cs = nullptr;
    cudaEvent_t e_rdy = nullptr, e_fin = nullptr;
    ncclComm_t comm = nullptr, ccomm = nullptr;
    // owner shard (row A7)
    TableSlot* tab = nullptr;
    uint32_t* tab_status = nullptr;
    TableView* d_tabv = nullptr;
    TableView* d_views = nullptr;  // p2p: the G owners' shards (peer memory)
    cudaEvent_t e_rst = nullptr;   // p2p: this wave's table resets issued
    uint64_t tab_cap = 0;
    dedup_record* recv = nullptr;
    uint64_t* reply = nullptr;
    uint32_t *roff = nullptr, *o_slot_idx = nullptr;
    const uint8_t** p_rep_src = nullptr;
    const uint32_t** p_rep_off = nullptr;
    std::deque<uint64_t> resets;  // deferred table resets: before the owner work of wave x
    uint64_t next_wave = 0, done_wave = 0;
    uint64_t timed_waves = 0;
};

struct Engine {
    dedup_config cfg{};
    uint32_t G = 1, depth = 1;  // depth: waves in flight (dist) / slots (ctx)
    uint32_t nslots = 1;        // slots per rank (dist: depth + 1, so a completed wave's
                                // results stay readable while the next one is submitted)
    bool copy = false, host_fed = false;
    bool p2p = false;  // transport 3: remote insert / lookup on the owners' shards
    uint64_t batch_bytes = 0, cap = 0;
    uint32_t batch_items = 0, lane_bytes = 16384, time_every = 1;
    std::vector<std::unique_ptr<Rank>> ranks;  // local ranks
    Barrier bar;
    std::atomic<bool> abort{false};
    std::mutex err_mu;
    std::string err = "no error";
    std::atomic<int> sticky{0};
    std::atomic<uint64_t> launches{0};
    std::atomic<uint64_t> a2a_sent{0};  // NCCL: record + reply bytes sent to other ranks
    uint32_t graph_kernels = 0;
    double timeout_s = 600.0;
    // DEDUP_MG_PROFILE=1: host seconds per section of the NCCL wave path,
    // printed to stderr when the engine is destroyed (kProf* below)
    bool profile = false;
    bool nccl_self = false;  // DEDUP_MG_NCCL_SELF: the own share through NCCL too
    double prof[8] = {0, 0, 0, 0, 0, 0, 0, 0};
    uint64_t prof_n[8] = {0, 0, 0, 0, 0, 0, 0, 0};

    dedup_status fail(dedup_status st, const std::string& m) {
        {
            std::lock_guard<std::mutex> lk(err_mu);
            if (sticky.load() == 0) {
                sticky.store(st);
                err = m;
            }
        }
        abort.store(true);
        bar.wake();
        if (st == DEDUP_ENCCL || st == DEDUP_ECUDA)
            for (auto& r : ranks) {  // unblock the peers' collectives
                if (r->comm) ncclCommAbort(r->comm), r->comm = nullptr;
                if (r->ccomm) ncclCommAbort(r->ccomm), r->ccomm = nullptr;
            }
        return st;
    }
    std::string error() {
        std::lock_guard<std::mutex> lk(err_mu);
        return err;
    }
    ~Engine();
};

enum { kProfLocal, kProfCounts, kProfWaitCnt, kProfRecords, kProfOwner, kProfReplies,
       kProfFinish, kProfSubmit };
struct ProfScope {  // accumulates the scope's host time into E->prof[i]
    Engine* E;
    int i;
    Clock::time_point t0;
    ProfScope(Engine* e, int k) : E(e), i(k) {
        if (E->profile) t0 = Clock::now();
    }
    ~ProfScope() {
        if (!E->profile) return;
        E->prof[i] += std::chrono::duration<double>(Clock::now() - t0).count();
        E->prof_n[i] += 1;
    }
};

#define MCU(x)                                                                        \
    do {                                                                              \
        cudaError_t e_ = (x);                                                         \
        if (e_ != cudaSuccess)                                                        \
            return E->fail(DEDUP_ECUDA, std::string(#x ": ") + cudaGetErrorString(e_)); \
    } while (0)
#define MNC(x)                                                                        \
    do {                                                                              \
        ncclResult_t r_ = (x);                                                        \
        if (r_ != ncclSuccess)                                                        \
            return E->fail(DEDUP_ENCCL, std::string(#x ": ") + ncclGetErrorString(r_)); \
    } while (0)
#define MTRY(x)                        \
    do {                               \
        dedup_status s_ = (x);         \
        if (s_ != DEDUP_OK) return s_; \
    } while (0)

template <class T>
dedup_status dmalloc(Engine* E, T** p, uint64_t n) {
    cudaError_t e = cudaMalloc(reinterpret_cast<void**>(p), sizeof(T) * (n ? n : 1));
    if (e != cudaSuccess) return E->fail(DEDUP_ENOMEM, std::string("cudaMalloc: ") +
                                                           cudaGetErrorString(e));
    return DEDUP_OK;
}
template <class T>
dedup_status hmalloc(Engine* E, T** p, uint64_t n, unsigned flags = cudaHostAllocPortable) {
    cudaError_t e = cudaHostAlloc(reinterpret_cast<void**>(p), sizeof(T) * (n ? n : 1), flags);
    if (e != cudaSuccess) return E->fail(DEDUP_ENOMEM, std::string("cudaHostAlloc: ") +
                                                           cudaGetErrorString(e));
    return DEDUP_OK;
}

void slot_free(Slot& sl) {
    if (sl.s) cudaStreamSynchronize(sl.s);
    if (sl.graph) cudaGraphExecDestroy(sl.graph);
    for (cudaEvent_t e : {sl.e_local, sl.e_cnt, sl.e_done, sl.e_prod, sl.e_rep, sl.e_a0, sl.e_a1,
                          sl.e_prod_foreign})
        if (e) cudaEventDestroy(e);
    for (void* p : {(void*)sl.d_desc, (void*)sl.d_item_off, (void*)sl.d_in, (void*)sl.bitmap,
                    (void*)sl.agg, (void*)sl.gagg, (void*)sl.gentry, (void*)sl.evbuf,
                    (void*)sl.counters, (void*)sl.slot_idx, (void*)sl.sha_ws, (void*)sl.mc_ws,
                    (void*)sl.cut, (void*)sl.small, (void*)sl.chunk_start, (void*)sl.item_first,
                    (void*)sl.send_off, (void*)sl.send_pos, (void*)sl.rep, (void*)sl.cnt_recv,
                    (void*)sl.route_scratch, (void*)sl.chunk_id, (void*)sl.first_id,
                    (void*)sl.reply_back, (void*)sl.digest, (void*)sl.is_dup, (void*)sl.send,
                    (void*)sl.lt, (void*)sl.lt_status, (void*)sl.d_lt, (void*)sl.p_rec_src,
                    (void*)sl.p_rec_off})
        if (p) cudaFree(p);
    for (void* p : {(void*)sl.h_desc, (void*)sl.h_item_off, (void*)sl.h_cnt, (void*)sl.h_self,
                    (void*)sl.h_res, (void*)sl.h_bounce})
        if (p) cudaFreeHost(p);
    if (sl.s) cudaStreamDestroy(sl.s);
}

void rank_free(Rank& r) {
    cudaSetDevice(r.dev);
    if (r.os) cudaStreamSynchronize(r.os);
    if (r.cs) cudaStreamSynchronize(r.cs);
    for (auto& sl : r.slots) slot_free(*sl);
    r.slots.clear();
    if (r.ccomm) ncclCommDestroy(r.ccomm);
    if (r.comm) ncclCommDestroy(r.comm);
    for (cudaEvent_t e : {r.e_rdy, r.e_fin, r.e_rst})
        if (e) cudaEventDestroy(e);
    for (void* p : {(void*)r.d_rtab, (void*)r.tab, (void*)r.tab_status, (void*)r.d_tabv,
                    (void*)r.d_views,
                    (void*)r.recv, (void*)r.reply, (void*)r.roff, (void*)r.o_slot_idx,
                    (void*)r.p_rep_src, (void*)r.p_rep_off})
        if (p) cudaFree(p);
    if (r.os) cudaStreamDestroy(r.os);
    if (r.cs) cudaStreamDestroy(r.cs);
}

void prof_dump(Engine* E) {  // DEDUP_MG_PROFILE: print and reset
    if (!E->profile || E->prof_n[kProfSubmit] + E->prof_n[kProfLocal] == 0) return;
    static const char* names[8] = {"local rows", "counts exchange", "wait counts", "records",
                                   "owner", "replies", "finish", "submit call"};
    for (int i = 0; i < 8; ++i) {
        if (E->prof_n[i])
            std::fprintf(stderr, "mg profile: %-16s %8llu calls %8.1f us/call\n", names[i],
                         (unsigned long long)E->prof_n[i], 1e6 * E->prof[i] / E->prof_n[i]);
        E->prof[i] = 0;
        E->prof_n[i] = 0;
    }
}

Engine::~Engine() {
    prof_dump(this);
    for (auto& r : ranks) rank_free(*r);
}

// Records the local-row graph of a slot (A2-A5 + the counts to pinned memory).
dedup_status capture_local(Engine* E, Rank& r, Slot& sl) {
    const dedup_config& c = E->cfg;
    cudaStream_t s = sl.s;
    MCU(cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal));
    cudaMemcpyAsync(sl.d_desc, sl.h_desc, sizeof(BatchDesc), cudaMemcpyHostToDevice, s);
    cudaMemcpyAsync(sl.d_item_off, sl.h_item_off, sizeof(uint64_t) * (E->batch_items + 1),
                    cudaMemcpyHostToDevice, s);
    cudaMemsetAsync(sl.small, 0, sizeof(uint32_t) * 16, s);
    launch_chunk_select(sl.d_desc, r.d_rtab, c.anchor_mask, c.anchor_value, sl.bitmap, sl.agg,
                        sl.gagg, sl.gentry, sl.evbuf, sl.max_tiles, sl.cut, E->cap, sl.small,
                        r.num_sms, s, nullptr, c.max_chunk, sl.mc_ws, (uint32_t)sl.item_cap,
                        c.min_chunk);
    launch_chunk_meta(sl.d_desc, sl.cut, sl.small, E->cap, sl.chunk_start, sl.chunk_id,
                      sl.item_first, E->batch_items, r.num_sms, s);
    launch_sha1(sl.d_desc, E->batch_bytes, sl.cut, sl.small, E->cap, sl.sha_ws, sl.digest,
                r.num_sms, s, E->lane_bytes);
    const TableView lv{sl.lt, sl.lt_cap - 1, sl.lt_status};
    launch_local_combine(lv, sl.digest, sl.small, E->cap, sl.slot_idx, sl.rep, r.num_sms, s,
                         sl.d_lt);
    launch_route(sl.digest, sl.chunk_id, sl.small, E->cap, sl.rep, E->G, sl.send, sl.send_off,
                 sl.send_pos, sl.route_scratch, r.num_sms, s);
    cudaMemcpyAsync(sl.h_self, sl.send_off, sizeof(uint32_t) * (E->G + 1),
                    cudaMemcpyDeviceToHost, s);
    cudaMemcpyAsync(sl.h_self + E->G + 1, sl.small, sizeof(uint32_t), cudaMemcpyDeviceToHost, s);
    cudaEventRecordWithFlags(sl.e_local, s, cudaEventRecordExternal);
    cudaGraph_t g = nullptr;
    cudaError_t e = cudaStreamEndCapture(s, &g);
    if (e != cudaSuccess)
        return E->fail(DEDUP_ECUDA, std::string("local-row capture: ") + cudaGetErrorString(e));
    size_t nn = 0;
    cudaGraphGetNodes(g, nullptr, &nn);
    std::vector<cudaGraphNode_t> nodes(nn);
    cudaGraphGetNodes(g, nodes.data(), &nn);
    uint32_t k = 0;
    for (auto& nd : nodes) {
        cudaGraphNodeType ty;
        cudaGraphNodeGetType(nd, &ty);
        k += ty == cudaGraphNodeTypeKernel ? 1 : 0;
    }
    E->graph_kernels = k;
    e = cudaGraphInstantiate(&sl.graph, g, 0);
    cudaGraphDestroy(g);
    if (e != cudaSuccess)
        return E->fail(DEDUP_ECUDA, std::string("graph instantiate: ") + cudaGetErrorString(e));
    MCU(cudaGraphUpload(sl.graph, s));
    return DEDUP_OK;
}

dedup_status slot_alloc(Engine* E, Rank& r, Slot& sl) {
    const uint64_t cap = E->cap, bb = E->batch_bytes;
    const uint32_t G = E->G, bi = E->batch_items;
    MCU(cudaStreamCreateWithFlags(&sl.s, cudaStreamNonBlocking));
    for (cudaEvent_t* e : {&sl.e_local, &sl.e_cnt, &sl.e_done, &sl.e_prod, &sl.e_rep})
        MCU(cudaEventCreateWithFlags(e, cudaEventDisableTiming));
    MCU(cudaEventCreate(&sl.e_a0));
    MCU(cudaEventCreate(&sl.e_a1));
    MTRY(dmalloc(E, &sl.d_desc, 1));
    MTRY(hmalloc(E, &sl.h_desc, 1));
    std::memset(sl.h_desc, 0, sizeof(BatchDesc));
    MTRY(dmalloc(E, &sl.d_item_off, bi + 1));
    MTRY(hmalloc(E, &sl.h_item_off, bi + 1));
    std::memset(sl.h_item_off, 0, sizeof(uint64_t) * (bi + 1));
    if (E->host_fed) MTRY(dmalloc(E, &sl.d_in, bb + 256));
    sl.max_tiles = (bb + kSelTile - 1) / kSelTile + 1;
    MTRY(dmalloc(E, &sl.bitmap, sl.max_tiles * kSelTileWords + 2));  // whole tiles
    MTRY(dmalloc(E, &sl.agg, sl.max_tiles * 32));
    MTRY(dmalloc(E, &sl.gagg, (select_groups(sl.max_tiles) + 1) * 32));
    MTRY(dmalloc(E, &sl.gentry, (select_groups(sl.max_tiles) + 1) * 2));
    MTRY(dmalloc(E, &sl.evbuf, event_words(sl.max_tiles)));
    MTRY(dmalloc(E, &sl.counters, 256));
    MCU(cudaMemset(sl.counters, 0, sizeof(uint32_t) * 256));
    MTRY(dmalloc(E, &sl.slot_idx, cap));
    MTRY(dmalloc(E, &sl.sha_ws, sha1_ws_words(cap)));
    if (E->cfg.max_chunk || E->cfg.min_chunk != 32) {
        sl.item_cap = cap;
        MTRY(dmalloc(E, &sl.mc_ws, maxchunk_ws_words(cap, sl.item_cap)));
    }
    MTRY(dmalloc(E, &sl.cut, cap));
    MTRY(dmalloc(E, &sl.small, 16));
    MTRY(dmalloc(E, &sl.chunk_start, cap));
    MTRY(dmalloc(E, &sl.item_first, bi + 1));
    MTRY(dmalloc(E, &sl.send_off, G + 1));
    MTRY(dmalloc(E, &sl.send_pos, cap));
    MTRY(dmalloc(E, &sl.rep, cap));
    MTRY(dmalloc(E, &sl.cnt_recv, 2 * G));
    MTRY(dmalloc(E, &sl.route_scratch, 128));
    MTRY(dmalloc(E, &sl.chunk_id, cap));
    MTRY(dmalloc(E, &sl.first_id, cap));
    MTRY(dmalloc(E, &sl.reply_back, cap));
    MTRY(dmalloc(E, &sl.digest, cap * 20));
    MTRY(dmalloc(E, &sl.is_dup, cap));
    MTRY(dmalloc(E, &sl.send, cap));
    sl.lt_cap = next_pow2(2 * cap);
    MTRY(dmalloc(E, &sl.lt, sl.lt_cap));
    MTRY(dmalloc(E, &sl.lt_status, 4));
    MTRY(dmalloc(E, &sl.d_lt, 1));
    MCU(cudaMemset(sl.lt, 0, sizeof(TableSlot) * sl.lt_cap));
    MCU(cudaMemset(sl.lt_status, 0, 16));
    const TableView lv{sl.lt, sl.lt_cap - 1, sl.lt_status};
    MCU(cudaMemcpy(sl.d_lt, &lv, sizeof(lv), cudaMemcpyHostToDevice));
    MTRY(hmalloc(E, &sl.h_cnt, 2 * G));
    MTRY(hmalloc(E, &sl.h_self, G + 2));
    std::memset(sl.h_self, 0, sizeof(uint32_t) * (G + 2));
    // results: header 64 B | chunk_start 4 cap | first_id 8 cap | digest 20 cap | is_dup cap
    //          | item_first 4 items
    const uint64_t o_cs = 64, o_fid = o_cs + ((4 * cap + 63) & ~63ull), o_dg = o_fid + 8 * cap,
                   o_dup = o_dg + 20 * cap, o_if = (o_dup + cap + 63) & ~63ull,
                   total = o_if + 4ull * bi + 64;
    MTRY(hmalloc(E, &sl.h_res, total, cudaHostAllocMapped | cudaHostAllocPortable));
    uint8_t* dres = nullptr;
    MCU(cudaHostGetDevicePointer(reinterpret_cast<void**>(&dres), sl.h_res, 0));
    auto lay = [&](uint8_t* b) {
        HostResultLayout h;
        h.header = reinterpret_cast<uint32_t*>(b);
        h.chunk_start = reinterpret_cast<uint32_t*>(b + o_cs);
        h.first_id = reinterpret_cast<uint64_t*>(b + o_fid);
        h.digest = b + o_dg;
        h.is_dup = b + o_dup;
        h.item_first_chunk = reinterpret_cast<uint32_t*>(b + o_if);
        return h;
    };
    sl.hdev = lay(dres);
    sl.hhost = lay(sl.h_res);
    if (E->copy) {
        MTRY(dmalloc(E, &sl.p_rec_src, G));
        MTRY(dmalloc(E, &sl.p_rec_off, G));
    }
    return capture_local(E, r, sl);
}

dedup_status rank_alloc(Engine* E, Rank& r, uint64_t shard_capacity) {
    MCU(cudaSetDevice(r.dev));
    MCU(cudaDeviceGetAttribute(&r.num_sms, cudaDevAttrMultiProcessorCount, r.dev));
    set_pipeline_carveout();
    if (const char* bad = chunk_unlaunchable())
        return E->fail(DEDUP_ECUDA, std::string(bad) + " cannot launch");
    if (const char* bad = sha1_unlaunchable())
        return E->fail(DEDUP_ECUDA, std::string(bad) + " cannot launch");
    uint32_t tab[512];
    rabin_tables(E->cfg.poly, tab);
    MTRY(dmalloc(E, &r.d_rtab, 512));
    MCU(cudaMemcpy(r.d_rtab, tab, sizeof(tab), cudaMemcpyHostToDevice));
    // the owner stream is serial across waves (exchange + table work), the
    // counts gate the host: both at the highest priority, so that their small
    // kernels take SMs ahead of the next waves' scan / SHA-1 CTAs
    int prio_lo = 0, prio_hi = 0;
    MCU(cudaDeviceGetStreamPriorityRange(&prio_lo, &prio_hi));
    MCU(cudaStreamCreateWithPriority(&r.os, cudaStreamNonBlocking, prio_hi));
    MCU(cudaStreamCreateWithPriority(&r.cs, cudaStreamNonBlocking, prio_hi));
    MCU(cudaEventCreateWithFlags(&r.e_rdy, cudaEventDisableTiming));
    MCU(cudaEventCreateWithFlags(&r.e_fin, cudaEventDisableTiming));
    MCU(cudaEventCreateWithFlags(&r.e_rst, cudaEventDisableTiming));
    r.tab_cap = next_pow2(2 * shard_capacity);
    MTRY(dmalloc(E, &r.tab, r.tab_cap));
    MTRY(dmalloc(E, &r.tab_status, 4));
    MTRY(dmalloc(E, &r.d_tabv, 1));
    MCU(cudaMemset(r.tab, 0, sizeof(TableSlot) * r.tab_cap));
    MCU(cudaMemset(r.tab_status, 0, 16));
    const TableView tv{r.tab, r.tab_cap - 1, r.tab_status};
    MCU(cudaMemcpy(r.d_tabv, &tv, sizeof(tv), cudaMemcpyHostToDevice));
    // an owner receives at most every rank's whole batch (distinct digests)
    // (p2p: no records or replies are copied; o_slot_idx holds the rank's
    // own records' slots between its insert and lookup)
    const uint64_t rcap = E->cap * E->G;
    if (!E->p2p) {
        MTRY(dmalloc(E, &r.recv, rcap));
        MTRY(dmalloc(E, &r.reply, rcap));
    }
    MTRY(dmalloc(E, &r.o_slot_idx, E->p2p ? E->cap : rcap));
    MTRY(dmalloc(E, &r.roff, E->G + 1));
    MCU(cudaMemset(r.roff, 0, sizeof(uint32_t) * (E->G + 1)));
    if (E->copy) {
        MTRY(dmalloc(E, &r.p_rep_src, E->G));
        MTRY(dmalloc(E, &r.p_rep_off, E->G));
    }
    if (E->p2p) MTRY(dmalloc(E, &r.d_views, E->G));
    r.slots.resize(E->nslots);
    for (auto& sl : r.slots) {
        sl.reset(new Slot());
        MTRY(slot_alloc(E, r, *sl));
    }
    MCU(cudaDeviceSynchronize());
    return DEDUP_OK;
}

// Copy transport: every rank's pointer arrays to the peers' buffers.
dedup_status wire_copy(Engine* E) {
    const uint32_t G = E->G;
    for (auto& rp : E->ranks) {
        Rank& r = *rp;
        MCU(cudaSetDevice(r.dev));
        std::vector<const void*> a(G), b(G);
        for (uint32_t s = 0; s < G; ++s) {
            a[s] = E->ranks[s]->reply;
            b[s] = E->ranks[s]->roff;
        }
        MCU(cudaMemcpy(r.p_rep_src, a.data(), sizeof(void*) * G, cudaMemcpyHostToDevice));
        MCU(cudaMemcpy(r.p_rep_off, b.data(), sizeof(void*) * G, cudaMemcpyHostToDevice));
        if (E->p2p) {  // every owner's shard, as this rank's kernels address it
            std::vector<TableView> v(G);
            for (uint32_t s = 0; s < G; ++s)
                v[s] = TableView{E->ranks[s]->tab, E->ranks[s]->tab_cap - 1,
                                 E->ranks[s]->tab_status};
            MCU(cudaMemcpy(r.d_views, v.data(), sizeof(TableView) * G, cudaMemcpyHostToDevice));
        }
        for (uint32_t i = 0; i < E->nslots; ++i) {
            for (uint32_t s = 0; s < G; ++s) {
                a[s] = E->ranks[s]->slots[i]->send;
                b[s] = E->ranks[s]->slots[i]->send_off;
            }
            Slot& sl = *r.slots[i];
            MCU(cudaMemcpy(sl.p_rec_src, a.data(), sizeof(void*) * G, cudaMemcpyHostToDevice));
            MCU(cudaMemcpy(sl.p_rec_off, b.data(), sizeof(void*) * G, cudaMemcpyHostToDevice));
        }
    }
    return DEDUP_OK;
}

// Host wait for an event of rank r, polling NCCL's asynchronous errors.
dedup_status wait_event(Engine* E, Rank& r, cudaEvent_t e) {
    const auto t0 = Clock::now();
    for (uint32_t spin = 0;; ++spin) {
        const cudaError_t q = cudaEventQuery(e);
        if (q == cudaSuccess) return DEDUP_OK;
        if (q != cudaErrorNotReady)
            return E->fail(DEDUP_ECUDA, std::string("wave failed: ") + cudaGetErrorString(q));
        if (E->abort.load()) return (dedup_status)E->sticky.load();
        for (ncclComm_t cm : {r.comm, r.ccomm}) {
            if (cm == nullptr) continue;
            ncclResult_t ar = ncclSuccess;
            if (ncclCommGetAsyncError(cm, &ar) == ncclSuccess && ar != ncclSuccess &&
                ar != ncclInProgress)
                return E->fail(DEDUP_ENCCL, std::string("NCCL: ") + ncclGetErrorString(ar));
        }
        if (std::chrono::duration<double>(Clock::now() - t0).count() > E->timeout_s)
            return E->fail(DEDUP_ENCCL, "timed out waiting for a peer of the exchange");
        if (spin > 64) std::this_thread::sleep_for(std::chrono::microseconds(20));
    }
}

// ---- local rows of wave w on rank r (the batch is already in the slot) ----
dedup_status rank_submit(Engine* E, Rank& r, uint64_t w) {
    Slot& sl = *r.slots[w % E->nslots];
    const uint32_t G = E->G;
    MCU(cudaSetDevice(r.dev));
    MCU(cudaStreamWaitEvent(sl.s, sl.e_done, 0));  // the slot's previous wave is out
    if (sl.d_bytes == nullptr) {
        for (const Slot::Range& g : sl.h2d)
            if (g.len)
                MCU(cudaMemcpyAsync(sl.d_in + g.dst, g.src, g.len, cudaMemcpyHostToDevice, sl.s));
    } else {
        MCU(cudaStreamWaitEvent(sl.s, sl.e_prod_foreign ? sl.e_prod_foreign : sl.e_prod, 0));
        if (sl.e_prod_foreign) {
            cudaEventDestroy(sl.e_prod_foreign);
            sl.e_prod_foreign = nullptr;
        }
    }
    {
        ProfScope ps(E, kProfLocal);
        MCU(cudaGraphLaunch(sl.graph, sl.s));
    }
    E->launches += E->graph_kernels;
    if (!E->copy) {
        ProfScope ps(E, kProfCounts);
        // counts of this wave to every peer right behind its local rows (ccomm, cs)
        MCU(cudaStreamWaitEvent(r.cs, sl.e_local, 0));
        // (the rank's own share is a device copy: no NCCL kernel for it,
        // unless DEDUP_MG_NCCL_SELF -- the tests' way to drive the NCCL calls
        // at world size 1)
        if (!E->nccl_self)
            MCU(cudaMemcpyAsync(sl.cnt_recv + 2 * r.me, sl.send_off + r.me,
                                2 * sizeof(uint32_t), cudaMemcpyDeviceToDevice, r.cs));
        if (G > 1 || E->nccl_self) {
            MNC(ncclGroupStart());
            for (uint32_t p = 0; p < G; ++p) {
                if (p == r.me && !E->nccl_self) continue;
                MNC(ncclSend(sl.send_off + p, 2, ncclUint32, (int)p, r.ccomm, r.cs));
                MNC(ncclRecv(sl.cnt_recv + 2 * p, 2, ncclUint32, (int)p, r.ccomm, r.cs));
            }
            MNC(ncclGroupEnd());
        }
        MCU(cudaMemcpyAsync(sl.h_cnt, sl.cnt_recv, sizeof(uint32_t) * 2 * G,
                            cudaMemcpyDeviceToHost, r.cs));
        MCU(cudaEventRecord(sl.e_cnt, r.cs));
    }
    ++r.next_wave;
    return DEDUP_OK;
}

dedup_status owner_work(Engine* E, Rank& r, const uint32_t* d_n, uint64_t n_host, uint64_t cap) {
    launch_table_insert(r.d_tabv, nullptr, nullptr, r.recv, d_n, n_host, cap, r.o_slot_idx,
                        r.num_sms, r.os);
    launch_table_lookup(r.d_tabv, nullptr, r.recv, d_n, n_host, cap, r.o_slot_idx, r.reply,
                        nullptr, nullptr, nullptr, nullptr, r.num_sms, r.os);
    E->launches += 2;
    MCU(cudaGetLastError());
    return DEDUP_OK;
}

// Rows A8 (scatter of the replies) and A9 (pack to pinned host memory) of a
// wave.  The shard's overflow flag and used slots are copied on the owner
// stream (before a later wave's reset can clear them) -> small[4..5]; a
// reply of ~0 (any owner overflowed) also sets small[4] (scatter).  With
// on_slot the scatter and pack run on the slot's stream behind the wave's
// replies, so the owner stream -- serial across waves -- carries only the
// exchange and the table work.
dedup_status finish(Engine* E, Rank& r, Slot& sl, bool on_slot = false) {
    MCU(cudaMemcpyAsync(sl.small + 4, r.tab_status, 2 * sizeof(uint32_t),
                        cudaMemcpyDeviceToDevice, r.os));
    cudaStream_t st = r.os;
    if (on_slot) {
        if (sl.timed) MCU(cudaEventRecord(sl.e_a1, r.os));
        MCU(cudaEventRecord(sl.e_rep, r.os));
        MCU(cudaStreamWaitEvent(sl.s, sl.e_rep, 0));
        st = sl.s;
    }
    launch_scatter(sl.reply_back, sl.send_pos, sl.rep, sl.chunk_id, sl.small, E->cap,
                   sl.first_id, sl.is_dup, r.num_sms, st, sl.small + 4);
    if (sl.timed && !on_slot) MCU(cudaEventRecord(sl.e_a1, r.os));
    launch_pack(sl.d_desc, sl.small, E->cap, E->batch_items, sl.chunk_start, sl.first_id,
                sl.digest, sl.is_dup, sl.item_first, sl.small + 4, sl.hdev, r.num_sms, st);
    E->launches += 2;
    MCU(cudaGetLastError());
    return DEDUP_OK;
}

dedup_status apply_resets(Engine* E, Rank& r, uint64_t w) {
    while (!r.resets.empty() && r.resets.front() <= w) {
        MCU(cudaMemsetAsync(r.tab, 0, sizeof(TableSlot) * r.tab_cap, r.os));
        MCU(cudaMemsetAsync(r.tab_status, 0, 16, r.os));
        r.resets.pop_front();
    }
    return DEDUP_OK;
}

// ---- completion of wave w on rank r: rows A6-A9 on the owner stream ----
dedup_status rank_complete(Engine* E, Rank& r, uint64_t w) {
    Slot& sl = *r.slots[w % E->nslots];
    const uint32_t G = E->G;
    if (sl.wave != w || r.done_wave != w || r.next_wave <= w)
        return E->fail(DEDUP_ECUDA, "protocol: completion of a wave this rank did not submit");
    MCU(cudaSetDevice(r.dev));
    sl.timed = (w % E->time_every) == 0;
    if (E->p2p) {
        // own shard's resets for this wave first (others insert into it next)
        MTRY(apply_resets(E, r, w));
        MCU(cudaEventRecord(r.e_rst, r.os));
        if (!E->bar.wait(E->abort)) return (dedup_status)E->sticky.load();  // submitted, reset
        MCU(cudaStreamWaitEvent(r.os, sl.e_local, 0));
        for (auto& q : E->ranks) MCU(cudaStreamWaitEvent(r.os, q->e_rst, 0));
        if (sl.timed) MCU(cudaEventRecord(sl.e_a0, r.os));
        launch_p2p_insert(r.d_views, G, sl.send, sl.send_off, E->cap, r.o_slot_idx, r.num_sms,
                          r.os);  // rows A6 + A7 (insert) over peer memory
        E->launches += 1;
        MCU(cudaGetLastError());
        MCU(cudaEventRecord(r.e_rdy, r.os));
        if (!E->bar.wait(E->abort)) return (dedup_status)E->sticky.load();  // all inserted
        for (auto& q : E->ranks) MCU(cudaStreamWaitEvent(r.os, q->e_rdy, 0));
        launch_p2p_lookup(r.d_views, G, sl.send, sl.send_off, E->cap, r.o_slot_idx,
                          sl.reply_back, r.num_sms, r.os);  // rows A7 (lookup) + A8
        E->launches += 1;
        MCU(cudaGetLastError());
        MTRY(finish(E, r, sl));
        MCU(cudaEventRecord(r.e_fin, r.os));
        if (!E->bar.wait(E->abort)) return (dedup_status)E->sticky.load();  // all looked up
        for (auto& q : E->ranks) MCU(cudaStreamWaitEvent(r.os, q->e_fin, 0));
    } else if (E->copy) {
        if (!E->bar.wait(E->abort)) return (dedup_status)E->sticky.load();  // all submitted w
        MTRY(apply_resets(E, r, w));
        for (auto& q : E->ranks)
            MCU(cudaStreamWaitEvent(r.os, q->slots[w % E->nslots]->e_local, 0));
        if (sl.timed) MCU(cudaEventRecord(sl.e_a0, r.os));
        launch_gather_rows(reinterpret_cast<const uint8_t* const*>(sl.p_rec_src),
                           reinterpret_cast<const uint32_t* const*>(sl.p_rec_off), r.me, G,
                           sizeof(dedup_record), reinterpret_cast<uint8_t*>(r.recv), nullptr,
                           r.roff, E->cap, r.num_sms, r.os);
        E->launches += 1;
        MTRY(owner_work(E, r, r.roff + G, 0, E->cap * G));
        MCU(cudaEventRecord(r.e_rdy, r.os));
        if (!E->bar.wait(E->abort)) return (dedup_status)E->sticky.load();  // all looked up
        for (auto& q : E->ranks) MCU(cudaStreamWaitEvent(r.os, q->e_rdy, 0));
        launch_gather_rows(reinterpret_cast<const uint8_t* const*>(r.p_rep_src),
                           reinterpret_cast<const uint32_t* const*>(r.p_rep_off), r.me, G,
                           sizeof(uint64_t), reinterpret_cast<uint8_t*>(sl.reply_back),
                           sl.send_off, nullptr, E->cap, r.num_sms, r.os);
        E->launches += 1;
        MTRY(finish(E, r, sl));
        MCU(cudaEventRecord(r.e_fin, r.os));
        if (!E->bar.wait(E->abort)) return (dedup_status)E->sticky.load();  // all pulled
        for (auto& q : E->ranks) MCU(cudaStreamWaitEvent(r.os, q->e_fin, 0));
    } else {
        {
            ProfScope ps(E, kProfWaitCnt);
            MTRY(wait_event(E, r, sl.e_cnt));  // sizes of the payload (host)
        }
        const uint32_t* soff = sl.h_self;
        std::vector<uint64_t> rcnt(G), ro(G + 1, 0);
        for (uint32_t p = 0; p < G; ++p) {
            rcnt[p] = (uint64_t)sl.h_cnt[2 * p + 1] - sl.h_cnt[2 * p];
            ro[p + 1] = ro[p] + rcnt[p];
        }
        if (ro[G] > E->cap * G) return E->fail(DEDUP_ECUDA, "received records exceed capacity");
        uint64_t sent = 0;
        for (uint32_t p = 0; p < G; ++p)
            if (p != r.me)
                sent += (uint64_t)(soff[p + 1] - soff[p]) * sizeof(dedup_record) +
                        rcnt[p] * sizeof(uint64_t);
        E->a2a_sent += sent;
        MTRY(apply_resets(E, r, w));
        MCU(cudaStreamWaitEvent(r.os, sl.e_cnt, 0));
        if (sl.timed) MCU(cudaEventRecord(sl.e_a0, r.os));
        {
            ProfScope ps(E, kProfRecords);
            const uint64_t nself = soff[r.me + 1] - soff[r.me];  // == rcnt[me]
            if (nself && !E->nccl_self)  // own records: a device copy
                MCU(cudaMemcpyAsync(r.recv + ro[r.me], sl.send + soff[r.me],
                                    nself * sizeof(dedup_record), cudaMemcpyDeviceToDevice, r.os));
            if (G > 1 || E->nccl_self) {
                MNC(ncclGroupStart());  // row A6
                for (uint32_t p = 0; p < G; ++p) {
                    const uint64_t ns = soff[p + 1] - soff[p], nr = rcnt[p];
                    if (p == r.me && !E->nccl_self) continue;
                    if (ns) MNC(ncclSend(sl.send + soff[p], ns * sizeof(dedup_record), ncclUint8,
                                         (int)p, r.comm, r.os));
                    if (nr) MNC(ncclRecv(r.recv + ro[p], nr * sizeof(dedup_record), ncclUint8,
                                         (int)p, r.comm, r.os));
                }
                MNC(ncclGroupEnd());
            }
        }
        {
            ProfScope ps(E, kProfOwner);
            if (ro[G]) MTRY(owner_work(E, r, nullptr, ro[G], ro[G]));  // row A7
        }
        {
            ProfScope ps(E, kProfReplies);
            const uint64_t nself = soff[r.me + 1] - soff[r.me];
            if (nself && !E->nccl_self)  // replies to the own records: a device copy
                MCU(cudaMemcpyAsync(sl.reply_back + soff[r.me], r.reply + ro[r.me],
                                    nself * sizeof(uint64_t), cudaMemcpyDeviceToDevice, r.os));
            if (G > 1 || E->nccl_self) {
                MNC(ncclGroupStart());  // row A8
                for (uint32_t p = 0; p < G; ++p) {
                    const uint64_t ns = soff[p + 1] - soff[p], nr = rcnt[p];
                    if (p == r.me && !E->nccl_self) continue;
                    if (nr) MNC(ncclSend(r.reply + ro[p], nr, ncclUint64, (int)p, r.comm, r.os));
                    if (ns)
                        MNC(ncclRecv(sl.reply_back + soff[p], ns, ncclUint64, (int)p, r.comm,
                                     r.os));
                }
                MNC(ncclGroupEnd());
            }
        }
        {
            ProfScope ps(E, kProfFinish);
            MTRY(finish(E, r, sl, true));
        }
    }
    MCU(cudaEventRecord(sl.e_done, E->copy ? r.os : sl.s));
    sl.done_wave.store(w, std::memory_order_release);
    ++r.done_wave;
    return DEDUP_OK;
}

// Results of a completed slot (e_done synchronised) -> per-item views + stats.
struct Counters {
    uint64_t items = 0, bytes = 0, chunks = 0, dup_chunks = 0, dup_bytes = 0, batches = 0,
             sha1_blocks = 0, a2a_bytes = 0, waves = 0, timed_batches = 0, table_used = 0;
    double ms_a2a = 0;
};

dedup_status parse_slot(Engine* E, Rank& r, Slot& sl, Counters* ct) {
    const HostResultLayout& h = sl.hhost;
    const uint32_t n = h.header[0];
    if (h.header[1] != 0)
        return E->fail(DEDUP_ETABLEFULL, "digest table overflow (a shard): raise table_capacity");
    if (n > E->cap) return E->fail(DEDUP_ECUDA, "chunk capacity exceeded");
    sl.n_chunks = n;
    sl.item_first_v.assign(sl.n_items, 0);
    sl.item_n.assign(sl.n_items, 0);
    uint32_t next = n;
    for (int64_t k = (int64_t)sl.n_items - 1; k >= 0; --k) {
        const uint32_t f = h.item_first_chunk[k];
        if (f == 0xFFFFFFFFu) {
            sl.item_first_v[k] = next;
        } else {
            sl.item_first_v[k] = f;
            sl.item_n[k] = next - f;
            next = f;
        }
    }
    if (ct != nullptr) {
        uint64_t dups = 0, dup_bytes = 0, blocks = 0;
        for (uint32_t k = 0; k < sl.n_items; ++k) {
            const uint32_t f = sl.item_first_v[k], m = sl.item_n[k];
            for (uint32_t j = 0; j < m; ++j) {
                const uint64_t e = j + 1 < m ? h.chunk_start[f + j + 1] : sl.item_len[k];
                const uint64_t len = e - h.chunk_start[f + j];
                blocks += (len + 9 + 63) / 64;
                if (h.is_dup[f + j]) {
                    ++dups;
                    dup_bytes += len;
                }
            }
        }
        ct->items += sl.n_items;
        ct->bytes += sl.nbytes;
        ct->chunks += n;
        ct->dup_chunks += dups;
        ct->dup_bytes += dup_bytes;
        ct->sha1_blocks += blocks;
        ct->batches += sl.n_items ? 1 : 0;
        ct->table_used += h.header[2];
        for (uint32_t p = 0; p < E->G; ++p)
            if (p != r.me)
                ct->a2a_bytes += (uint64_t)(sl.h_self[p + 1] - sl.h_self[p]) *
                                 (sizeof(dedup_record) + sizeof(uint64_t));
        if (sl.timed) {
            float ms = 0;
            if (cudaEventElapsedTime(&ms, sl.e_a0, sl.e_a1) == cudaSuccess) {
                ct->ms_a2a += ms;
                ct->timed_batches += 1;
            }
            cudaGetLastError();
        }
    }
    sl.parsed = true;
    sl.next_item = 0;
    return DEDUP_OK;
}

dedup_status check_offsets(const uint64_t* item_off, uint32_t n_items, uint64_t nbytes) {
    if (item_off == nullptr || item_off[0] != 0 || item_off[n_items] != nbytes)
        return DEDUP_EINVAL;
    for (uint32_t k = 0; k < n_items; ++k)
        if (item_off[k + 1] < item_off[k] || item_off[k + 1] - item_off[k] > 0xFFFFFFFFull)
            return DEDUP_EINVAL;
    return DEDUP_OK;
}

// Fills a slot's descriptor and staging for a batch (the submitting thread).
void stage_batch(Engine* E, Slot& sl, uint64_t w, uint64_t first_seq, const uint8_t* d_bytes,
                 uint64_t nbytes, const uint64_t* item_off, uint32_t n_items) {
    sl.wave = w;
    sl.first_seq = first_seq;
    sl.nbytes = nbytes;
    sl.n_items = n_items;
    sl.d_bytes = d_bytes;
    sl.item_len.resize(n_items);
    for (uint32_t k = 0; k < n_items; ++k) sl.item_len[k] = item_off[k + 1] - item_off[k];
    std::memcpy(sl.h_item_off, item_off, sizeof(uint64_t) * (n_items + 1));
    BatchDesc& d = *sl.h_desc;
    d.bytes = d_bytes ? d_bytes : sl.d_in;
    d.nbytes = nbytes;
    d.first_seq = first_seq;
    d.item_off = sl.d_item_off;
    d.n_items = n_items;
    d.fresh = 0;
    d.table = TableView{nullptr, 0, nullptr};
    sl.busy = true;
    sl.parsed = false;
    sl.next_item = 0;
    (void)E;
}

// Records the producer stream's current work into the slot (or a foreign
// event when the producer is on another device).
dedup_status record_producer(Engine* E, Rank& r, Slot& sl, void* producer) {
    cudaStream_t ps = static_cast<cudaStream_t>(producer);
    int pdev = r.dev;
    if (ps != nullptr && cudaStreamGetDevice(ps, &pdev) != cudaSuccess) pdev = r.dev;
    if (ps == nullptr) cudaGetDevice(&pdev);
    if (pdev == r.dev) {
        MCU(cudaSetDevice(r.dev));
        MCU(cudaEventRecord(sl.e_prod, ps));
        return DEDUP_OK;
    }
    MCU(cudaSetDevice(pdev));
    MCU(cudaEventCreateWithFlags(&sl.e_prod_foreign, cudaEventDisableTiming));
    MCU(cudaEventRecord(sl.e_prod_foreign, ps));
    return DEDUP_OK;
}

dedup_status engine_init(Engine* E, const dedup_config* cfg, uint32_t G, uint32_t depth,
                         uint64_t batch_bytes, uint32_t batch_items) {
    E->cfg = *cfg;
    E->G = G;
    E->depth = depth;
    E->nslots = depth;
    E->batch_bytes = batch_bytes;
    E->batch_items = batch_items;
    E->cap = batch_bytes / 32 + batch_items + 2;
    E->host_fed = cfg->host_fed != 0;
    E->lane_bytes = cfg->sha_lane_bytes ? cfg->sha_lane_bytes : 16384;
    if (const char* v = std::getenv("DEDUP_TIME_EVERY"))
        E->time_every = std::atoi(v) > 0 ? (uint32_t)std::atoi(v) : 1u;
    if (const char* v = std::getenv("DEDUP_MG_TIMEOUT_S")) E->timeout_s = std::atof(v);
    E->profile = std::getenv("DEDUP_MG_PROFILE") != nullptr;
    E->nccl_self = std::getenv("DEDUP_MG_NCCL_SELF") != nullptr;
    return DEDUP_OK;
}

}  // namespace

// ===========================================================================
// The ctx engine: G ranks in this process, one worker thread per rank.
// ===========================================================================
struct CtxEngine {
    Engine E;
    struct Cmd {
        enum Kind { SUBMIT, COMPLETE, END_STREAM, QUIT } k;
        uint64_t w;
    };
    struct Queue {
        std::mutex m;
        std::condition_variable cv;
        std::deque<Cmd> q;
        std::atomic<uint64_t> pushed{0}, processed{0};
    };
    std::vector<std::unique_ptr<Queue>> queues;
    std::vector<std::thread> workers;
    // API-thread state (a ctx is not thread-safe: calls are serialised)
    uint64_t fill_wave = 0;      // next batch goes to (fill_wave, fill_rank)
    uint32_t fill_rank = 0;
    uint64_t complete_issued = 0;
    uint64_t drain_wave = 0;     // next batch handed out by drain
    uint32_t drain_rank = 0;
    uint64_t next_seq = 0, pending_items = 0;
    std::vector<Slot*> to_release;
    Counters ct;
    uint32_t lag = 1;

    void push(uint32_t r, Cmd c) {
        Queue& q = *queues[r];
        {
            std::lock_guard<std::mutex> lk(q.m);
            q.q.push_back(c);
            ++q.pushed;
        }
        q.cv.notify_one();
    }
    void push_all(Cmd c) {
        for (uint32_t r = 0; r < E.G; ++r) push(r, c);
    }
    void worker(uint32_t r) {
        Rank& rk = *E.ranks[r];
        cudaSetDevice(rk.dev);
        Queue& q = *queues[r];
        for (;;) {
            Cmd c;
            {
                std::unique_lock<std::mutex> lk(q.m);
                q.cv.wait(lk, [&] { return !q.q.empty(); });
                c = q.q.front();
                q.q.pop_front();
            }
            if (c.k == Cmd::QUIT) {
                ++q.processed;
                return;
            }
            if (!E.abort.load()) {
                switch (c.k) {
                    case Cmd::SUBMIT: rank_submit(&E, rk, c.w); break;
                    case Cmd::COMPLETE: rank_complete(&E, rk, c.w); break;
                    case Cmd::END_STREAM: rk.resets.push_back(c.w); break;
                    default: break;
                }
            }
            ++q.processed;
        }
    }
    // waits until every worker processed everything pushed so far
    dedup_status wait_idle() {
        for (auto& qp : queues)
            while (qp->processed.load() < qp->pushed.load()) {
                if (E.abort.load()) return (dedup_status)E.sticky.load();
                std::this_thread::sleep_for(std::chrono::microseconds(10));
            }
        return DEDUP_OK;
    }
    Slot& slot(uint64_t w, uint32_t r) { return *E.ranks[r]->slots[w % E.nslots]; }
    bool assigned(uint64_t w, uint32_t r) const {
        return w < fill_wave || (w == fill_wave && r < fill_rank);
    }
    // after a batch is assigned to (fill_wave, fill_rank): advance, issue completions
    void advance() {
        if (++fill_rank == E.G) {
            fill_rank = 0;
            ++fill_wave;
            while (fill_wave - complete_issued > lag) push_all({Cmd::COMPLETE, complete_issued++});
        }
    }
    // empty batches for the ranks of a partly filled wave; false if a slot is busy
    bool close_partial() {
        if (fill_rank == 0) return true;
        for (uint32_t r = fill_rank; r < E.G; ++r)
            if (slot(fill_wave, r).busy) return false;
        static const uint64_t zero = 0;
        while (fill_rank != 0) {
            const uint32_t r = fill_rank;
            Slot& sl = slot(fill_wave, r);
            stage_batch(&E, sl, fill_wave, next_seq, nullptr, 0, &zero, 0);
            sl.h2d.clear();
            push(r, {Cmd::SUBMIT, fill_wave});
            advance();
        }
        return true;
    }
    void complete_all_closed() {
        while (complete_issued < fill_wave) push_all({Cmd::COMPLETE, complete_issued++});
    }
};

namespace {

dedup_status sticky_or(CtxEngine* e, dedup_status st) {
    const int s = e->E.sticky.load();
    return s ? (dedup_status)s : st;
}

}  // namespace

dedup_status create(const dedup_config* cfg, CtxEngine** out, const char** why) {
    *out = nullptr;
    *why = "bad multi-GPU config";
    const uint32_t G = cfg->num_devices ? cfg->num_devices : 1;
    if (G > 64 || cfg->owner_rank != 0 || cfg->num_owners != 1) return DEDUP_EINVAL;
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess) {
        *why = "no CUDA device";
        return DEDUP_ECUDA;
    }
    std::vector<int> devs(G);
    bool distinct = true;
    for (uint32_t r = 0; r < G; ++r) {
        devs[r] = cfg->device_ids ? cfg->device_ids[r] : (int)r;
        if (devs[r] < 0 || devs[r] >= ndev) {
            *why = "device id out of range";
            return DEDUP_EINVAL;
        }
        for (uint32_t q = 0; q < r; ++q) distinct = distinct && devs[q] != devs[r];
    }
    const bool p2p = cfg->transport == 3;
    bool copy = cfg->transport == 2 || p2p || (cfg->transport == 0 && !distinct);
    if (!copy && !distinct) {
        *why = "NCCL needs distinct devices (one rank per GPU)";
        return DEDUP_EUNSUPPORTED;
    }
    auto* e = new CtxEngine();
    Engine& E = e->E;
    E.copy = copy;
    E.p2p = p2p;
    engine_init(&E, cfg, G, cfg->slots, cfg->batch_bytes, cfg->batch_items);
    E.bar.n = G;
    e->lag = E.depth > 1 ? E.depth - 1 : 1;
    if (copy && distinct) {  // peer loads over NVLink
        for (uint32_t a = 0; a < G; ++a)
            for (uint32_t b = 0; b < G; ++b) {
                if (a == b) continue;
                int ok = 0;
                cudaDeviceCanAccessPeer(&ok, devs[a], devs[b]);
                if (!ok) {
                    delete e;
                    *why = "copy transport: no peer access between the devices";
                    return DEDUP_EUNSUPPORTED;
                }
                cudaSetDevice(devs[a]);
                const cudaError_t pe = cudaDeviceEnablePeerAccess(devs[b], 0);
                if (pe != cudaSuccess && pe != cudaErrorPeerAccessAlreadyEnabled) {
                    delete e;
                    *why = "cudaDeviceEnablePeerAccess failed";
                    return DEDUP_ECUDA;
                }
                cudaGetLastError();
            }
    }
    const uint64_t shard = cfg->table_capacity / G + 1024;
    for (uint32_t r = 0; r < G; ++r) {
        E.ranks.emplace_back(new Rank());
        Rank& rk = *E.ranks.back();
        rk.E = &E;
        rk.me = r;
        rk.dev = devs[r];
        const dedup_status st = rank_alloc(&E, rk, shard);
        if (st != DEDUP_OK) {
            *why = "rank allocation failed";
            delete e;
            return st;
        }
    }
    if (copy) {
        if (wire_copy(&E) != DEDUP_OK) {
            *why = "copy transport wiring failed";
            delete e;
            return DEDUP_ECUDA;
        }
    } else {
        std::vector<ncclComm_t> comms(G), ccomms(G);
        if (ncclCommInitAll(comms.data(), (int)G, devs.data()) != ncclSuccess ||
            ncclCommInitAll(ccomms.data(), (int)G, devs.data()) != ncclSuccess) {
            *why = "ncclCommInitAll failed";
            delete e;
            return DEDUP_ENCCL;
        }
        for (uint32_t r = 0; r < G; ++r) {
            E.ranks[r]->comm = comms[r];
            E.ranks[r]->ccomm = ccomms[r];
        }
    }
    for (uint32_t r = 0; r < G; ++r) e->queues.emplace_back(new CtxEngine::Queue());
    for (uint32_t r = 0; r < G; ++r) e->workers.emplace_back([e, r] { e->worker(r); });
    *out = e;
    return DEDUP_OK;
}

void destroy(CtxEngine* e) {
    if (e == nullptr) return;
    if (!e->E.abort.load()) {  // finish the waves in flight (their ranks wait for each other)
        if (e->close_partial()) {
            e->complete_all_closed();
            e->wait_idle();
        } else {
            e->E.abort.store(true);
            e->E.bar.wake();
        }
    }
    e->push_all({CtxEngine::Cmd::QUIT, 0});
    for (auto& t : e->workers) t.join();
    delete e;
}

const char* last_error(const CtxEngine* e) {
    // the string only changes on the first error (sticky), before abort is set
    return const_cast<CtxEngine*>(e)->E.err.c_str();
}

int32_t next_device(const CtxEngine* e) { return e->E.ranks[e->fill_rank]->dev; }

dedup_status submit_host(CtxEngine* e, uint32_t n_items, const uint8_t* const* item_ptr,
                         const uint64_t* item_len, uint64_t* first_seq_out) {
    Engine& E = e->E;
    if (E.sticky.load()) return E.sticky.load();
    if (!E.host_fed) return DEDUP_EINVAL;
    if (n_items > 0 && (item_ptr == nullptr || item_len == nullptr)) return DEDUP_EINVAL;
    // plan batches of whole items
    std::vector<std::pair<uint32_t, uint32_t>> plan;
    uint32_t b0 = 0;
    uint64_t bytes = 0;
    for (uint32_t k = 0; k < n_items; ++k) {
        const uint64_t L = item_len[k];
        if (L > E.batch_bytes || L > 0xFFFFFFFFull) return DEDUP_EINVAL;
        if (L > 0 && item_ptr[k] == nullptr) return DEDUP_EINVAL;
        if (k > b0 && (bytes + L > E.batch_bytes || k - b0 >= E.batch_items)) {
            plan.emplace_back(b0, k);
            b0 = k;
            bytes = 0;
        }
        bytes += L;
    }
    if (n_items > b0) plan.emplace_back(b0, n_items);
    {  // every batch needs a free slot
        uint64_t w = e->fill_wave;
        uint32_t r = e->fill_rank;
        for (size_t j = 0; j < plan.size(); ++j) {
            if (j >= (size_t)E.depth * E.G || e->slot(w, r).busy) return DEDUP_EAGAIN;
            if (++r == E.G) r = 0, ++w;
        }
    }
    if (first_seq_out) *first_seq_out = e->next_seq;
    std::vector<uint64_t> off;
    for (auto& pr : plan) {
        const uint32_t r = e->fill_rank, n = pr.second - pr.first;
        Slot& sl = e->slot(e->fill_wave, r);
        off.assign(n + 1, 0);
        for (uint32_t k = 0; k < n; ++k) off[k + 1] = off[k] + item_len[pr.first + k];
        stage_batch(&E, sl, e->fill_wave, e->next_seq, nullptr, off[n], off.data(), n);
        sl.h2d.clear();
        uint32_t k = 0;
        while (k < n) {  // merge contiguous host ranges
            const uint8_t* p = item_ptr[pr.first + k];
            uint64_t len = item_len[pr.first + k];
            const uint64_t dst = off[k];
            uint32_t j = k + 1;
            while (j < n && item_ptr[pr.first + j] == p + len) len += item_len[pr.first + j++];
            if (len) {
                cudaPointerAttributes pa{};
                const bool locked = cudaPointerGetAttributes(&pa, p) == cudaSuccess &&
                                    pa.type == cudaMemoryTypeHost;
                cudaGetLastError();
                if (!locked) {  // pageable: into the slot's page-locked bounce buffer now
                    if (sl.h_bounce == nullptr) {
                        cudaSetDevice(E.ranks[r]->dev);
                        if (cudaHostAlloc(reinterpret_cast<void**>(&sl.h_bounce), E.batch_bytes,
                                          cudaHostAllocPortable) != cudaSuccess) {
                            sl.h_bounce = nullptr;
                            return E.fail(DEDUP_ENOMEM, "bounce buffer allocation failed");
                        }
                    }
                    std::memcpy(sl.h_bounce + dst, p, len);
                    p = sl.h_bounce + dst;
                }
            }
            sl.h2d.push_back({p, dst, len});
            k = j;
        }
        e->next_seq += n;
        e->pending_items += n;
        e->push(r, {CtxEngine::Cmd::SUBMIT, e->fill_wave});
        e->advance();
    }
    return sticky_or(e, DEDUP_OK);
}

dedup_status submit_device(CtxEngine* e, const uint8_t* d_bytes, uint64_t nbytes,
                           const uint64_t* item_off, uint32_t n_items, void* producer,
                           uint64_t* first_seq_out) {
    Engine& E = e->E;
    if (E.sticky.load()) return E.sticky.load();
    if (nbytes > 0 && d_bytes == nullptr) return DEDUP_EINVAL;
    if (reinterpret_cast<uintptr_t>(d_bytes) & 15) return DEDUP_EINVAL;
    if (nbytes > E.batch_bytes || n_items > E.batch_items) return DEDUP_EINVAL;
    if (check_offsets(item_off, n_items, nbytes) != DEDUP_OK) return DEDUP_EINVAL;
    const uint32_t r = e->fill_rank;
    Slot& sl = e->slot(e->fill_wave, r);
    if (sl.busy) return DEDUP_EAGAIN;
    stage_batch(&E, sl, e->fill_wave, e->next_seq,
                d_bytes ? d_bytes : reinterpret_cast<const uint8_t*>(E.ranks[r]->d_rtab),
                nbytes, item_off, n_items);  // (an empty batch reads nothing)
    sl.h2d.clear();
    const dedup_status st = record_producer(&E, *E.ranks[r], sl, producer);
    if (st != DEDUP_OK) return st;
    if (first_seq_out) *first_seq_out = e->next_seq;
    e->next_seq += n_items;
    e->pending_items += n_items;
    e->push(r, {CtxEngine::Cmd::SUBMIT, e->fill_wave});
    e->advance();
    return sticky_or(e, DEDUP_OK);
}

dedup_status join(CtxEngine* e, void* stream) {
    Engine& E = e->E;
    if (E.sticky.load()) return E.sticky.load();
    if (!e->close_partial()) return DEDUP_EAGAIN;
    e->complete_all_closed();
    MTRY(e->wait_idle());
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    for (auto& rp : E.ranks)
        for (auto& sl : rp->slots)
            if (sl->busy && cudaStreamWaitEvent(s, sl->e_done, 0) != cudaSuccess)
                return E.fail(DEDUP_ECUDA, "join: cudaStreamWaitEvent failed");
    return sticky_or(e, DEDUP_OK);
}

dedup_status end_stream(CtxEngine* e) {
    Engine& E = e->E;
    if (E.sticky.load()) return E.sticky.load();
    if (!e->close_partial()) return DEDUP_EAGAIN;
    // the table resets go in on every owner stream right before the owner
    // work of the new stream's first wave (no drain of the pipeline)
    e->push_all({CtxEngine::Cmd::END_STREAM, e->fill_wave});
    return DEDUP_OK;
}

dedup_status drain(CtxEngine* e, uint32_t max_items, int32_t wait_ms, dedup_item_result* out,
                   uint32_t* n_out) {
    Engine& E = e->E;
    *n_out = 0;
    if (E.sticky.load()) return E.sticky.load();
    for (Slot* s : e->to_release) s->busy = false;
    e->to_release.clear();
    const auto deadline = Clock::now() + std::chrono::milliseconds(wait_ms < 0 ? 0 : wait_ms);
    uint32_t got = 0;
    while (got < max_items) {
        const uint64_t w = e->drain_wave;
        const uint32_t r = e->drain_rank;
        // block only if the caller waits (nothing handed out yet); an assigned
        // slot is waited for even if it holds no items (a padded wave's empty
        // batch), since it occupies the ring
        const bool may_block = got == 0 && wait_ms != 0;
        if (!e->assigned(w, r)) {  // the rest of this wave is not submitted yet
            if (!may_block || e->pending_items == 0 || !e->close_partial()) break;
            continue;
        }
        Slot& sl = e->slot(w, r);
        if (!sl.parsed) {
            if (w >= e->complete_issued) {
                if (!may_block) break;
                // a wave completes only once every rank has its batch: pad
                // the partly filled one first (its other ranks get empty batches)
                if (w >= e->fill_wave && !e->close_partial()) break;
                while (e->complete_issued <= w)
                    e->push_all({CtxEngine::Cmd::COMPLETE, e->complete_issued++});
            }
            // the worker records e_done, then publishes the wave
            bool ready = false;
            for (;;) {
                if (E.abort.load()) return E.sticky.load();
                if (sl.done_wave.load(std::memory_order_acquire) == w) {
                    const cudaError_t q = cudaEventQuery(sl.e_done);
                    if (q == cudaSuccess) {
                        ready = true;
                        break;
                    }
                    if (q != cudaErrorNotReady)
                        return E.fail(DEDUP_ECUDA, std::string("wave failed: ") +
                                                       cudaGetErrorString(q));
                }
                if (!may_block) break;
                if (wait_ms > 0 && Clock::now() > deadline) {
                    *n_out = got;
                    return DEDUP_ETIMEDOUT;
                }
                std::this_thread::sleep_for(std::chrono::microseconds(20));
            }
            if (!ready) break;
            MTRY(parse_slot(&E, *E.ranks[r], sl, &e->ct));
            if (r == 0) ++e->ct.waves;
        }
        while (got < max_items && sl.next_item < sl.n_items) {
            const uint32_t k = sl.next_item++;
            dedup_item_result& o = out[got++];
            o.seq = sl.first_seq + k;
            o.item_len = sl.item_len[k];
            o.n_chunks = sl.item_n[k];
            o.carried = 0;
            if (o.n_chunks) {
                const uint32_t f = sl.item_first_v[k];
                o.chunk_start = sl.hhost.chunk_start + f;
                o.digest = sl.hhost.digest + 20ull * f;
                o.is_dup = sl.hhost.is_dup + f;
                o.first_id = sl.hhost.first_id + f;
            } else {
                o.chunk_start = nullptr;
                o.digest = nullptr;
                o.is_dup = nullptr;
                o.first_id = nullptr;
            }
            --e->pending_items;
        }
        if (sl.next_item == sl.n_items) {
            e->to_release.push_back(&sl);  // results stay valid until the next drain
            if (++e->drain_rank == E.G) e->drain_rank = 0, ++e->drain_wave;
        }
    }
    *n_out = got;
    return DEDUP_OK;
}

uint64_t pending(const CtxEngine* e) { return e->pending_items; }

dedup_status stats(const CtxEngine* e, dedup_stats_t* out) {
    std::memset(out, 0, sizeof(*out));
    const Counters& c = e->ct;
    out->items = c.items;
    out->bytes = c.bytes;
    out->chunks = c.chunks;
    out->dup_chunks = c.dup_chunks;
    out->dup_bytes = c.dup_bytes;
    out->unique_chunks = c.chunks - c.dup_chunks;
    out->batches = c.batches;
    out->table_used = c.table_used;
    out->sha1_blocks = c.sha1_blocks;
    out->num_owners = e->E.G;
    out->num_devices = e->E.G;
    out->waves = c.waves;
    out->a2a_bytes = c.a2a_bytes;
    out->ms_a2a = c.ms_a2a;
    out->timed_batches = c.timed_batches;
    out->kernel_launches = e->E.launches.load();
    uint64_t slots = 0;
    for (auto& r : e->E.ranks) slots += r->tab_cap;
    out->table_slots = slots;
    return DEDUP_OK;
}

uint64_t kernel_launches(const CtxEngine* e) { return e->E.launches.load(); }

}  // namespace mg
}  // namespace dd

// ===========================================================================
// dedup_dist_*: one rank per process (NCCL), driven by the caller's thread.
// ===========================================================================
using namespace dd::mg;

struct dedup_dist {
    Engine E;
    int last_done = -1;
    std::vector<uint64_t> res_item_off;
};

extern "C" {

dedup_status dedup_nccl_unique_id(uint8_t out[128]) {
    static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId is 128 bytes");
    if (out == nullptr) return DEDUP_EINVAL;
    ncclUniqueId id;
    if (ncclGetUniqueId(&id) != ncclSuccess) return DEDUP_ENCCL;
    std::memcpy(out, &id, 128);
    return DEDUP_OK;
}

dedup_status dedup_dist_create(const dedup_config* cfg, const uint8_t nccl_id[128], int nranks,
                               int rank, uint32_t depth, uint64_t batch_bytes,
                               uint32_t batch_items, dedup_dist** out) {
    if (out == nullptr) return DEDUP_EINVAL;
    *out = nullptr;
    if (cfg == nullptr || nccl_id == nullptr || nranks < 1 || nranks > 64 || rank < 0 ||
        rank >= nranks || depth < 1 || depth > 64 || batch_bytes < 1 ||
        batch_bytes > (1ull << 30) || batch_items < 1 || (uint32_t)nranks != cfg->num_owners ||
        (uint32_t)rank != cfg->owner_rank)
        return DEDUP_EINVAL;
    auto* d = new dedup_dist();
    Engine* E = &d->E;
    dedup_config c = *cfg;
    c.host_fed = 0;
    engine_init(E, &c, (uint32_t)nranks, depth, batch_bytes, batch_items);
    E->nslots = depth + 1;
    E->ranks.emplace_back(new Rank());
    Rank& rk = *E->ranks.back();
    rk.E = E;
    rk.me = (uint32_t)rank;
    rk.dev = cfg->device;
    // cfg->table_capacity: this shard's expected distinct digests
    if (rank_alloc(E, rk, cfg->table_capacity) != DEDUP_OK) {
        delete d;
        return DEDUP_ENOMEM;
    }
    ncclUniqueId id;
    std::memcpy(&id, nccl_id, 128);
    if (ncclCommInitRank(&rk.comm, nranks, id, rank) != ncclSuccess ||
        ncclCommSplit(rk.comm, 0, rank, &rk.ccomm, nullptr) != ncclSuccess) {
        delete d;
        return DEDUP_ENCCL;
    }
    *out = d;
    return DEDUP_OK;
}

void dedup_dist_destroy(dedup_dist* d) { delete d; }

const char* dedup_dist_last_error(const dedup_dist* d) {
    return d ? d->E.err.c_str() : "null dist";
}

dedup_status dedup_dist_submit(dedup_dist* d, const uint8_t* d_bytes, uint64_t nbytes,
                               const uint64_t* item_off, uint32_t n_items, uint64_t first_seq,
                               void* producer, uint32_t* completed) {
    if (d == nullptr || completed == nullptr) return DEDUP_EINVAL;
    *completed = 0;
    Engine* E = &d->E;
    if (E->sticky.load()) return E->sticky.load();
    ProfScope ps(E, kProfSubmit);
    // argument checks before anything is enqueued (every rank then issues
    // the same NCCL sequence or none)
    if (n_items > E->batch_items || nbytes > E->batch_bytes ||
        check_offsets(item_off, n_items, nbytes) != DEDUP_OK ||
        (nbytes > 0 && d_bytes == nullptr) || (reinterpret_cast<uintptr_t>(d_bytes) & 15)) {
        E->err = "bad batch";
        return DEDUP_EINVAL;
    }
    Rank& rk = *E->ranks[0];
    if (rk.next_wave - rk.done_wave >= E->depth) {
        MTRY(rank_complete(E, rk, rk.done_wave));
        d->last_done = (int)((rk.done_wave - 1) % E->nslots);
        Slot& ds = *rk.slots[d->last_done];
        d->res_item_off.assign(ds.h_item_off, ds.h_item_off + ds.n_items + 1);
        *completed = 1;
    }
    const uint64_t w = rk.next_wave;
    // depth + 1 slots: this wave's slot last held wave w - depth - 1, completed
    // (its counts, hence its graph's staging copies, waited for) one call ago
    Slot& sl = *rk.slots[w % E->nslots];
    stage_batch(E, sl, w, first_seq,
                d_bytes ? d_bytes : reinterpret_cast<const uint8_t*>(rk.d_rtab), nbytes,
                item_off, n_items);
    sl.h2d.clear();
    MTRY(record_producer(E, rk, sl, producer));
    return rank_submit(E, rk, w);
}

dedup_status dedup_dist_flush(dedup_dist* d, uint32_t* completed) {
    if (d == nullptr || completed == nullptr) return DEDUP_EINVAL;
    *completed = 0;
    Engine* E = &d->E;
    if (E->sticky.load()) return E->sticky.load();
    Rank& rk = *E->ranks[0];
    if (rk.done_wave == rk.next_wave) {
        prof_dump(E);  // drained: one profile per drained run
        return DEDUP_OK;
    }
    MTRY(rank_complete(E, rk, rk.done_wave));
    d->last_done = (int)((rk.done_wave - 1) % E->nslots);
    Slot& ds = *rk.slots[d->last_done];
    d->res_item_off.assign(ds.h_item_off, ds.h_item_off + ds.n_items + 1);
    *completed = 1;
    return DEDUP_OK;
}

dedup_status dedup_dist_join(dedup_dist* d, void* stream) {
    if (d == nullptr) return DEDUP_EINVAL;
    Engine* E = &d->E;
    if (E->sticky.load()) return E->sticky.load();
    Rank& rk = *E->ranks[0];
    if (cudaSetDevice(rk.dev) != cudaSuccess) return DEDUP_ECUDA;
    for (auto& sl : rk.slots)
        if (sl->done_wave.load() != ~0ull &&
            cudaStreamWaitEvent(static_cast<cudaStream_t>(stream), sl->e_done, 0) != cudaSuccess)
            return E->fail(DEDUP_ECUDA, "join: cudaStreamWaitEvent failed");
    return DEDUP_OK;
}

uint64_t dedup_dist_kernel_launches(const dedup_dist* d) {
    return d ? d->E.launches.load() : 0;
}

uint64_t dedup_dist_a2a_bytes(const dedup_dist* d) { return d ? d->E.a2a_sent.load() : 0; }

dedup_status dedup_dist_end_stream(dedup_dist* d) {
    if (d == nullptr) return DEDUP_EINVAL;
    Engine* E = &d->E;
    if (E->sticky.load()) return E->sticky.load();
    Rank& rk = *E->ranks[0];
    if (rk.done_wave != rk.next_wave) {
        rk.resets.push_back(rk.next_wave);  // before the next stream's first wave's owner work
        return DEDUP_OK;
    }
    if (cudaSetDevice(rk.dev) != cudaSuccess) return DEDUP_ECUDA;
    rk.resets.clear();  // subsumed
    rk.resets.push_back(0);
    return apply_resets(E, rk, ~0ull);
}

dedup_status dedup_dist_last_counts(const dedup_dist* d, uint32_t* n_items, uint32_t* n_chunks,
                                    uint64_t* nbytes) {
    if (d == nullptr || d->last_done < 0) return DEDUP_EINVAL;
    const Engine& E = d->E;
    const Slot& sl = *E.ranks[0]->slots[d->last_done];
    if (n_items) *n_items = sl.n_items;
    if (n_chunks) *n_chunks = sl.h_self[E.G + 1];  // the counts arrived before completion
    if (nbytes) *nbytes = sl.nbytes;
    return DEDUP_OK;
}

dedup_status dedup_dist_result(const dedup_dist* d_, dedup_wave_result* out) {
    if (d_ == nullptr || out == nullptr || d_->last_done < 0) return DEDUP_EINVAL;
    dedup_dist* d = const_cast<dedup_dist*>(d_);
    Engine* E = &d->E;
    Rank& rk = *E->ranks[0];
    Slot& sl = *rk.slots[d->last_done];
    if (cudaSetDevice(rk.dev) != cudaSuccess) return DEDUP_ECUDA;
    MTRY(wait_event(E, rk, sl.e_done));
    if (!sl.parsed) MTRY(parse_slot(E, rk, sl, nullptr));
    out->first_seq = sl.first_seq;
    out->n_items = sl.n_items;
    out->n_chunks = sl.n_chunks;
    out->item_off = d->res_item_off.data();
    out->item_first_chunk = sl.hhost.item_first_chunk;
    out->chunk_start = sl.hhost.chunk_start;
    out->digest = sl.hhost.digest;
    out->first_id = sl.hhost.first_id;
    out->is_dup = sl.hhost.is_dup;
    return DEDUP_OK;
}

}  // extern "C"
