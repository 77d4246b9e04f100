// api.cpp -- C ABI (include/dedup.h) and the per-GPU streaming engine.
//
// Engine (rows A1 + A9 of the hot path): a ring of `slots` batch slots used
// strictly round-robin ("memory spaces").  Each
// slot owns a CUDA stream, device buffers, a mapped pinned result buffer and
// ONE CUDA GRAPH holding the whole per-batch launch sequence:
//   desc + item offsets H2D -> rabin_scan -> select (agg, scan, emit)
//   -> chunk_meta -> long_list -> sha1 -> [wait: previous slot's table event]
//   -> table_prepare -> insert -> lookup -> [record table event]
//   -> pack (kernel stores results straight into pinned host memory)
// Per-batch parameters live in a device-side BatchDesc copied by the graph
// from the slot's pinned staging, so a submit is a host memcpy plus one
// cudaGraphLaunch (+ an event pair for the producer stream or the H2D of
// host items).  Table work of consecutive batches is chained through the
// previous slot's table event, so every lookup sees the inserts of all
// earlier batches (the sequential stream-order answer, reading O12) and a
// table is only cleared after every earlier batch is done with it.
// dedup_drain waits on the slot's completion event and hands items out
// strictly in sequence order.
#include <cuda_runtime.h>

#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <deque>
#include <string>
#include <thread>
#include <vector>

#include "dedup.h"
#include "internal.h"
#include "mg.h"

using namespace dd;

namespace {

constexpr int kOpRing = 64;  // descriptors in flight for the dedup_op_* layer

struct Workspace {
    uint32_t* bitmap = nullptr;      // candidate bitmap, one bit per byte
    uint32_t* agg = nullptr;         // per-tile transfer functions (32 u32 per tile)
    uint32_t* gagg = nullptr;        // per-group transfer functions (32 u32 per group)
    uint32_t* gentry = nullptr;      // per-group entry state + cut offset
    uint32_t* evbuf = nullptr;       // per-tile event lists (scan -> cut emission)
    uint32_t* counters = nullptr;    // [0..1] sha1 work/long counters, [64..191] route
    uint32_t* slot_idx = nullptr;    // table slot per record
    uint32_t* sha_ws = nullptr;      // SHA-1 sort of the chunks by length + task counter
    uint32_t* mc_ws = nullptr;       // max_chunk selection scratch (maxchunk_ws_words)
    uint64_t max_tiles = 0;
    uint64_t item_cap = 0;           // items the max_chunk scratch holds
};

struct Slot {
    cudaStream_t stream = nullptr;
    cudaEvent_t ev_host = nullptr, ev_start = nullptr, ev_h2d = nullptr, ev_scan = nullptr,
                ev_chunk = nullptr, ev_sha = nullptr, ev_table = nullptr, ev_done = nullptr;
    cudaEvent_t ev_prod = nullptr;  // producer-stream dependency (no timing)
    // carry-over mode: this slot's batch done with its history / selection /
    // continued chunk (the next slot's batch waits on them)
    cudaEvent_t ev_hist = nullptr, ev_sel = nullptr, ev_carry = nullptr;
    cudaGraphExec_t graph = nullptr;
    BatchDesc* d_desc = nullptr;    // device descriptor (graph copies h_desc into it)
    BatchDesc* h_desc = nullptr;    // pinned staging
    uint8_t* d_bytes = nullptr;     // host-fed input copy
    uint8_t* h_bounce = nullptr;    // page-locked bounce buffer for pageable items (lazy)
    uint64_t* d_item_off = nullptr;
    uint64_t* h_item_off = nullptr;  // pinned staging of item offsets
    Workspace ws;
    uint32_t* d_cut_pos = nullptr;
    uint32_t* d_chunk_start = nullptr;
    uint32_t* d_item_first = nullptr;
    uint32_t* d_small = nullptr;    // [0] n_chunks, [4..5] table status copy
    uint64_t* d_chunk_id = nullptr;
    uint64_t* d_first_id = nullptr;
    uint8_t* d_digest = nullptr;
    uint8_t* d_is_dup = nullptr;
    uint8_t* h_res = nullptr;       // mapped pinned results
    HostResultLayout hdev{};        // device view of h_res
    HostResultLayout hhost{};       // host view of h_res
    // batch in flight
    bool busy = false;
    bool parsed = false;
    bool host_fed = false;
    uint64_t first_seq = 0;
    uint32_t n_items = 0;
    uint64_t nbytes = 0;
    std::vector<uint64_t> item_len;
    std::vector<uint32_t> item_first, item_n;
    uint32_t next_item = 0;  // next item of this batch to hand out
    uint32_t carried = 0;    // carry-over: bytes of chunk 0 in earlier pieces (saturated)
};

struct TableBuf {
    TableSlot* slots = nullptr;
    uint32_t* status = nullptr;
    uint64_t capacity = 0;
};

}  // namespace

struct dedup_ctx {
    dedup_config cfg{};
    dd::mg::CtxEngine* mg = nullptr;  // num_devices >= 2: the multi-GPU engine (mg.cpp)
    int num_sms = 0;
    uint32_t* d_tab = nullptr;  // R[256] then W256[256]
    std::vector<Slot> slots;
    uint32_t next_slot = 0;     // round-robin cursor
    TableBuf tables[2];
    int cur_table = 0;
    TableBuf local;                   // local-combine table (dedup_op_local_combine)
    TableView* d_local_view = nullptr;
    bool stream_fresh = false;  // next batch starts a new dedup stream
    // carry-over mode (row NEXT-2): one CarryState per slot (batch in slot i
    // writes d_carry[i], reads d_carry[i - 1]); carry_started: the current
    // dedup stream has bytes (its next piece continues it, end_stream closes it)
    CarryState* d_carry = nullptr;
    bool carry_started = false;
    uint64_t chunk_cap = 0;     // chunks per slot
    std::deque<int> inflight;   // slot indices in seq order
    std::vector<int> to_release;
    uint64_t next_seq = 0;
    uint64_t pending_items = 0;
    // dedup_op_* layer
    Workspace op_ws;
    BatchDesc* op_d_desc = nullptr;  // [kOpRing]
    BatchDesc* op_h_desc = nullptr;  // [kOpRing] pinned
    cudaEvent_t op_ev[kOpRing] = {};
    bool op_ev_used[kOpRing] = {};
    int op_next = 0;
    // status
    dedup_status sticky = DEDUP_OK;
    std::string err = "no error";
    uint64_t launches = 0;
    uint32_t graph_kernels = 0;  // kernels per batch graph
    dedup_stats_t st{};
    bool trace = false;           // DEDUP_TRACE environment variable
    bool stage_events = true;     // per-stage timing events in the batch graphs
    uint32_t time_every = 1;      // query stage times of every n-th batch (DEDUP_TIME_EVERY)
    uint64_t parsed_batches = 0;
    cudaEvent_t ev_ref = nullptr;  // time origin of the trace
};

namespace {

dedup_status fail(dedup_ctx* c, dedup_status s, const std::string& msg) {
    if (c) {
        c->err = msg;
        if (s == DEDUP_ECUDA || s == DEDUP_ETABLEFULL) c->sticky = s;
    }
    return s;
}

#define CU(call)                                                                             \
    do {                                                                                     \
        cudaError_t e_ = (call);                                                             \
        if (e_ != cudaSuccess)                                                               \
            return fail(c, DEDUP_ECUDA, std::string(#call ": ") + cudaGetErrorString(e_));   \
    } while (0)

#define TRY(x)                         \
    do {                               \
        dedup_status s_ = (x);         \
        if (s_ != DEDUP_OK) return s_; \
    } while (0)

uint64_t next_pow2(uint64_t v) {
    uint64_t p = 1;
    while (p < v) p <<= 1;
    return p;
}

template <class T>
dedup_status dalloc(dedup_ctx* c, T** p, uint64_t count) {
    if (count == 0) count = 1;
    cudaError_t e = cudaMalloc(reinterpret_cast<void**>(p), sizeof(T) * count);
    if (e != cudaSuccess)
        return fail(c, DEDUP_ENOMEM, std::string("cudaMalloc: ") + cudaGetErrorString(e));
    return DEDUP_OK;
}

template <class T>
dedup_status halloc(dedup_ctx* c, T** p, uint64_t count, unsigned flags = cudaHostAllocPortable) {
    if (count == 0) count = 1;
    cudaError_t e = cudaHostAlloc(reinterpret_cast<void**>(p), sizeof(T) * count, flags);
    if (e != cudaSuccess)
        return fail(c, DEDUP_ENOMEM, std::string("cudaHostAlloc: ") + cudaGetErrorString(e));
    return DEDUP_OK;
}

dedup_status ws_alloc(dedup_ctx* c, Workspace& w, uint64_t batch_bytes, uint64_t cap) {
    w.max_tiles = (batch_bytes + kSelTile - 1) / kSelTile + 1;
    // whole tiles: the scan writes every word of the last (partial) tile
    TRY(dalloc(c, &w.bitmap, w.max_tiles * kSelTileWords + 2));
    TRY(dalloc(c, &w.agg, w.max_tiles * 32));
    TRY(dalloc(c, &w.gagg, (select_groups(w.max_tiles) + 1) * 32));
    TRY(dalloc(c, &w.gentry, (select_groups(w.max_tiles) + 1) * 2));
    TRY(dalloc(c, &w.evbuf, event_words(w.max_tiles)));
    TRY(dalloc(c, &w.counters, 256));
    TRY(dalloc(c, &w.slot_idx, cap));
    TRY(dalloc(c, &w.sha_ws, sha1_ws_words(cap)));
    if (c->cfg.max_chunk || c->cfg.min_chunk != 32) {
        w.item_cap = cap;
        TRY(dalloc(c, &w.mc_ws, maxchunk_ws_words(cap, w.item_cap)));
    }
    CU(cudaMemset(w.counters, 0, sizeof(uint32_t) * 256));
    return DEDUP_OK;
}

void ws_free(Workspace& w) {
    cudaFree(w.bitmap);
    cudaFree(w.agg);
    cudaFree(w.gagg);
    cudaFree(w.gentry);
    cudaFree(w.evbuf);
    cudaFree(w.counters);
    cudaFree(w.slot_idx);
    cudaFree(w.sha_ws);
    cudaFree(w.mc_ws);
    w = Workspace{};
}

bool usable(const dedup_ctx* c) { return c != nullptr && c->sticky == DEDUP_OK; }

// dedup_op_* apply to a single-GPU ctx
#define NO_MG(c)                                                                        \
    do {                                                                                \
        if ((c)->mg) return fail(c, DEDUP_EUNSUPPORTED, "dedup_op_* need a single-GPU ctx"); \
    } while (0)


TableView table_view(const dedup_ctx* c) {
    const TableBuf& t = c->tables[c->cur_table];
    return TableView{t.slots, t.capacity - 1, t.status};
}

// Kernel sequence of rows A2-A4 for one batch described by *d (device).
void enqueue_chunk_sha(dedup_ctx* c, Workspace& w, cudaStream_t s, const BatchDesc* d,
                       uint64_t max_bytes, uint32_t* cut_pos, uint64_t cap, uint32_t* n_chunks,
                       uint8_t* digest, cudaEvent_t ev_scan, cudaEvent_t ev_chunk,
                       uint32_t* chunk_start, uint64_t* chunk_id, uint32_t* item_first,
                       uint32_t max_items) {
    launch_chunk_select(d, c->d_tab, c->cfg.anchor_mask, c->cfg.anchor_value, w.bitmap,
                            w.agg, w.gagg, w.gentry, w.evbuf,
                            (max_bytes + kSelTile - 1) / kSelTile, cut_pos, cap, n_chunks,
                            c->num_sms, s, ev_scan, c->cfg.max_chunk, w.mc_ws,
                            (uint32_t)w.item_cap, c->cfg.min_chunk);
    if (chunk_start)
        launch_chunk_meta(d, cut_pos, n_chunks, cap, chunk_start, chunk_id, item_first,
                          max_items, c->num_sms, s);
    if (ev_chunk) cudaEventRecordWithFlags(ev_chunk, s, cudaEventRecordExternal);
    if (digest)
        launch_sha1(d, max_bytes, cut_pos, n_chunks, cap, w.sha_ws, digest, c->num_sms, s,
                    c->cfg.sha_lane_bytes);
}

// Carry-over mode (row NEXT-2, csrc/carry.cu): the piece's rows A2-A4, chained
// to the previous slot's piece through its CarryState and three events.
// d_small: [0] reported chunks, [4..8] table status, [9] cuts, [10..12] extra.
void enqueue_carry_chunk_sha(dedup_ctx* c, Slot& sl, Slot& prev, cudaStream_t s, bool se) {
    const uint64_t cap = c->chunk_cap;
    uint32_t* n_cuts = sl.d_small + 9;
    cudaStreamWaitEvent(s, prev.ev_hist, cudaEventWaitExternal);
    launch_carry_hist(sl.d_desc, s);  // (the scan reads the previous piece's history)
    cudaEventRecordWithFlags(sl.ev_hist, s, cudaEventRecordExternal);
    launch_chunk_select(sl.d_desc, c->d_tab, c->cfg.anchor_mask, c->cfg.anchor_value,
                        sl.ws.bitmap, sl.ws.agg, sl.ws.gagg, sl.ws.gentry, sl.ws.evbuf,
                        (c->cfg.batch_bytes + kSelTile - 1) / kSelTile, sl.d_cut_pos, cap, n_cuts,
                        c->num_sms, s, se ? sl.ev_scan : nullptr, 0, nullptr, 0, 32, prev.ev_sel);
    launch_carry_meta(sl.d_desc, n_cuts, sl.d_cut_pos, cap, sl.d_small, sl.d_chunk_start,
                      sl.d_chunk_id, sl.d_item_first, sl.d_small + 10, s);
    cudaEventRecordWithFlags(sl.ev_sel, s, cudaEventRecordExternal);
    if (se) cudaEventRecordWithFlags(sl.ev_chunk, s, cudaEventRecordExternal);
    launch_sha1(sl.d_desc, c->cfg.batch_bytes, sl.d_cut_pos, n_cuts, cap, sl.ws.sha_ws,
                sl.d_digest, c->num_sms, s, c->cfg.sha_lane_bytes);
    cudaStreamWaitEvent(s, prev.ev_carry, cudaEventWaitExternal);
    launch_carry_cont(sl.d_desc, n_cuts, sl.d_cut_pos, cap, sl.d_digest, sl.d_small + 10, s);
    cudaEventRecordWithFlags(sl.ev_carry, s, cudaEventRecordExternal);
}

// Records the per-batch graph of slot i (capture of the slot's stream).
dedup_status build_graph(dedup_ctx* c, int i) {
    Slot& sl = c->slots[i];
    Slot& prev = c->slots[(i + c->slots.size() - 1) % c->slots.size()];
    const uint64_t cap = c->chunk_cap;
    cudaStream_t s = sl.stream;
    const bool se = c->stage_events;  // per-stage timing events (DEDUP_STAGE_EVENTS=0: off)
    const bool carry = c->cfg.carry_over != 0;
    CU(cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal));
    if (se) cudaEventRecordWithFlags(sl.ev_start, s, cudaEventRecordExternal);
    cudaMemcpyAsync(sl.d_desc, sl.h_desc, sizeof(BatchDesc), cudaMemcpyHostToDevice, s);
    cudaMemcpyAsync(sl.d_item_off, sl.h_item_off, sizeof(uint64_t) * (c->cfg.batch_items + 1),
                    cudaMemcpyHostToDevice, s);
    cudaMemsetAsync(sl.d_small, 0, sizeof(uint32_t) * 16, s);  // counts + batch statistics
    if (se) cudaEventRecordWithFlags(sl.ev_h2d, s, cudaEventRecordExternal);
    if (carry)
        enqueue_carry_chunk_sha(c, sl, prev, s, se);
    else
        enqueue_chunk_sha(c, sl.ws, s, sl.d_desc, c->cfg.batch_bytes, sl.d_cut_pos, cap,
                          sl.d_small, sl.d_digest, se ? sl.ev_scan : nullptr,
                          se ? sl.ev_chunk : nullptr, sl.d_chunk_start, sl.d_chunk_id,
                          sl.d_item_first, c->cfg.batch_items);
    if (se) cudaEventRecordWithFlags(sl.ev_sha, s, cudaEventRecordExternal);
    // table work waits for the previous batch's table work (global chain)
    cudaStreamWaitEvent(s, prev.ev_table, cudaEventWaitExternal);
    const TableView* tv = &sl.d_desc->table;
    launch_table_prepare(sl.d_desc, c->tables[0].capacity, c->num_sms, s);
    launch_table_insert(tv, sl.d_digest, sl.d_chunk_id, nullptr, sl.d_small, 0, cap,
                        sl.ws.slot_idx, c->num_sms, s);
    // (carry-over: the batch statistics are computed on the host, parse_slot)
    launch_table_lookup(tv, sl.d_chunk_id, nullptr, sl.d_small, 0, cap, sl.ws.slot_idx,
                            sl.d_first_id, sl.d_is_dup, sl.d_small + 4,
                            carry ? nullptr : sl.d_cut_pos, sl.d_desc, c->num_sms, s);
    cudaEventRecordWithFlags(sl.ev_table, s, cudaEventRecordExternal);
    launch_pack(sl.d_desc, sl.d_small, cap, c->cfg.batch_items, sl.d_chunk_start, sl.d_first_id,
                sl.d_digest, sl.d_is_dup, sl.d_item_first, sl.d_small + 4, sl.hdev, c->num_sms,
                s, carry ? sl.d_small + 10 : nullptr);
    cudaEventRecordWithFlags(sl.ev_done, s, cudaEventRecordExternal);
    cudaGraph_t g = nullptr;
    cudaError_t e = cudaStreamEndCapture(s, &g);
    if (e != cudaSuccess)
        return fail(c, DEDUP_ECUDA, std::string("graph capture: ") + cudaGetErrorString(e));
    size_t n_nodes = 0;
    cudaGraphGetNodes(g, nullptr, &n_nodes);
    std::vector<cudaGraphNode_t> nodes(n_nodes);
    cudaGraphGetNodes(g, nodes.data(), &n_nodes);
    uint32_t kern = 0;
    for (auto& nd : nodes) {
        cudaGraphNodeType ty;
        cudaGraphNodeGetType(nd, &ty);
        kern += ty == cudaGraphNodeTypeKernel ? 1 : 0;
    }
    c->graph_kernels = kern;
    e = cudaGraphInstantiate(&sl.graph, g, 0);
    cudaGraphDestroy(g);
    if (e != cudaSuccess)
        return fail(c, DEDUP_ECUDA, std::string("graph instantiate: ") + cudaGetErrorString(e));
    CU(cudaGraphUpload(sl.graph, s));  // keep the first launch off the critical path
    return DEDUP_OK;
}

dedup_status slot_alloc(dedup_ctx* c, Slot& sl) {
    const dedup_config& g = c->cfg;
    const uint64_t cap = c->chunk_cap;
    CU(cudaStreamCreateWithFlags(&sl.stream, cudaStreamNonBlocking));
    for (cudaEvent_t* e : {&sl.ev_host, &sl.ev_start, &sl.ev_h2d, &sl.ev_scan, &sl.ev_chunk,
                           &sl.ev_sha, &sl.ev_table, &sl.ev_done})
        CU(cudaEventCreate(e));
    CU(cudaEventCreateWithFlags(&sl.ev_prod, cudaEventDisableTiming));
    for (cudaEvent_t* e : {&sl.ev_hist, &sl.ev_sel, &sl.ev_carry})
        CU(cudaEventCreateWithFlags(e, cudaEventDisableTiming));
    TRY(dalloc(c, &sl.d_desc, 1));
    TRY(halloc(c, &sl.h_desc, 1));
    std::memset(sl.h_desc, 0, sizeof(BatchDesc));
    if (g.host_fed) TRY(dalloc(c, &sl.d_bytes, g.batch_bytes + 256));
    TRY(dalloc(c, &sl.d_item_off, (uint64_t)g.batch_items + 1));
    TRY(halloc(c, &sl.h_item_off, (uint64_t)g.batch_items + 1));
    TRY(ws_alloc(c, sl.ws, g.batch_bytes, cap));
    TRY(dalloc(c, &sl.d_cut_pos, cap));
    TRY(dalloc(c, &sl.d_chunk_start, cap));
    TRY(dalloc(c, &sl.d_item_first, g.batch_items));
    TRY(dalloc(c, &sl.d_small, 16));
    TRY(dalloc(c, &sl.d_chunk_id, cap));
    TRY(dalloc(c, &sl.d_first_id, cap));
    TRY(dalloc(c, &sl.d_digest, cap * 20));
    TRY(dalloc(c, &sl.d_is_dup, cap));
    // results: header 64 B | chunk_start 4*cap | first_id 8*cap | digest 20*cap | is_dup cap
    //          | item_first 4*items
    const uint64_t o_cs = 64, o_fid = o_cs + ((4 * cap + 63) & ~63ull),
                   o_dg = o_fid + 8 * cap, o_dup = o_dg + 20 * cap,
                   o_if = (o_dup + cap + 63) & ~63ull, total = o_if + 4ull * g.batch_items + 64;
    TRY(halloc(c, &sl.h_res, total, cudaHostAllocMapped | cudaHostAllocPortable));
    uint8_t* dres = nullptr;
    CU(cudaHostGetDevicePointer(reinterpret_cast<void**>(&dres), sl.h_res, 0));
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
    return DEDUP_OK;
}

void slot_free(Slot& sl) {
    if (sl.stream) cudaStreamSynchronize(sl.stream);
    if (sl.graph) cudaGraphExecDestroy(sl.graph);
    for (cudaEvent_t e : {sl.ev_host, sl.ev_start, sl.ev_h2d, sl.ev_scan, sl.ev_chunk, sl.ev_sha,
                          sl.ev_table, sl.ev_done, sl.ev_prod, sl.ev_hist, sl.ev_sel, sl.ev_carry})
        if (e) cudaEventDestroy(e);
    cudaFree(sl.d_desc);
    if (sl.h_desc) cudaFreeHost(sl.h_desc);
    cudaFree(sl.d_bytes);
    cudaFree(sl.d_item_off);
    if (sl.h_item_off) cudaFreeHost(sl.h_item_off);
    ws_free(sl.ws);
    cudaFree(sl.d_cut_pos);
    cudaFree(sl.d_chunk_start);
    cudaFree(sl.d_item_first);
    cudaFree(sl.d_small);
    cudaFree(sl.d_chunk_id);
    cudaFree(sl.d_first_id);
    cudaFree(sl.d_digest);
    cudaFree(sl.d_is_dup);
    if (sl.h_res) cudaFreeHost(sl.h_res);
    if (sl.h_bounce) cudaFreeHost(sl.h_bounce);
    if (sl.stream) cudaStreamDestroy(sl.stream);
    sl = Slot{};
}

// Carry-over flags of the next piece (nbytes long); a non-empty piece starts
// (or continues) the stream's chunking domain.
uint32_t carry_flags(dedup_ctx* c, uint64_t nbytes) {
    if (!c->cfg.carry_over) return 0;
    const uint32_t f = kCarryMode | (c->carry_started ? kCarryCont : 0u);
    if (nbytes > 0) c->carry_started = true;
    return f;
}

// Prepare slot i's descriptor for a batch and launch its graph.
dedup_status launch_batch(dedup_ctx* c, int i, const uint8_t* d_bytes, uint32_t carry = 0) {
    Slot& sl = c->slots[i];
    BatchDesc& d = *sl.h_desc;
    d.carry = carry;
    d.bytes = d_bytes;
    d.nbytes = sl.nbytes;
    d.first_seq = sl.first_seq;
    d.item_off = sl.d_item_off;
    d.n_items = sl.n_items;
    d.fresh = c->stream_fresh ? 1u : 0u;
    d.table = table_view(c);
    c->stream_fresh = false;
    if (c->cfg.carry_over) {
        const int np = (int)c->slots.size();
        d.carry_in = c->d_carry + (i + np - 1) % np;
        d.carry_out = c->d_carry + i;
        // (carry flags: set by the submitting call)
    }
    const auto t0 = std::chrono::steady_clock::now();
    CU(cudaGraphLaunch(sl.graph, sl.stream));
    c->st.ms_host_launch +=
        std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    c->launches += c->graph_kernels;
    sl.busy = true;
    sl.parsed = false;
    sl.next_item = 0;
    c->next_slot = (uint32_t)((i + 1) % c->slots.size());
    c->inflight.push_back(i);
    c->pending_items += sl.n_items;
    c->st.batches += 1;
    return DEDUP_OK;
}

dedup_status check_cfg(const dedup_config* g) {
    if (g == nullptr || g->struct_size != sizeof(dedup_config)) return DEDUP_EINVAL;
    if (g->window == 0 || g->window > 64 || g->min_chunk < g->window) return DEDUP_EINVAL;
    if (g->max_chunk != 0 && g->max_chunk < g->min_chunk) return DEDUP_EINVAL;
    if (g->slots < 1 || g->slots > 64 || g->batch_items < 1) return DEDUP_EINVAL;
    if (g->batch_bytes < 1 || g->batch_bytes > (1ull << 30)) return DEDUP_EINVAL;
    if (g->num_owners < 1 || g->num_owners > 64 || g->owner_rank >= g->num_owners)
        return DEDUP_EINVAL;
    if (g->table_capacity < 1 || g->table_capacity > (1ull << 31)) return DEDUP_EINVAL;
    if (g->num_devices > 64 || g->transport > 3) return DEDUP_EINVAL;
    if (g->carry_over && (mg::wanted(g) || g->min_chunk != 32 || g->max_chunk != 0 ||
                          g->slots < 2 || g->num_owners != 1))
        return DEDUP_EUNSUPPORTED;  // carry-over: single-GPU engine, the 32-state selection
    if (mg::wanted(g) && (g->owner_rank != 0 || g->num_owners != 1)) return DEDUP_EINVAL;
    if (g->sha_lane_bytes != 0 && (g->sha_lane_bytes < 64 || g->sha_lane_bytes > (1u << 24)))
        return DEDUP_EINVAL;
    // max_chunk and min_chunk > window (NEXT-2): selected by maxchunk.cu's walk
    if (g->window != 32) return DEDUP_EUNSUPPORTED;
    if (g->max_chunk != 0 && g->max_chunk < 64) return DEDUP_EUNSUPPORTED;
    return DEDUP_OK;
}

// Turn a completed slot's host results into per-item views + stats.
dedup_status parse_slot(dedup_ctx* c, Slot& sl) {
    const auto t_parse = std::chrono::steady_clock::now();
    const uint32_t n = sl.hhost.header[0];
    if (sl.hhost.header[1] != 0)
        return fail(c, DEDUP_ETABLEFULL, "digest table overflow: raise table_capacity");
    if (n > c->chunk_cap) return fail(c, DEDUP_ECUDA, "chunk capacity exceeded");
    sl.item_first.assign(sl.n_items, 0);
    sl.item_n.assign(sl.n_items, 0);
    uint32_t next = n;
    for (int64_t k = (int64_t)sl.n_items - 1; k >= 0; --k) {
        const uint32_t f = sl.hhost.item_first_chunk[k];
        if (f == 0xFFFFFFFFu) {
            sl.item_first[k] = next;
            sl.item_n[k] = 0;
        } else {
            sl.item_first[k] = f;
            sl.item_n[k] = next - f;
            next = f;
        }
    }
    // batch statistics reduced on the device by the lookup kernel
    uint64_t dups = sl.hhost.header[3], dup_bytes = sl.hhost.header[4];
    c->st.sha1_blocks += sl.hhost.header[5];
    sl.carried = 0;
    if (c->cfg.carry_over) {
        // one piece: chunk 0 may continue from earlier pieces (carried bytes);
        // the last reported chunk ends at header[8] (the open chunk's start)
        const HostResultLayout& h = sl.hhost;
        const uint64_t carried = (uint64_t)h.header[6] | ((uint64_t)h.header[7] << 32);
        sl.carried = carried > 0xFFFFFFFFull ? 0xFFFFFFFFu : (uint32_t)carried;
        dups = dup_bytes = 0;
        for (uint32_t r = 0; r < n; ++r) {
            const uint64_t e = r + 1 < n ? h.chunk_start[r + 1] : h.header[8];
            const uint64_t len = e - h.chunk_start[r] + (r == 0 ? carried : 0);
            c->st.sha1_blocks += (len + 9 + 63) / 64;
            if (h.is_dup[r]) {
                ++dups;
                dup_bytes += len;
            }
        }
    }
    c->st.chunks += n;
    c->st.dup_chunks += dups;
    c->st.unique_chunks += n - dups;
    c->st.dup_bytes += dup_bytes;
    c->st.items += sl.n_items;
    c->st.bytes += sl.nbytes;
    c->st.table_used = sl.hhost.header[2];
    // CUDA-event stage times of every time_every-th batch (event queries cost
    // host time, so they are sampled; timed_batches counts the samples)
    if (c->stage_events && c->parsed_batches++ % c->time_every == 0) {
        float ms = 0;
        c->st.timed_batches += 1;
        c->st.timed_bytes += sl.nbytes;
        if (sl.host_fed && cudaEventElapsedTime(&ms, sl.ev_host, sl.ev_start) == cudaSuccess)
            c->st.ms_h2d += ms;
        if (cudaEventElapsedTime(&ms, sl.ev_h2d, sl.ev_scan) == cudaSuccess) c->st.ms_scan += ms;
        if (cudaEventElapsedTime(&ms, sl.ev_scan, sl.ev_chunk) == cudaSuccess)
            c->st.ms_select += ms;
        if (cudaEventElapsedTime(&ms, sl.ev_chunk, sl.ev_sha) == cudaSuccess) c->st.ms_sha1 += ms;
        if (cudaEventElapsedTime(&ms, sl.ev_sha, sl.ev_table) == cudaSuccess)
            c->st.ms_table += ms;
        if (cudaEventElapsedTime(&ms, sl.ev_table, sl.ev_done) == cudaSuccess) c->st.ms_d2h += ms;
        c->st.timed_sha1_blocks += sl.hhost.header[5];
    }
    if (c->trace && c->stage_events) {  // DEDUP_TRACE=1: per-batch event timeline (ms)
        // host: the items' H2D starts at `host` (host-fed batches; else = start)
        float t[8] = {0, 0, 0, 0, 0, 0, 0, 0};
        const cudaEvent_t ev[8] = {sl.host_fed ? sl.ev_host : sl.ev_start, sl.ev_start,
                                   sl.ev_h2d, sl.ev_scan, sl.ev_chunk, sl.ev_sha, sl.ev_table,
                                   sl.ev_done};
        for (int k = 0; k < 8; ++k) cudaEventElapsedTime(&t[k], c->ev_ref, ev[k]);
        std::fprintf(stderr,
                     "trace seq=%llu bytes=%llu host=%.3f start=%.3f h2d=%.3f scan=%.3f "
                     "chunk=%.3f sha=%.3f table=%.3f done=%.3f\n",
                     (unsigned long long)sl.first_seq, (unsigned long long)sl.nbytes, t[0], t[1],
                     t[2], t[3], t[4], t[5], t[6], t[7]);
    }
    cudaGetLastError();  // clear a possible error from a timing query
    sl.parsed = true;
    c->st.ms_host_parse +=
        std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t_parse)
            .count();
    return DEDUP_OK;
}

// Descriptor for one dedup_op_* call: next entry of the pinned/device ring.
dedup_status op_desc(dedup_ctx* c, cudaStream_t s, const BatchDesc& h, const BatchDesc** out) {
    const int k = c->op_next;
    c->op_next = (k + 1) % kOpRing;
    if (c->op_ev_used[k]) CU(cudaEventSynchronize(c->op_ev[k]));
    c->op_h_desc[k] = h;
    CU(cudaMemcpyAsync(c->op_d_desc + k, c->op_h_desc + k, sizeof(BatchDesc),
                       cudaMemcpyHostToDevice, s));
    CU(cudaEventRecord(c->op_ev[k], s));
    c->op_ev_used[k] = true;
    *out = c->op_d_desc + k;
    return DEDUP_OK;
}

}  // namespace

extern "C" {

void dedup_config_default(dedup_config* g) {
    std::memset(g, 0, sizeof(*g));
    g->struct_size = sizeof(dedup_config);
    g->window = 32;
    g->poly = 0x45C2B6A1u;
    g->anchor_mask = 0xFFFu;
    g->anchor_value = 0;
    g->min_chunk = 32;
    g->max_chunk = 0;
    g->device = 0;
    g->slots = 4;
    g->batch_items = 4096;
    g->batch_bytes = 64ull << 20;
    g->table_capacity = 1ull << 20;
    g->owner_rank = 0;
    g->num_owners = 1;
    g->host_fed = 1;
}

dedup_status dedup_init(const dedup_config* cfg, dedup_ctx** out) {
    if (out == nullptr) return DEDUP_EINVAL;
    *out = nullptr;
    dedup_status s = check_cfg(cfg);
    if (s != DEDUP_OK) return s;
    dedup_ctx* c = new dedup_ctx();
    c->cfg = *cfg;
    if (mg::wanted(cfg)) {  // G ranks, one worker thread per rank (mg.cpp)
        const char* why = nullptr;
        s = mg::create(cfg, &c->mg, &why);
        if (s != DEDUP_OK) {
            std::fprintf(stderr, "dedup_init (multi-GPU): %s\n", why ? why : "failed");
            delete c;
            return s;
        }
        c->cfg.device_ids = nullptr;  // not retained
        *out = c;
        return DEDUP_OK;
    }
    auto bail = [&](dedup_status r) {
        dedup_destroy(c);
        return r;
    };
    if (cudaSetDevice(cfg->device) != cudaSuccess) return bail(DEDUP_ECUDA);
    if (cudaDeviceGetAttribute(&c->num_sms, cudaDevAttrMultiProcessorCount, cfg->device) !=
        cudaSuccess)
        return bail(DEDUP_ECUDA);
    set_pipeline_carveout();
    for (const char* bad : {chunk_unlaunchable(), sha1_unlaunchable()}) {
        if (bad) {
            std::fprintf(stderr, "dedup_init: %s cannot launch on device %d\n", bad,
                         cfg->device);
            return bail(DEDUP_ECUDA);
        }
    }
    c->chunk_cap = cfg->batch_bytes / 32 + cfg->batch_items + 2;
    uint32_t tab[512];
    rabin_tables(cfg->poly, tab);
    if ((s = dalloc(c, &c->d_tab, 512)) != DEDUP_OK) return bail(s);
    if (cudaMemcpy(c->d_tab, tab, sizeof(tab), cudaMemcpyHostToDevice) != cudaSuccess)
        return bail(DEDUP_ECUDA);
    for (TableBuf& t : c->tables) {
        t.capacity = next_pow2(2 * cfg->table_capacity);
        if ((s = dalloc(c, &t.slots, t.capacity)) != DEDUP_OK) return bail(s);
        if ((s = dalloc(c, &t.status, 4)) != DEDUP_OK) return bail(s);
        if (cudaMemset(t.slots, 0, sizeof(TableSlot) * t.capacity) != cudaSuccess ||
            cudaMemset(t.status, 0, 16) != cudaSuccess)
            return bail(DEDUP_ECUDA);
    }
    if ((s = ws_alloc(c, c->op_ws, cfg->batch_bytes, c->chunk_cap)) != DEDUP_OK) return bail(s);
    if (cfg->carry_over) {
        if ((s = dalloc(c, &c->d_carry, cfg->slots)) != DEDUP_OK) return bail(s);
        if (cudaMemset(c->d_carry, 0, sizeof(CarryState) * cfg->slots) != cudaSuccess)
            return bail(DEDUP_ECUDA);
    }
    if ((s = dalloc(c, &c->op_d_desc, kOpRing)) != DEDUP_OK) return bail(s);
    if ((s = halloc(c, &c->op_h_desc, kOpRing)) != DEDUP_OK) return bail(s);
    for (cudaEvent_t& e : c->op_ev)
        if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess)
            return bail(DEDUP_ECUDA);
    if (const char* v = std::getenv("DEDUP_STAGE_EVENTS")) c->stage_events = std::atoi(v) != 0;
    if (const char* v = std::getenv("DEDUP_TIME_EVERY"))
        c->time_every = std::atoi(v) > 0 ? (uint32_t)std::atoi(v) : 1u;
    c->slots.resize(cfg->slots);
    for (Slot& sl : c->slots)
        if ((s = slot_alloc(c, sl)) != DEDUP_OK) return bail(s);
    for (size_t i = 0; i < c->slots.size(); ++i)
        if ((s = build_graph(c, (int)i)) != DEDUP_OK) return bail(s);
    if (cudaDeviceSynchronize() != cudaSuccess) return bail(DEDUP_ECUDA);
    c->st.table_slots = c->tables[0].capacity;
    c->st.num_owners = cfg->num_owners;
    c->st.owner_rank = cfg->owner_rank;
    c->trace = std::getenv("DEDUP_TRACE") != nullptr;
    if (cudaEventCreate(&c->ev_ref) != cudaSuccess || cudaEventRecord(c->ev_ref, 0) != cudaSuccess)
        return bail(DEDUP_ECUDA);
    *out = c;
    return DEDUP_OK;
}

void dedup_destroy(dedup_ctx* c) {
    if (c == nullptr) return;
    if (c->mg) {
        mg::destroy(c->mg);
        delete c;
        return;
    }
    cudaSetDevice(c->cfg.device);
    for (Slot& sl : c->slots) slot_free(sl);
    ws_free(c->op_ws);
    cudaDeviceSynchronize();
    for (cudaEvent_t e : c->op_ev)
        if (e) cudaEventDestroy(e);
    cudaFree(c->op_d_desc);
    if (c->op_h_desc) cudaFreeHost(c->op_h_desc);
    for (TableBuf& t : c->tables) {
        cudaFree(t.slots);
        cudaFree(t.status);
    }
    cudaFree(c->local.slots);
    cudaFree(c->local.status);
    cudaFree(c->d_local_view);
    cudaFree(c->d_tab);
    cudaFree(c->d_carry);
    if (c->ev_ref) cudaEventDestroy(c->ev_ref);
    delete c;
}

const char* dedup_last_error(const dedup_ctx* c) {
    if (c != nullptr && c->mg && c->err == "no error") return mg::last_error(c->mg);
    return c == nullptr ? "null ctx" : c->err.c_str();
}

dedup_status dedup_submit_batch(dedup_ctx* c, uint32_t n_items, const uint8_t* const* item_ptr,
                                const uint64_t* item_len, uint64_t* first_seq_out) {
    if (c == nullptr) return DEDUP_EINVAL;
    if (c->mg) return mg::submit_host(c->mg, n_items, item_ptr, item_len, first_seq_out);
    if (!usable(c)) return c->sticky;
    if (!c->cfg.host_fed) return fail(c, DEDUP_EINVAL, "ctx was created with host_fed = 0");
    if (c->cfg.num_owners != 1)
        return fail(c, DEDUP_EUNSUPPORTED, "num_owners > 1: use the dedup_op_* orchestration");
    if (n_items > 0 && (item_ptr == nullptr || item_len == nullptr))
        return fail(c, DEDUP_EINVAL, "null item arrays");
    CU(cudaSetDevice(c->cfg.device));
    // plan batches of whole items
    std::vector<std::pair<uint32_t, uint32_t>> plan;
    uint32_t b0 = 0;
    uint64_t bytes = 0;
    for (uint32_t k = 0; k < n_items; ++k) {
        const uint64_t L = item_len[k];
        if (L > c->cfg.batch_bytes || L > 0xFFFFFFFFull)
            return fail(c, DEDUP_EINVAL, "item larger than batch_bytes");
        if (L > 0 && item_ptr[k] == nullptr) return fail(c, DEDUP_EINVAL, "null item pointer");
        // (carry-over: one piece per batch)
        if (k > b0 && (bytes + L > c->cfg.batch_bytes || k - b0 >= c->cfg.batch_items ||
                       c->cfg.carry_over)) {
            plan.emplace_back(b0, k);
            b0 = k;
            bytes = 0;
        }
        bytes += L;
    }
    if (n_items > b0) plan.emplace_back(b0, n_items);
    // round-robin slots must all be free (carry-over: and the slot after the
    // last, whose batch reads the state the last one overwrites)
    const size_t need = plan.size() + (c->cfg.carry_over && !plan.empty() ? 1 : 0);
    for (size_t j = 0; j < need; ++j)
        if (j >= c->slots.size() || c->slots[(c->next_slot + j) % c->slots.size()].busy)
            return fail(c, DEDUP_EAGAIN, "no free batch slot");
    if (first_seq_out) *first_seq_out = c->next_seq;
    for (auto& r : plan) {
        const int i = (int)c->next_slot;
        Slot& sl = c->slots[i];
        sl.host_fed = true;
        sl.first_seq = c->next_seq;
        sl.n_items = r.second - r.first;
        sl.item_len.assign(item_len + r.first, item_len + r.second);
        uint64_t off = 0;
        sl.h_item_off[0] = 0;
        for (uint32_t k = 0; k < sl.n_items; ++k) sl.h_item_off[k + 1] = (off += sl.item_len[k]);
        sl.nbytes = off;
        CU(cudaEventRecord(sl.ev_host, sl.stream));
        // H2D of the items (row A1), merging contiguous host ranges
        uint32_t k = 0;
        while (k < sl.n_items) {
            const uint8_t* p = item_ptr[r.first + k];
            const uint64_t dst = sl.h_item_off[k];
            uint64_t len = sl.item_len[k];
            uint32_t j = k + 1;
            while (j < sl.n_items && item_ptr[r.first + j] == p + len) len += sl.item_len[j++];
            if (len) {
                cudaPointerAttributes pa{};
                const bool locked = cudaPointerGetAttributes(&pa, p) == cudaSuccess &&
                                    pa.type == cudaMemoryTypeHost;
                cudaGetLastError();
                if (!locked) {  // pageable: through the slot's page-locked bounce buffer
                    if (sl.h_bounce == nullptr)
                        TRY(halloc(c, &sl.h_bounce, c->cfg.batch_bytes));
                    std::memcpy(sl.h_bounce + dst, p, len);
                    p = sl.h_bounce + dst;
                }
                CU(cudaMemcpyAsync(sl.d_bytes + dst, p, len, cudaMemcpyHostToDevice, sl.stream));
            }
            k = j;
        }
        TRY(launch_batch(c, i, sl.d_bytes, carry_flags(c, sl.nbytes)));
        c->next_seq += sl.n_items;
    }
    return DEDUP_OK;
}

dedup_status dedup_submit_device(dedup_ctx* c, const uint8_t* d_bytes, uint64_t nbytes,
                                 const uint64_t* item_off, uint32_t n_items, void* producer,
                                 uint64_t* first_seq_out) {
    if (c == nullptr) return DEDUP_EINVAL;
    if (c->mg)
        return mg::submit_device(c->mg, d_bytes, nbytes, item_off, n_items, producer,
                                 first_seq_out);
    if (!usable(c)) return c->sticky;
    if (c->cfg.num_owners != 1)
        return fail(c, DEDUP_EUNSUPPORTED, "num_owners > 1: use the dedup_op_* orchestration");
    if (item_off == nullptr || (nbytes > 0 && d_bytes == nullptr))
        return fail(c, DEDUP_EINVAL, "null argument");
    if (reinterpret_cast<uintptr_t>(d_bytes) & 15)
        return fail(c, DEDUP_EINVAL, "d_bytes must be 16-byte aligned");
    if (nbytes > c->cfg.batch_bytes || n_items > c->cfg.batch_items)
        return fail(c, DEDUP_EINVAL, "batch larger than batch_bytes / batch_items");
    if (item_off[0] != 0 || item_off[n_items] != nbytes)
        return fail(c, DEDUP_EINVAL, "item_off must start at 0 and end at nbytes");
    for (uint32_t k = 0; k < n_items; ++k)
        if (item_off[k + 1] < item_off[k]) return fail(c, DEDUP_EINVAL, "item_off decreasing");
    const int i = (int)c->next_slot;
    if (c->slots[i].busy) return fail(c, DEDUP_EAGAIN, "no free batch slot");
    if (c->cfg.carry_over) {
        if (n_items != 1) return fail(c, DEDUP_EINVAL, "carry-over: one piece per batch");
        if (c->slots[(i + 1) % c->slots.size()].busy)
            return fail(c, DEDUP_EAGAIN, "no free batch slot");
    }
    CU(cudaSetDevice(c->cfg.device));
    Slot& sl = c->slots[i];
    sl.host_fed = false;
    sl.first_seq = c->next_seq;
    sl.n_items = n_items;
    sl.nbytes = nbytes;
    sl.item_len.resize(n_items);
    for (uint32_t k = 0; k < n_items; ++k) sl.item_len[k] = item_off[k + 1] - item_off[k];
    std::memcpy(sl.h_item_off, item_off, sizeof(uint64_t) * (n_items + 1));
    CU(cudaEventRecord(sl.ev_prod, static_cast<cudaStream_t>(producer)));
    CU(cudaStreamWaitEvent(sl.stream, sl.ev_prod, 0));
    if (first_seq_out) *first_seq_out = c->next_seq;
    TRY(launch_batch(c, i, d_bytes, carry_flags(c, nbytes)));
    c->next_seq += n_items;
    return DEDUP_OK;
}

dedup_status dedup_join(dedup_ctx* c, void* stream) {
    if (c == nullptr) return DEDUP_EINVAL;
    if (c->mg) return mg::join(c->mg, stream);
    if (!usable(c)) return c->sticky;
    CU(cudaSetDevice(c->cfg.device));
    for (int i : c->inflight)
        CU(cudaStreamWaitEvent(static_cast<cudaStream_t>(stream), c->slots[i].ev_done, 0));
    return DEDUP_OK;
}

dedup_status dedup_end_stream(dedup_ctx* c) {
    if (c == nullptr) return DEDUP_EINVAL;
    if (c->mg) return mg::end_stream(c->mg);
    if (!usable(c)) return c->sticky;
    if (c->cfg.carry_over && c->carry_started) {
        // the closing batch: an empty piece that reports the stream's last
        // (open) chunk, checked against the stream's table
        const int i = (int)c->next_slot;
        if (c->slots[i].busy || c->slots[(i + 1) % c->slots.size()].busy)
            return fail(c, DEDUP_EAGAIN, "no free batch slot for the closing batch");
        CU(cudaSetDevice(c->cfg.device));
        Slot& sl = c->slots[i];
        sl.host_fed = false;
        sl.first_seq = c->next_seq;
        sl.n_items = 1;
        sl.nbytes = 0;
        sl.item_len.assign(1, 0);
        sl.h_item_off[0] = sl.h_item_off[1] = 0;
        TRY(launch_batch(c, i, reinterpret_cast<const uint8_t*>(c->d_tab),
                         kCarryMode | kCarryCont | kCarryClose));
        c->next_seq += 1;
        c->carry_started = false;
    }
    c->cur_table ^= 1;
    c->stream_fresh = true;
    return DEDUP_OK;
}

dedup_status dedup_drain(dedup_ctx* c, uint32_t max_items, int32_t wait_ms,
                         dedup_item_result* out, uint32_t* n_out) {
    if (c == nullptr || n_out == nullptr || (max_items > 0 && out == nullptr)) return DEDUP_EINVAL;
    *n_out = 0;
    if (c->mg) return mg::drain(c->mg, max_items, wait_ms, out, n_out);
    if (!usable(c)) return c->sticky;
    CU(cudaSetDevice(c->cfg.device));
    for (int i : c->to_release) c->slots[i].busy = false;
    c->to_release.clear();
    uint32_t got = 0;
    const auto deadline = std::chrono::steady_clock::now() + std::chrono::milliseconds(wait_ms);
    while (got < max_items && !c->inflight.empty()) {
        const int i = c->inflight.front();
        Slot& sl = c->slots[i];
        if (!sl.parsed) {
            cudaError_t q = cudaEventQuery(sl.ev_done);
            if (q == cudaErrorNotReady) {
                if (got > 0 || wait_ms == 0) break;
                if (wait_ms < 0) {
                    q = cudaEventSynchronize(sl.ev_done);
                } else {
                    while ((q = cudaEventQuery(sl.ev_done)) == cudaErrorNotReady &&
                           std::chrono::steady_clock::now() < deadline)
                        std::this_thread::sleep_for(std::chrono::microseconds(20));
                    if (q == cudaErrorNotReady)
                        return fail(c, DEDUP_ETIMEDOUT, "no batch completed within wait_ms");
                }
            }
            if (q != cudaSuccess)
                return fail(c, DEDUP_ECUDA, std::string("batch failed: ") + cudaGetErrorString(q));
            TRY(parse_slot(c, sl));
        }
        while (got < max_items && sl.next_item < sl.n_items) {
            const uint32_t k = sl.next_item++;
            dedup_item_result& r = out[got++];
            r.seq = sl.first_seq + k;
            r.item_len = sl.item_len[k];
            r.n_chunks = sl.item_n[k];
            r.carried = sl.carried;
            if (r.n_chunks) {
                const uint32_t f = sl.item_first[k];
                r.chunk_start = sl.hhost.chunk_start + f;
                r.digest = sl.hhost.digest + 20ull * f;
                r.is_dup = sl.hhost.is_dup + f;
                r.first_id = sl.hhost.first_id + f;
            } else {
                r.chunk_start = nullptr;
                r.digest = nullptr;
                r.is_dup = nullptr;
                r.first_id = nullptr;
            }
            --c->pending_items;
        }
        if (sl.next_item == sl.n_items) {
            c->inflight.pop_front();
            c->to_release.push_back(i);  // results stay valid until the next drain
        }
    }
    *n_out = got;
    return DEDUP_OK;
}

uint64_t dedup_pending(const dedup_ctx* c) {
    if (c && c->mg) return mg::pending(c->mg);
    return c ? c->pending_items : 0;
}

int32_t dedup_next_device(const dedup_ctx* c) {
    if (c == nullptr) return -1;
    return c->mg ? mg::next_device(c->mg) : c->cfg.device;
}

dedup_status dedup_stats(const dedup_ctx* c, dedup_stats_t* out) {
    if (c == nullptr || out == nullptr) return DEDUP_EINVAL;
    if (c->mg) return mg::stats(c->mg, out);
    *out = c->st;
    out->kernel_launches = c->launches;
    out->num_devices = 1;
    return DEDUP_OK;
}

void* dedup_host_alloc(dedup_ctx* c, size_t bytes) {
    if (c == nullptr) return nullptr;
    if (!c->mg) cudaSetDevice(c->cfg.device);
    void* p = nullptr;
    if (cudaHostAlloc(&p, bytes, cudaHostAllocPortable) != cudaSuccess) return nullptr;
    return p;
}

void dedup_host_free(dedup_ctx* c, void* p) {
    (void)c;
    if (p) cudaFreeHost(p);
}

uint64_t dedup_kernel_launches(const dedup_ctx* c) {
    if (c && c->mg) return mg::kernel_launches(c->mg);
    return c ? c->launches : 0;
}

// ---------------------------------------------------------------------------
// Stream-ordered device operations
// ---------------------------------------------------------------------------
dedup_status dedup_op_chunk(dedup_ctx* c, void* stream, const uint8_t* d_bytes, uint64_t nbytes,
                            const uint64_t* d_item_off, uint32_t n_items, uint32_t* d_cut_pos,
                            uint64_t cap, uint32_t* d_n_chunks) {
    if (c == nullptr) return DEDUP_EINVAL;
    NO_MG(c);
    if (!usable(c)) return c->sticky;
    if (nbytes > c->cfg.batch_bytes) return fail(c, DEDUP_EINVAL, "nbytes > batch_bytes");
    if (reinterpret_cast<uintptr_t>(d_bytes) & 15)
        return fail(c, DEDUP_EINVAL, "d_bytes must be 16-byte aligned");
    if ((c->cfg.max_chunk || c->cfg.min_chunk != 32) && n_items > c->op_ws.item_cap)
        return fail(c, DEDUP_EINVAL, "n_items larger than the max_chunk workspace");
    CU(cudaSetDevice(c->cfg.device));
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    BatchDesc h{};
    h.bytes = d_bytes;
    h.nbytes = nbytes;
    h.item_off = d_item_off;
    h.n_items = n_items;
    const BatchDesc* d = nullptr;
    TRY(op_desc(c, s, h, &d));
    enqueue_chunk_sha(c, c->op_ws, s, d, nbytes, d_cut_pos, cap, d_n_chunks, nullptr, nullptr,
                      nullptr, nullptr, nullptr, nullptr, 0);
    c->launches += 4;
    CU(cudaGetLastError());
    return DEDUP_OK;
}

dedup_status dedup_op_chunk_meta(dedup_ctx* c, void* stream, const uint64_t* d_item_off,
                                 uint32_t n_items, const uint32_t* d_cut_pos,
                                 const uint32_t* d_n_chunks, uint64_t cap, uint64_t first_seq,
                                 uint32_t* d_chunk_start, uint64_t* d_chunk_id,
                                 uint32_t* d_item_first_chunk) {
    if (c == nullptr) return DEDUP_EINVAL;
    NO_MG(c);
    if (!usable(c)) return c->sticky;
    CU(cudaSetDevice(c->cfg.device));
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    BatchDesc h{};
    h.item_off = d_item_off;
    h.n_items = n_items;
    h.first_seq = first_seq;
    const BatchDesc* d = nullptr;
    TRY(op_desc(c, s, h, &d));
    launch_chunk_meta(d, d_cut_pos, d_n_chunks, cap, d_chunk_start, d_chunk_id,
                      d_item_first_chunk, n_items, c->num_sms, s);
    c->launches += 1;
    CU(cudaGetLastError());
    return DEDUP_OK;
}

dedup_status dedup_op_sha1(dedup_ctx* c, void* stream, const uint8_t* d_bytes, uint64_t nbytes,
                           const uint32_t* d_cut_pos, const uint32_t* d_n_chunks, uint64_t cap,
                           uint8_t* d_digest) {
    if (c == nullptr) return DEDUP_EINVAL;
    if (!usable(c)) return c->sticky;
    if (reinterpret_cast<uintptr_t>(d_bytes) & 15)
        return fail(c, DEDUP_EINVAL, "d_bytes must be 16-byte aligned");
    if (reinterpret_cast<uintptr_t>(d_digest) & 3)
        return fail(c, DEDUP_EINVAL, "d_digest must be 4-byte aligned");
    if (nbytes > c->cfg.batch_bytes) return fail(c, DEDUP_EINVAL, "nbytes > batch_bytes");
    CU(cudaSetDevice(c->cfg.device));
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    BatchDesc h{};
    h.bytes = d_bytes;
    h.nbytes = nbytes;
    const BatchDesc* d = nullptr;
    TRY(op_desc(c, s, h, &d));
    if (cap > c->chunk_cap) return fail(c, DEDUP_EINVAL, "cap larger than the ctx workspace");
    launch_sha1(d, nbytes, d_cut_pos, d_n_chunks, cap, c->op_ws.sha_ws, d_digest, c->num_sms, s,
                c->cfg.sha_lane_bytes);
    c->launches += 2;
    CU(cudaGetLastError());
    return DEDUP_OK;
}

dedup_status dedup_op_findmatch(dedup_ctx* c, void* stream, const uint8_t* d_bytes,
                                uint64_t nbytes, const uint32_t* d_start,
                                const uint32_t* d_n_blocks, uint64_t cap, const uint8_t* d_skip,
                                uint32_t window, uint32_t max_coded, uint8_t* d_match_len,
                                uint16_t* d_match_off) {
    if (c == nullptr) return DEDUP_EINVAL;
    NO_MG(c);
    if (!usable(c)) return c->sticky;
    if (reinterpret_cast<uintptr_t>(d_bytes) & 15)
        return fail(c, DEDUP_EINVAL, "d_bytes must be 16-byte aligned");
    if (reinterpret_cast<uintptr_t>(d_match_off) & 1)
        return fail(c, DEDUP_EINVAL, "d_match_off must be 2-byte aligned");
    if (nbytes >= (1ull << 31)) return fail(c, DEDUP_EINVAL, "nbytes >= 2^31");
    if (window < 1 || window > 16384) return fail(c, DEDUP_EINVAL, "window not in [1, 16384]");
    if (max_coded < 1 || max_coded > 255)
        return fail(c, DEDUP_EINVAL, "max_coded not in [1, 255]");
    if (nbytes > 0 && (d_start == nullptr || d_n_blocks == nullptr || cap == 0))
        return fail(c, DEDUP_EINVAL, "no block starts");
    CU(cudaSetDevice(c->cfg.device));
    if (const char* k = findmatch_unlaunchable(window, max_coded))
        return fail(c, DEDUP_EINVAL, std::string(k) + " does not fit this window");
    launch_findmatch(d_bytes, (uint32_t)nbytes, d_start, d_n_blocks, cap, d_skip, window,
                     max_coded, d_match_len, d_match_off, c->num_sms,
                     static_cast<cudaStream_t>(stream));
    c->launches += nbytes ? 1 : 0;
    CU(cudaGetLastError());
    return DEDUP_OK;
}

dedup_status dedup_op_table_insert_lookup(dedup_ctx* c, void* stream, const uint8_t* d_digest,
                                          const uint64_t* d_id, const uint32_t* d_n, uint64_t cap,
                                          uint64_t* d_first_id, uint8_t* d_is_dup) {
    if (c == nullptr) return DEDUP_EINVAL;
    NO_MG(c);
    if (!usable(c)) return c->sticky;
    if (cap > c->chunk_cap) return fail(c, DEDUP_EINVAL, "cap larger than the ctx workspace");
    CU(cudaSetDevice(c->cfg.device));
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    BatchDesc h{};
    h.table = table_view(c);
    const BatchDesc* d = nullptr;
    TRY(op_desc(c, s, h, &d));
    launch_table_insert(&d->table, d_digest, d_id, nullptr, d_n, 0, cap, c->op_ws.slot_idx,
                        c->num_sms, s);
    launch_table_lookup(&d->table, d_id, nullptr, d_n, 0, cap, c->op_ws.slot_idx, d_first_id,
                        d_is_dup, nullptr, nullptr, nullptr, c->num_sms, s);
    c->launches += cap ? 2 : 1;
    CU(cudaGetLastError());
    return DEDUP_OK;
}

dedup_status dedup_op_table_reset(dedup_ctx* c, void* stream) {
    if (c == nullptr) return DEDUP_EINVAL;
    NO_MG(c);
    if (!usable(c)) return c->sticky;
    CU(cudaSetDevice(c->cfg.device));
    TableBuf& t = c->tables[c->cur_table];
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    CU(cudaMemsetAsync(t.slots, 0, sizeof(TableSlot) * t.capacity, s));
    CU(cudaMemsetAsync(t.status, 0, 16, s));
    return DEDUP_OK;
}

dedup_status dedup_op_table_status(dedup_ctx* c, void* stream, uint64_t* used, uint64_t* slots,
                                   int32_t* overflow) {
    if (c == nullptr) return DEDUP_EINVAL;
    NO_MG(c);
    CU(cudaSetDevice(c->cfg.device));
    TableBuf& t = c->tables[c->cur_table];
    uint32_t st[4];
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    CU(cudaMemcpyAsync(st, t.status, 16, cudaMemcpyDeviceToHost, s));
    CU(cudaStreamSynchronize(s));
    if (used) *used = st[1];
    if (slots) *slots = t.capacity;
    if (overflow) *overflow = (int32_t)st[0];
    return DEDUP_OK;
}

dedup_status dedup_op_local_combine(dedup_ctx* c, void* stream, const uint8_t* d_digest,
                                    const uint32_t* d_n, uint64_t cap, uint32_t* d_rep) {
    if (c == nullptr) return DEDUP_EINVAL;
    NO_MG(c);
    if (!usable(c)) return c->sticky;
    if (cap > c->chunk_cap) return fail(c, DEDUP_EINVAL, "cap larger than the ctx workspace");
    if (d_rep == nullptr || (cap > 0 && (d_digest == nullptr || d_n == nullptr)))
        return fail(c, DEDUP_EINVAL, "null argument");
    CU(cudaSetDevice(c->cfg.device));
    if (c->local.slots == nullptr) {  // first call: an empty local table
        TableBuf& t = c->local;
        t.capacity = next_pow2(2 * c->chunk_cap);
        TRY(dalloc(c, &t.slots, t.capacity));
        TRY(dalloc(c, &t.status, 4));
        TRY(dalloc(c, &c->d_local_view, 1));
        CU(cudaMemset(t.slots, 0, sizeof(TableSlot) * t.capacity));
        CU(cudaMemset(t.status, 0, 16));
        const TableView v{t.slots, t.capacity - 1, t.status};
        CU(cudaMemcpy(c->d_local_view, &v, sizeof(v), cudaMemcpyHostToDevice));
    }
    const TableView v{c->local.slots, c->local.capacity - 1, c->local.status};
    launch_local_combine(v, d_digest, d_n, cap, c->op_ws.slot_idx, d_rep, c->num_sms,
                         static_cast<cudaStream_t>(stream), c->d_local_view);
    c->launches += cap ? 3 : 0;
    CU(cudaGetLastError());
    return DEDUP_OK;
}

dedup_status dedup_op_route(dedup_ctx* c, void* stream, const uint8_t* d_digest,
                            const uint64_t* d_id, const uint32_t* d_n, uint64_t cap,
                            const uint32_t* d_rep, uint32_t num_owners, dedup_record* d_send,
                            uint32_t* d_send_off, uint32_t* d_send_pos) {
    if (c == nullptr) return DEDUP_EINVAL;
    NO_MG(c);
    if (!usable(c)) return c->sticky;
    if (num_owners < 1 || num_owners > 64) return fail(c, DEDUP_EINVAL, "num_owners in 1..64");
    CU(cudaSetDevice(c->cfg.device));
    launch_route(d_digest, d_id, d_n, cap, d_rep, num_owners, d_send, d_send_off, d_send_pos,
                 c->op_ws.counters + 64, c->num_sms, static_cast<cudaStream_t>(stream));
    c->launches += cap ? 3 : 1;
    CU(cudaGetLastError());
    return DEDUP_OK;
}

dedup_status dedup_op_owner(dedup_ctx* c, void* stream, const dedup_record* d_recv,
                            uint64_t n_recv, uint64_t* d_reply) {
    if (c == nullptr) return DEDUP_EINVAL;
    NO_MG(c);
    if (!usable(c)) return c->sticky;
    if (n_recv > c->chunk_cap) return fail(c, DEDUP_EINVAL, "n_recv larger than the workspace");
    CU(cudaSetDevice(c->cfg.device));
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    BatchDesc h{};
    h.table = table_view(c);
    const BatchDesc* d = nullptr;
    TRY(op_desc(c, s, h, &d));
    if (n_recv) {
        launch_table_insert(&d->table, nullptr, nullptr, d_recv, nullptr, n_recv, n_recv,
                            c->op_ws.slot_idx, c->num_sms, s);
        launch_table_lookup(&d->table, nullptr, d_recv, nullptr, n_recv, n_recv,
                            c->op_ws.slot_idx, d_reply, nullptr, nullptr, nullptr, nullptr,
                            c->num_sms, s);
        c->launches += 2;
    }
    CU(cudaGetLastError());
    return DEDUP_OK;
}

dedup_status dedup_op_scatter(dedup_ctx* c, void* stream, const uint64_t* d_reply_back,
                              const uint32_t* d_send_pos, const uint32_t* d_rep,
                              const uint64_t* d_id, const uint32_t* d_n, uint64_t cap,
                              uint64_t* d_first_id, uint8_t* d_is_dup) {
    if (c == nullptr) return DEDUP_EINVAL;
    NO_MG(c);
    if (!usable(c)) return c->sticky;
    CU(cudaSetDevice(c->cfg.device));
    launch_scatter(d_reply_back, d_send_pos, d_rep, d_id, d_n, cap, d_first_id, d_is_dup,
                   c->num_sms, static_cast<cudaStream_t>(stream));
    c->launches += cap ? 1 : 0;
    CU(cudaGetLastError());
    return DEDUP_OK;
}

}  // extern "C"
