// Internal launcher declarations shared by the CUDA translation units of
// libdedup_b200.so.  Not part of the C ABI (see include/dedup.h).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

// DEDUP_CHECK builds (tools/gpu_checked.sh): device-side bounds checks in
// the kernels, a trap with the failed condition printed; nothing otherwise.
#ifdef DEDUP_CHECK
#include <cstdio>
#define DD_CHECK(cond)                                                                \
    do {                                                                              \
        if (!(cond)) {                                                                \
            printf("DD_CHECK failed: %s (%s:%d)\n", #cond, __FILE__, __LINE__);       \
            __trap();                                                                 \
        }                                                                             \
    } while (0)
#else
#define DD_CHECK(cond) \
    do {               \
    } while (0)
#endif

namespace dd {

// ---- digest table --------------------------------------------------------
struct TableSlot {
    uint32_t key[5];   // raw digest bytes (as little-endian words)
    uint32_t state;    // 0 empty, 1 being written, 2 published
    uint64_t inv_min;  // ~(minimum id); 0 = none yet (table is zero-initialised)
};
static_assert(sizeof(TableSlot) == 32, "slot is one 32-byte sector");

struct TableView {
    TableSlot* slots;
    uint64_t mask;       // capacity - 1 (power of two)
    uint32_t* status;    // [0] overflow flag, [1] used slots
};

// Per-batch parameters, read by the kernels from device memory so that the
// launch sequence of a batch slot is a fixed CUDA graph.
// Carry-over mode (row NEXT-2, dedup_config.carry_over): the state of the
// chunker after a piece of the stream, passed to the next piece's batch.
struct CarryState {
    uint32_t H[5];        // SHA-1 state of the open chunk (after its full blocks)
    uint32_t exit_state;  // positions still blocked at the piece end (0..32)
    uint64_t open_len;    // bytes of the open chunk so far
    uint32_t left_n;      // bytes of it not yet compressed (< 64), in left[]
    uint32_t pad_;
    uint8_t left[64];
    uint8_t hist[32];     // the last 32 bytes of the stream so far
};

// BatchDesc.carry flags
constexpr uint32_t kCarryMode = 1;   // the batch is one piece of a carry-over stream
constexpr uint32_t kCarryCont = 2;   // ... continuing the previous piece (not the stream start)
constexpr uint32_t kCarryClose = 4;  // ... the (empty) closing batch of the stream

struct alignas(64) BatchDesc {
    const uint8_t* bytes;      // batch bytes (16-byte aligned)
    uint64_t nbytes;
    uint64_t first_seq;        // seq of the batch's first item
    const uint64_t* item_off;  // [n_items + 1] device
    uint32_t n_items;
    uint32_t fresh;            // 1: clear the table before inserting
    TableView table;
    uint32_t carry;            // kCarry* flags (0: the item model, reading O8)
    uint32_t pad_c;
    const CarryState* carry_in;  // the previous piece's state (kCarryCont)
    CarryState* carry_out;       // this piece's state
};

// ---- product-side Rabin tables (independent of the oracle) ---------------
// P(t) = t^32 + poly over GF(2); tab[b] = R[b] = b t^32 mod P (reduction of
// the byte shifted out of the top), tab[256 + b] = W256[b] = b t^256 mod P
// (the byte leaving the 32-byte window, applied after the shift).
inline uint32_t gf2_mul_tk(uint32_t x, unsigned k, uint32_t poly) {
    while (k--) x = (x & 0x80000000u) ? ((x << 1) ^ poly) : (x << 1);
    return x;
}
inline void rabin_tables(uint32_t poly, uint32_t tab[512]) {
    for (uint32_t b = 0; b < 256; ++b) {
        tab[b] = gf2_mul_tk(b, 32, poly);
        tab[256 + b] = gf2_mul_tk(b, 256, poly);
    }
}

// ---- chunking (rabin.cu) --------------------------------------------------
// Positions per cut-selection tile (e-space), words of the candidate bitmap.
constexpr uint32_t kSelTile = 8192;
constexpr uint32_t kSelTileWords = kSelTile / 32;

// Rows A2 + A3: Rabin scan fused with the per-tile 32-entry transfer
// functions of the greedy cut selection (agg, 32 u32 per kSelTile tile) and
// their per-group composition (gagg, 32 u32 per group of 32 tiles); a one-CTA
// prefix over the groups (gentry, 2 u32 per group: entry state, cut offset);
// a replay writing cut_pos.  bitmap: e-space candidate words (nbytes/32 + 1);
// evbuf: event_words(max_tiles) words.
// after_scan (optional) is recorded between the scan and the selection.
uint64_t select_groups(uint64_t max_tiles);
// Per-tile event slots (evbuf) written by the scan for the cut emission.
uint64_t event_words(uint64_t max_tiles);

// Launch-configuration check (dedup_init fails with DEDUP_ECUDA instead of
// losing a launch inside a graph): true iff one CTA of fn fits on an SM.
inline bool fits(const void* fn, int threads, size_t dyn_smem) {
    int n = 0;
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, fn, threads, dyn_smem) ==
               cudaSuccess &&
           n >= 1;
}
// Name of a kernel of rabin.cu / sha1.cu that cannot launch with its
// configuration, or nullptr.
const char* chunk_unlaunchable();
const char* sha1_unlaunchable();
// Preferred shared-memory carveout (percent) of the pipeline's kernels;
// set_pipeline_carveout applies the engine's setting (table.cu) to all of
// them on the current device.
void set_pipeline_carveout();
void sha1_set_carveout(int pct);
void chunk_set_carveout(int pct);
void table_set_carveout(int pct);
void launch_chunk_select(const BatchDesc* d, const uint32_t* d_tab, uint32_t mask,
                         uint32_t value, uint32_t* bitmap, uint32_t* agg, uint32_t* gagg,
                         uint32_t* gentry, uint32_t* evbuf, uint64_t max_tiles,
                         uint32_t* cut_pos, uint64_t cap, uint32_t* n_chunks, int num_sms,
                         cudaStream_t s, cudaEvent_t after_scan, uint32_t max_chunk = 0,
                         uint32_t* mc_ws = nullptr, uint32_t max_items = 0,
                         uint32_t min_chunk = 32, cudaEvent_t before_select = nullptr);
// max_chunk workspace words: fsm count (1) + fsm cuts (cap) + item counts and
// flags (2 x (max_items + 1)).
inline uint64_t maxchunk_ws_words(uint64_t cap, uint64_t max_items) {
    return 1 + cap + 2 * (max_items + 1);
}
// NEXT-2 max_chunk selection (maxchunk.cu): the state machine's cuts
// (fsm_cut, *fsm_n) are kept for items without a chunk > max_chunk; the
// other items are walked over the scan's candidate bitmap.
void launch_select_walk(const BatchDesc* d, const uint32_t* bitmap, uint32_t max_chunk,
                        uint32_t min_chunk, uint32_t* item_cnt, uint32_t* item_flag,
                        uint32_t max_items, const uint32_t* fsm_cut, const uint32_t* fsm_n,
                        uint32_t* cut_pos, uint64_t cap, uint32_t* n_chunks, int num_sms,
                        cudaStream_t s);

void launch_chunk_meta(const BatchDesc* d, const uint32_t* cut_pos, const uint32_t* n_chunks,
                       uint64_t cap, uint32_t* chunk_start, uint64_t* chunk_id,
                       uint32_t* item_first_chunk, uint32_t max_items, int num_sms,
                       cudaStream_t s);

// ---- SHA-1 (sha1.cu) -------------------------------------------------------
// ws: sha1_ws_words(cap) words of scratch (the sort of the chunks by length
// and the warps' task counter).  max_bytes: largest nbytes this launch may see
// (grid sizing); lane_bytes: batch bytes per SHA-1 lane (0 = 32 KiB).
uint64_t sha1_ws_words(uint64_t cap);
void launch_sha1(const BatchDesc* d, uint64_t max_bytes, const uint32_t* cut_pos,
                 const uint32_t* n_chunks, uint64_t cap, uint32_t* ws, uint8_t* digest,
                 int num_sms, cudaStream_t s, uint32_t lane_bytes = 0);

// ---- digest table and routing (table.cu) ----------------------------------
// Insert records then look them up.  Records come either as (digest bytes,
// id) arrays or as packed 32-byte records (rec != nullptr).
// The table is read from *tv (device memory) at run time.
void launch_table_prepare(const BatchDesc* d, uint64_t max_slots, int num_sms, cudaStream_t s);
void launch_table_insert(const TableView* tv, const uint8_t* digest, const uint64_t* id,
                         const void* rec, const uint32_t* d_n, uint64_t n_host, uint64_t cap,
                         uint32_t* slot_idx, int num_sms, cudaStream_t s);
// Transport 3 (p2p, one process): the routed records of a rank (send,
// grouped by owner, send_off[G] of them, <= cap) inserted directly into the
// owners' shards (views: device array of the G owners' TableViews, peer
// memory), and after every rank's inserts their first ids read back into
// reply_back (send order).  slot_idx: cap words of scratch kept between the
// two calls.
void launch_p2p_insert(const TableView* views, uint32_t G, const void* send,
                       const uint32_t* send_off, uint64_t cap, uint32_t* slot_idx, int num_sms,
                       cudaStream_t s);
void launch_p2p_lookup(const TableView* views, uint32_t G, const void* send,
                       const uint32_t* send_off, uint64_t cap, const uint32_t* slot_idx,
                       uint64_t* reply_back, int num_sms, cudaStream_t s);
void launch_table_lookup(const TableView* tv, const uint64_t* id, const void* rec,
                         const uint32_t* d_n, uint64_t n_host, uint64_t cap,
                         const uint32_t* slot_idx, uint64_t* first_id, uint8_t* is_dup,
                         uint32_t* status_out, const uint32_t* cut_pos,
                         const BatchDesc* desc, int num_sms, cudaStream_t s);

// rep (optional): local-combine representatives; only records with
// rep[r] == r are routed, and scatter gives chunk r the reply of rep[r].
void launch_route(const uint8_t* digest, const uint64_t* id, const uint32_t* d_n, uint64_t cap,
                  const uint32_t* rep, uint32_t num_owners, void* send, uint32_t* send_off,
                  uint32_t* send_pos, uint32_t* scratch_counts, int num_sms, cudaStream_t s);
// overflow (optional): set to 1 if a reply is ~0 (the owner's shard overflowed)
void launch_scatter(const uint64_t* reply, const uint32_t* send_pos, const uint32_t* rep,
                    const uint64_t* id, const uint32_t* d_n, uint64_t cap, uint64_t* first_id,
                    uint8_t* is_dup, int num_sms, cudaStream_t s, uint32_t* overflow = nullptr);
// Copy exchange of the multi-GPU engine (mg.cpp): rank `me` pulls rows
// [src_off[s][me], src_off[s][me+1]) of src[s] for every rank s (pointer
// arrays in device memory) to dst_off[s] or, without dst_off, to the prefix
// of the counts, which is written to out_off[0..G].
void launch_gather_rows(const uint8_t* const* src, const uint32_t* const* src_off, uint32_t me,
                        uint32_t G, uint32_t row_bytes, uint8_t* dst, const uint32_t* dst_off,
                        uint32_t* out_off, uint64_t max_rows_per_src, int num_sms,
                        cudaStream_t s);
// cnt[2s], cnt[2s+1] = src_off[s][me], src_off[s][me+1]
void launch_gather_counts(const uint32_t* const* src_off, uint32_t me, uint32_t G, uint32_t* cnt,
                          cudaStream_t s);
// Row A5 local combine: rep[r] = smallest record index with digest r's digest,
// through the (empty) local table `local` (*d_local: the same view in device
// memory); the used slots are cleared again afterwards.
void launch_local_combine(TableView local, const uint8_t* digest, const uint32_t* d_n,
                          uint64_t cap, uint32_t* slot_idx, uint32_t* rep, int num_sms,
                          cudaStream_t s, const TableView* d_local);

// ---- carry-over mode (carry.cu, row NEXT-2) ---------------------------------
void launch_carry_hist(const BatchDesc* d, cudaStream_t s);
// m_out = reported chunks; extra[0..1] = bytes of chunk 0 in earlier pieces,
// extra[2] = end of the last reported chunk (piece-relative)
void launch_carry_meta(const BatchDesc* d, const uint32_t* n_cuts, const uint32_t* cut_pos,
                       uint64_t cap, uint32_t* m_out, uint32_t* chunk_start, uint64_t* chunk_id,
                       uint32_t* item_first, uint32_t* extra, cudaStream_t s);
void launch_carry_cont(const BatchDesc* d, const uint32_t* n_cuts, const uint32_t* cut_pos,
                       uint64_t cap, uint8_t* digest, uint32_t* extra, cudaStream_t s);

// ---- LZSS FindMatch (lzss.cu, row NEXT-1) ----------------------------------
uint32_t findmatch_smem(uint32_t window, uint32_t max_coded);
const char* findmatch_unlaunchable(uint32_t window, uint32_t max_coded);
void launch_findmatch(const uint8_t* bytes, uint32_t nbytes, const uint32_t* cut_pos,
                      const uint32_t* n_chunks, uint64_t cap, const uint8_t* skip,
                      uint32_t window, uint32_t max_coded, uint8_t* out_len, uint16_t* out_off,
                      int num_sms, cudaStream_t s);

// ---- Mandelbrot Streaming (mandel.cu, row NEXT-4) -----------------------------
const char* mandel_unlaunchable();
void launch_mandel(int32_t dim, int32_t niter, double init_a, double init_b, double step,
                   int32_t row0, int32_t nrows, uint8_t* img, uint32_t* counter,
                   uint64_t* iters, int num_sms, cudaStream_t s);

// Results of one batch written straight into mapped pinned host memory.
struct HostResultLayout {
    uint32_t* header;          // [0] n_chunks, [1] table overflow flag, [2] used slots
    uint32_t* chunk_start;
    uint64_t* first_id;
    uint8_t* digest;
    uint8_t* is_dup;
    uint32_t* item_first_chunk;
};
// extra (optional, carry-over mode): 3 words copied to header[6..8]
void launch_pack(const BatchDesc* d, const uint32_t* n_chunks, uint64_t cap, uint32_t max_items,
                 const uint32_t* chunk_start, const uint64_t* first_id, const uint8_t* digest,
                 const uint8_t* is_dup, const uint32_t* item_first_chunk,
                 const uint32_t* table_status, HostResultLayout h, int num_sms,
                 cudaStream_t s, const uint32_t* extra = nullptr);

}  // namespace dd
