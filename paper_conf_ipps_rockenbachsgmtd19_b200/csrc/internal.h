// Internal launcher declarations shared by the CUDA translation units of
// libdedup_b200.so.  Not part of the C ABI (see include/dedup.h).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace dd {

// ---- chunking (rabin.cu) --------------------------------------------------
// Positions per cut-selection tile (e-space), words of the candidate bitmap.
constexpr uint32_t kSelTile = 8192;
constexpr uint32_t kSelTileWords = kSelTile / 32;
// u64 words of look-back descriptor per tile: [0] inclusive, [1..32] aggregate.
constexpr uint32_t kDescWords = 33;

struct ScanCfg {
    int num_sms;
};

// Bitmap bit i (i < nbytes) set iff (fp(bytes[i-31..i]) & mask) == value.
void launch_rabin_scan(const uint8_t* bytes, uint64_t nbytes, const uint32_t* d_tab,
                       uint32_t mask, uint32_t value, uint32_t* bitmap, int num_sms,
                       cudaStream_t s);

// Greedy cut selection with decoupled look-back over kSelTile-position tiles.
void launch_select(const uint32_t* bitmap, uint64_t nbytes, const uint64_t* item_off,
                   uint32_t n_items, uint64_t* desc, uint32_t* tile_counter, uint32_t epoch,
                   uint32_t* cut_pos, uint64_t cap, uint32_t* n_chunks, int num_sms,
                   cudaStream_t s);

void launch_chunk_meta(const uint64_t* item_off, uint32_t n_items, const uint32_t* cut_pos,
                       const uint32_t* n_chunks, uint64_t cap, uint64_t first_seq,
                       uint32_t* chunk_start, uint64_t* chunk_id, uint32_t* item_first_chunk,
                       int num_sms, cudaStream_t s);

// ---- SHA-1 (sha1.cu) -------------------------------------------------------
void launch_sha1(const uint8_t* bytes, uint64_t nbytes, const uint32_t* cut_pos,
                 const uint32_t* n_chunks, uint64_t cap, uint32_t* work_counter,
                 uint8_t* digest, int num_sms, cudaStream_t s);

// ---- digest table and routing (table.cu) ----------------------------------
struct TableSlot {
    uint32_t key[5];   // raw digest bytes (as little-endian words)
    uint32_t state;    // 0 empty, 1 being written, 2 published
    uint64_t inv_min;  // ~(minimum id); 0 = none yet (table is zero-initialised)
};
static_assert(sizeof(TableSlot) == 32, "slot is one 32-byte sector");

struct TableView {
    TableSlot* slots;
    uint64_t mask;       // capacity - 1 (power of two)
    uint32_t* status;    // [0] overflow flag, [1] used slots (low 32), [2] used hi
};

// Insert records then look them up.  Records come either as (digest bytes,
// id) arrays or as packed 32-byte records (rec != nullptr).
void launch_table_insert(TableView t, const uint8_t* digest, const uint64_t* id,
                         const void* rec, const uint32_t* d_n, uint64_t n_host, uint64_t cap,
                         uint32_t* slot_idx, int num_sms, cudaStream_t s);
void launch_table_lookup(TableView t, const uint64_t* id, const void* rec,
                         const uint32_t* d_n, uint64_t n_host, uint64_t cap,
                         const uint32_t* slot_idx, uint64_t* first_id, uint8_t* is_dup,
                         int num_sms, cudaStream_t s);

void launch_route(const uint8_t* digest, const uint64_t* id, const uint32_t* d_n, uint64_t cap,
                  uint32_t num_owners, void* send, uint32_t* send_off, uint32_t* send_pos,
                  uint32_t* scratch_counts, int num_sms, cudaStream_t s);
void launch_scatter(const uint64_t* reply, const uint32_t* send_pos, const uint64_t* id,
                    const uint32_t* d_n, uint64_t cap, uint64_t* first_id, uint8_t* is_dup,
                    int num_sms, cudaStream_t s);

// Results of one batch written straight into mapped pinned host memory.
struct HostResultLayout {
    uint32_t* header;          // [0] n_chunks, [1] table overflow flag
    uint32_t* chunk_start;
    uint64_t* first_id;
    uint8_t* digest;
    uint8_t* is_dup;
    uint32_t* item_first_chunk;
};
void launch_pack(const uint32_t* n_chunks, uint64_t cap, uint32_t n_items,
                 const uint32_t* chunk_start, const uint64_t* first_id, const uint8_t* digest,
                 const uint8_t* is_dup, const uint32_t* item_first_chunk,
                 const uint32_t* table_status, HostResultLayout h, int num_sms,
                 cudaStream_t s);

}  // namespace dd
