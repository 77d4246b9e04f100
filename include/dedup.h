/*
 * dedup.h -- C ABI of the B200-native GPU Dedup hot path.
 *
 * The hot path is the data-parallel core of the GPU Dedup of Rockenbach et
 * al., "Stream Processing on Multi-Cores with GPUs: Parallel Programming
 * Models' Challenges" (IPDPSW 2019), Section IV-B.  "P:NNN" = line NNN of the
 * paper text:
 *   - P:197  fixed-size batches; Rabin fingerprint fragmentation; "saved all
 *            the indexes where the algorithm would fragment the data".
 *   - P:199  Fig. 2: startPos = chunk start indexes of a batch.
 *   - P:213  stage 1: batches of 1 MB, Rabin blocks.
 *   - P:214  stage 2: SHA-1 of every block on the GPU, results in an array.
 *   - P:215  stage 3: check whether blocks are duplicated.
 *   - P:217  stage 5: reorder batches (results in sequence order).
 * A stream item is one of the paper's batches (an "item" here); a GPU batch
 * groups whole items and never changes results (reading O8).
 *
 * Method parameters (readings O1-O7): window 32 bytes,
 * P(t) = t^32 + poly (0x45c2b6a1), cut iff (fp & anchor_mask) == anchor_value
 * (0xFFF / 0), minimum chunk = window (restart semantics), no maximum chunk.
 *
 * Two layers:
 *   1. Streaming API (dedup_init / dedup_submit_batch / dedup_submit_device /
 *      dedup_drain / dedup_stats / dedup_end_stream / dedup_destroy): items
 *      in, per-item results out in sequence order.  One ctx per GPU.
 *   2. Stream-ordered device operations (dedup_op_*): the individual hot-path
 *      steps on caller-owned DEVICE buffers, enqueued on a caller-provided
 *      cudaStream_t (passed as void*).  Used by the multi-GPU orchestrator
 *      (digest all-to-all between the route / owner / scatter steps) and by
 *      the per-kernel parity tests.
 *
 * Conventions for every call:
 *   - Return value: dedup_status, 0 = DEDUP_OK, < 0 = error.  DEDUP_ECUDA is
 *     sticky: afterwards the ctx accepts only dedup_stats, dedup_last_error
 *     and dedup_destroy.
 *   - A ctx is NOT thread-safe: calls on one ctx must be serialised by the
 *     caller (the paper's multi-thread GPU pitfall).
 *   - "device pointer" arguments must be allocations on the ctx's device;
 *     "host pointer" arguments are ordinary process memory.
 *   - No function here allocates memory that the caller must free, except
 *     dedup_host_alloc (freed by dedup_host_free).
 */
#ifndef DEDUP_B200_H
#define DEDUP_B200_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef int32_t dedup_status;
#define DEDUP_OK 0
#define DEDUP_EINVAL (-1)       /* bad config or arguments; nothing enqueued */
#define DEDUP_EAGAIN (-2)       /* in-flight window full: drain first */
#define DEDUP_ENOMEM (-3)       /* device or pinned allocation failed */
#define DEDUP_ETABLEFULL (-4)   /* digest table overflow (sticky) */
#define DEDUP_EUNSUPPORTED (-5) /* config valid for the method, not for GPU v1 */
#define DEDUP_ECUDA (-6)        /* CUDA error (sticky) */
#define DEDUP_ETIMEDOUT (-7)    /* dedup_drain: nothing completed within wait_ms */
#define DEDUP_ENCCL (-8)        /* NCCL error or a failed peer of the exchange (sticky) */

#define DEDUP_ABI_VERSION 2

typedef struct dedup_ctx dedup_ctx; /* opaque; owns its device buffers and tables */

typedef struct {
    uint32_t struct_size;    /* = sizeof(dedup_config) */
    uint32_t window;         /* 32 (GPU v1 requires 32) */
    uint32_t poly;           /* P(t) = t^32 + poly over GF(2) */
    uint32_t anchor_mask;    /* cut iff (fp & anchor_mask) == anchor_value */
    uint32_t anchor_value;
    uint32_t min_chunk;      /* >= window; != 32 selects cuts by a walk per item (NEXT-2) */
    uint32_t max_chunk;      /* 0 = none; else >= 64: forced cut at c + max_chunk (NEXT-2) */
    int32_t device;          /* CUDA device ordinal of this ctx */
    uint32_t slots;          /* in-flight batches ("memory spaces"), 1..64 */
    uint32_t batch_items;    /* max items per GPU batch */
    uint64_t batch_bytes;    /* max bytes per GPU batch (<= 1 GiB) */
    uint64_t table_capacity; /* expected distinct digests per stream (this owner's share) */
    uint32_t owner_rank;     /* digest-prefix owner index of this ctx's table shard */
    uint32_t num_owners;     /* number of table shards (GPUs); 1 = single GPU */
    uint32_t host_fed;       /* 1: allocate device input slots for dedup_submit_batch */
    uint32_t sha_lane_bytes; /* SHA-1 grid: one lane per this many batch bytes; 0 = 16384
                                (tuned for many batches in flight; a ctx that runs one
                                batch at a time wants fewer bytes per lane, e.g. 8192) */
    /* Multi-GPU (the paper's GPUs take batches round-robin,
     * P:185, one host thread per device).  num_devices >= 2 (or
     * transport != 0) selects the multi-GPU engine: G = num_devices logical
     * ranks, rank r on device_ids[r]; batches go to the ranks round-robin
     * (batch b -> rank b % G, wave b / G), rank r owns the digest-table shard
     * of the digests whose BE32 prefix p has floor(p G / 2^32) = r, and
     * dedup_drain returns every rank's items merged in sequence order
     * (P:217).  `slots` is then the waves in flight per rank and
     * table_capacity the expected distinct digests of the whole stream.
     * owner_rank / num_owners must be 0 / 1 (they describe the op layer). */
    uint32_t num_devices;       /* 0 or 1: single-GPU engine on `device`; 2..64: ranks */
    uint32_t transport;         /* exchange of rows A6/A8: 0 auto (NCCL if the devices are
                                   distinct, else copy), 1 NCCL (ncclCommInitAll; distinct
                                   devices), 2 in-process copy (peer loads over NVLink, or
                                   the loopback when device ids repeat), 3 in-process p2p
                                   (the exchange fused into the table kernels: records
                                   inserted into and first ids read from the owners' shards
                                   with system-scope atomics / loads on peer memory) */
    const int32_t* device_ids;  /* [num_devices] CUDA ordinals, may repeat; NULL = 0..G-1 */
    /* Carry-over mode (row NEXT-2; north_star: "the chunking is identical when
     * the input is split at arbitrary batch cuts"): 1 = the bytes of a dedup
     * stream form ONE chunking domain and every submitted item is a PIECE of
     * it, cut anywhere (pieces of 0 bytes allowed); one piece per GPU batch.
     * A piece's results are the chunks that END in it: chunk 0 may have begun
     * in earlier pieces (dedup_item_result.carried = its bytes there), the
     * chunk open at the piece end is reported by a later piece, and
     * dedup_end_stream submits a closing item (0 bytes, seq = the next seq)
     * that reports the stream's last chunk.  Ids are (piece seq << 32) |
     * index: stream order.  Requires the single-GPU engine, min_chunk 32,
     * max_chunk 0 and slots >= 2 (EUNSUPPORTED otherwise); at most slots - 1
     * pieces are in flight. */
    uint32_t carry_over;
    uint32_t reserved[1];
} dedup_config;

/* Fills *cfg with the defaults above (struct_size set). */
void dedup_config_default(dedup_config* cfg);

/* Creates a ctx (the GPU side of the paper's Dedup pipeline, stages 1-3 of
 * P:211-215 plus the reorder of P:217) on cfg->device -- or, with
 * num_devices >= 2, on G GPUs (memory spaces assigned to GPUs
 * round-robin; one host thread per device): copies the config,
 * builds the Rabin tables,
 * allocates `slots` batch slots (device + pinned host result buffers) and two
 * digest tables of >= 2 * table_capacity slots (power of two).
 * Errors: EINVAL (bad config), EUNSUPPORTED (window other than 32, or
 * 0 < max_chunk < 64), ENOMEM, ECUDA.  *out is NULL on error. */
dedup_status dedup_init(const dedup_config* cfg, dedup_ctx** out);

/* Releases everything; waits for in-flight work.  Accepts NULL. */
void dedup_destroy(dedup_ctx* c);

/* Human-readable description of the last error on c (never NULL). */
const char* dedup_last_error(const dedup_ctx* c);

/* ------------------------------------------------------------------------ */
/* 1. Streaming API                                                         */
/* ------------------------------------------------------------------------ */

/* Submits n_items host items (item k = item_len[k] bytes at item_ptr[k]): the
 * paper's stream of fixed-size batches read by the first pipeline stage
 * ("read the input file and generate batches of 1MB"), each item a
 * chunking domain (reading O8).  Items receive consecutive sequence numbers
 * *first_seq_out + k (the order P:217's reorder stage restores).  Items are
 * packed in order into GPU batches of <= batch_bytes / batch_items; every
 * batch needs a free slot ("memory space"), otherwise nothing is
 * submitted and DEDUP_EAGAIN is returned.  An item longer than batch_bytes or
 * 2^32-1 is EINVAL.
 * Ownership: buffers from dedup_host_alloc (or otherwise page-locked) are
 * DMA'd directly and BORROWED until the item is returned by dedup_drain;
 * other (pageable) memory is first copied by the calling thread into the
 * slot's internal page-locked bounce buffer (allocated on first use, one
 * batch_bytes buffer per slot), so it may be reused as soon as the call
 * returns.  Requires cfg.host_fed = 1. */
dedup_status dedup_submit_batch(dedup_ctx* c, uint32_t n_items, const uint8_t* const* item_ptr,
                                const uint64_t* item_len, uint64_t* first_seq_out);

/* Submits ONE GPU batch whose bytes are already resident on the device:
 * d_bytes (device pointer, 16-byte aligned, readable up to nbytes rounded up
 * to 16) holds n_items items back to back; item_off (HOST pointer,
 * n_items + 1 entries, item_off[0] = 0, non-decreasing, item_off[n_items] =
 * nbytes) gives their offsets.  `producer` (cudaStream_t as void*, NULL =
 * legacy default stream) is the stream that wrote d_bytes: the batch starts
 * after the work enqueued on it so far.  item_off is copied before return;
 * d_bytes is borrowed until the items are drained.  nbytes <= batch_bytes and
 * n_items <= batch_items, else EINVAL; EAGAIN if no slot is free. */
dedup_status dedup_submit_device(dedup_ctx* c, const uint8_t* d_bytes, uint64_t nbytes,
                                 const uint64_t* item_off, uint32_t n_items, void* producer,
                                 uint64_t* first_seq_out);

/* Makes `stream` (cudaStream_t as void*) wait for all work submitted so far
 * (no host synchronisation).  Used to bracket the engine with CUDA events. */
dedup_status dedup_join(dedup_ctx* c, void* stream);

/* Marks the end of the current dedup stream: items submitted afterwards are
 * checked against a fresh (empty) digest table.  Sequence numbers continue.
 * Carry-over mode: first submits the stream's closing item (see carry_over;
 * EAGAIN if no slot is free for it). */
dedup_status dedup_end_stream(dedup_ctx* c);

typedef struct {
    uint64_t seq;             /* sequence number (submission order) */
    uint64_t item_len;        /* bytes */
    uint32_t n_chunks;        /* 0 for an empty item */
    uint32_t carried;         /* carry-over mode: bytes of chunk 0 that lie in earlier pieces
                                 (chunk 0 then starts `carried` bytes before this item,
                                 chunk_start[0] = 0; saturated at 2^32 - 1); else 0 */
    const uint32_t* chunk_start; /* [n_chunks] item-relative starts, [0] = 0, increasing (startPos) */
    const uint8_t* digest;    /* [n_chunks * 20] SHA-1, FIPS byte order */
    const uint8_t* is_dup;    /* [n_chunks] 1 iff an earlier chunk of the stream has the same digest */
    const uint64_t* first_id; /* [n_chunks] (seq << 32) | chunk index of the first occurrence */
} dedup_item_result;

/* Returns up to max_items completed items, strictly in sequence order
 * (P:217).  wait_ms < 0 waits without limit for the next item, 0 polls,
 * > 0 waits up to wait_ms milliseconds.  *n_out = number returned (0 with
 * DEDUP_ETIMEDOUT when nothing completed in time; 0 with DEDUP_OK when
 * nothing is in flight).  Result arrays are ctx-owned and valid until the
 * next dedup_drain / dedup_destroy on c. */
dedup_status dedup_drain(dedup_ctx* c, uint32_t max_items, int32_t wait_ms,
                         dedup_item_result* out, uint32_t* n_out);

/* Number of submitted items not yet returned by dedup_drain. */
uint64_t dedup_pending(const dedup_ctx* c);

/* CUDA device of the rank that receives the next batch (multi-GPU ctx:
 * dedup_submit_device's d_bytes should live there; on another device it is
 * read over peer access).  The single-GPU engine returns cfg.device. */
int32_t dedup_next_device(const dedup_ctx* c);

typedef struct {
    uint64_t items, bytes, chunks, dup_chunks, dup_bytes, unique_chunks;
    uint64_t batches, table_used, table_slots, kernel_launches;
    uint32_t num_owners, owner_rank;
    /* summed CUDA-event stage times over drained batches (ms): H2D of the
     * input, Rabin scan kernel, cut selection + chunk metadata, SHA-1 kernel,
     * table insert + lookup, pack of results into pinned host memory */
    double ms_h2d, ms_scan, ms_select, ms_sha1, ms_table, ms_d2h;
    double ms_host_launch, ms_host_parse; /* host time in cudaGraphLaunch / result parsing */
    uint64_t sha1_blocks; /* 64-byte SHA-1 compressions over drained batches */
    /* the ms_* stage times cover only the sampled batches (every
     * DEDUP_TIME_EVERY-th drained batch, default 1; none if
     * DEDUP_STAGE_EVENTS=0): their count, bytes and SHA-1 blocks */
    uint64_t timed_batches, timed_bytes, timed_sha1_blocks;
    /* multi-GPU engine: waves completed, bytes of 32-byte records and 8-byte
     * replies that left their rank (rows A6 + A8), and the summed device time
     * of the exchange + owner phase (records .. scatter) of the sampled waves */
    uint64_t waves, a2a_bytes;
    double ms_a2a;
    uint32_t num_devices, reserved_;
} dedup_stats_t;

/* Counters over all drained batches of the ctx (all streams): items, bytes,
 * chunks and duplicates (the paper's stage-3 outcome; duplicate ratio
 * by chunk count and by bytes, reading O15), per-stage CUDA-event times and,
 * for the multi-GPU engine, the bytes of the digest exchange. */
dedup_status dedup_stats(const dedup_ctx* c, dedup_stats_t* out);

/* Pinned, portable host memory usable as zero-copy DMA source for
 * dedup_submit_batch.  Returns NULL on failure. */
void* dedup_host_alloc(dedup_ctx* c, size_t bytes);
void dedup_host_free(dedup_ctx* c, void* p);

/* ------------------------------------------------------------------------ */
/* 2. Stream-ordered device operations (caller-owned device buffers)        */
/* ------------------------------------------------------------------------ */
/* All pointers below are DEVICE pointers unless marked (host).  `stream` is a
 * cudaStream_t of the ctx's device (NULL = legacy default stream).  The calls
 * only enqueue work; outputs are valid once the stream reaches that point.
 * Device-side counts (d_n_*) are read by the kernels, so no host
 * synchronisation is needed between steps.  Ops on one ctx use one internal
 * workspace and must not overlap in time on different streams. */

/* Rows A2+A3: Rabin candidate scan over the whole batch
 * (d_bytes[0..nbytes), 16-byte aligned, readable to nbytes rounded up to 16)
 * with items at d_item_off[0..n_items] (u64, item_off[0] = 0,
 * item_off[n_items] = nbytes), then greedy cut selection with forced cuts at
 * every non-empty item start.  Writes the batch-relative chunk starts
 * d_cut_pos[0..n) (u32, increasing) and n to *d_n_chunks (u32).
 * cap = capacity of d_cut_pos; if n would exceed cap, *d_n_chunks = n but
 * only cap entries are written and the call returns DEDUP_OK (check n).
 * nbytes <= cfg.batch_bytes (workspace size), else EINVAL. */
dedup_status dedup_op_chunk(dedup_ctx* c, void* stream, const uint8_t* d_bytes, uint64_t nbytes,
                            const uint64_t* d_item_off, uint32_t n_items, uint32_t* d_cut_pos,
                            uint64_t cap, uint32_t* d_n_chunks);

/* Per-chunk metadata from the cuts: item-relative d_chunk_start (u32),
 * d_chunk_id = ((first_seq + item) << 32) | index within item (u64), and
 * d_item_first_chunk[item] (u32, 0xFFFFFFFF for empty items). cap as above. */
dedup_status dedup_op_chunk_meta(dedup_ctx* c, void* stream, const uint64_t* d_item_off,
                                 uint32_t n_items, const uint32_t* d_cut_pos,
                                 const uint32_t* d_n_chunks, uint64_t cap, uint64_t first_seq,
                                 uint32_t* d_chunk_start, uint64_t* d_chunk_id,
                                 uint32_t* d_item_first_chunk);

/* Row A4: SHA-1 (FIPS 180-4) of every chunk k = d_bytes[cut[k],
 * cut[k+1]) (last chunk ends at nbytes) for k < min(*d_n_chunks, cap);
 * writes d_digest[20k..20k+20).  Any increasing cut list starting at 0
 * describes a valid partition. */
dedup_status dedup_op_sha1(dedup_ctx* c, void* stream, const uint8_t* d_bytes, uint64_t nbytes,
                           const uint32_t* d_cut_pos, const uint32_t* d_n_chunks, uint64_t cap,
                           uint8_t* d_digest);

/* Row A7 on this ctx's table of the CURRENT stream: insert every
 * record (d_digest[20r..], d_id[r]) keeping the minimum id per digest, then
 * look each one up: d_first_id[r] = min id over all records inserted so far
 * with that digest; d_is_dup[r] = (d_first_id[r] != d_id[r]).  Records are
 * r < min(*d_n, cap).  Results equal the sequential stream-order answer
 * provided every record with a smaller id was inserted earlier or in this
 * call.  d_is_dup may be NULL.  Table overflow sets a sticky device flag
 * reported by dedup_op_table_status. */
dedup_status dedup_op_table_insert_lookup(dedup_ctx* c, void* stream, const uint8_t* d_digest,
                                          const uint64_t* d_id, const uint32_t* d_n, uint64_t cap,
                                          uint64_t* d_first_id, uint8_t* d_is_dup);

/* Clears the current stream's table (stream-ordered). */
dedup_status dedup_op_table_reset(dedup_ctx* c, void* stream);

/* Reads table occupancy and the overflow flag (synchronises `stream`). */
dedup_status dedup_op_table_status(dedup_ctx* c, void* stream, uint64_t* used, uint64_t* slots,
                                   int32_t* overflow);

/* 32-byte digest record exchanged between GPUs (rows A5/A6). */
typedef struct {
    uint8_t digest[20];
    uint32_t pad;
    uint64_t id;
} dedup_record;

/* Row A5, local combine ("per batch: collapse equal digests to
 * their min id"): for the *d_n (<= cap <= this ctx's chunk capacity) digests
 * of one batch (d_digest, 20 B each, chunk order), writes d_rep[r] = the
 * smallest index r' with digest r' == digest r (r itself for a first
 * occurrence).  Only representatives (d_rep[r] == r) need to travel to their
 * owner: the batch's chunks are in stream order, so the representative holds
 * the smallest id of its digest in the batch and the owner's minimum over
 * representatives is the global first occurrence (reading O12).  Uses a
 * ctx-owned local digest table (allocated on the first call, 2 x the ctx's
 * chunk capacity slots) that is left empty again. */
dedup_status dedup_op_local_combine(dedup_ctx* c, void* stream, const uint8_t* d_digest,
                                    const uint32_t* d_n, uint64_t cap, uint32_t* d_rep);

/* Row A5: owner(r) = floor(BE32(digest[0..3]) * num_owners / 2^32).
 * Writes records grouped by owner into d_send (capacity cap records):
 * owner o's records occupy d_send[d_send_off[o] .. d_send_off[o+1]) (u32
 * exclusive offsets, num_owners + 1 entries); d_send_pos[r] = slot of record r
 * in d_send.  d_rep (optional, from dedup_op_local_combine): only records with
 * d_rep[r] == r are routed (d_send_pos of the others is not written).
 * num_owners <= 64. */
dedup_status dedup_op_route(dedup_ctx* c, void* stream, const uint8_t* d_digest,
                            const uint64_t* d_id, const uint32_t* d_n, uint64_t cap,
                            const uint32_t* d_rep, uint32_t num_owners, dedup_record* d_send,
                            uint32_t* d_send_off, uint32_t* d_send_pos);

/* Row A7 on the owner: insert all n_recv (host count) received records into
 * this ctx's table shard, then write d_reply[i] = first id of record i. */
dedup_status dedup_op_owner(dedup_ctx* c, void* stream, const dedup_record* d_recv,
                            uint64_t n_recv, uint64_t* d_reply);

/* Row A8: d_first_id[r] = d_reply_back[d_send_pos[q]] with q = d_rep[r] (or
 * q = r when d_rep is NULL), d_is_dup[r] = (d_first_id[r] != d_id[r]). */
dedup_status dedup_op_scatter(dedup_ctx* c, void* stream, const uint64_t* d_reply_back,
                              const uint32_t* d_send_pos, const uint32_t* d_rep,
                              const uint64_t* d_id, const uint32_t* d_n, uint64_t cap,
                              uint64_t* d_first_id, uint8_t* d_is_dup);

/* Row NEXT-1: LZSS FindMatch over a resident batch -- stage 4
 * of the paper's GPU Dedup ("compress every not duplicated blocks on GPU ...
 * reuses data already on GPU"), one launch over all blocks of the
 * batch bounded by startPos (Listing 3 at P:227-290; readings
 * L1-L6 in DESIGN.md).  Blocks: k < n = min(*d_n_blocks, cap), block k =
 * d_bytes[d_start[k], d_start[k+1]) (the last one ends at nbytes); d_start
 * must be strictly increasing with d_start[0] == 0 (e.g. dedup_op_chunk's
 * d_cut_pos) -- other lists give unspecified (but in-bounds) results.
 * For every byte i < nbytes, inside its block [bs, be), writes the longest
 * match length L = d_match_len[i] (u8) of block[c..c+L) == block[i..i+L) over
 *     max(i - window, bs) <= c < i,  c + L <= i,  i + L <= be,  L <= max_coded
 * (the earliest c among the longest; L = 0 when no earlier byte in the
 * window equals byte i) and d_match_off[i] = (c - bs) mod window (u16; 0 when
 * L = 0).  d_skip (optional, u8 per block): positions of blocks with a
 * non-zero flag (duplicates) get L = 0, offset 0.
 * d_bytes 16-byte aligned and readable to nbytes rounded up to 16;
 * nbytes < 2^31; 1 <= window <= 16384; 1 <= max_coded <= 255; else EINVAL. */
dedup_status dedup_op_findmatch(dedup_ctx* c, void* stream, const uint8_t* d_bytes,
                                uint64_t nbytes, const uint32_t* d_start,
                                const uint32_t* d_n_blocks, uint64_t cap, const uint8_t* d_skip,
                                uint32_t window, uint32_t max_coded, uint8_t* d_match_len,
                                uint16_t* d_match_off);

/* ------------------------------------------------------------------------ */
/* 3. Row NEXT-3: the host-side archive writer               */
/* ------------------------------------------------------------------------ */
/* The paper's CPU consumer of the GPU stages: "we used the result of the
 * kernel function to run the compression on each block and generate the
 * compressed data", then "reorders the batches and writes it in the
 * output".  All pointers HOST; no GPU work.  Format (reading A1 in
 * DESIGN.md): per chunk in order, 'U' digest[20] u32 raw_len u32 tok_len
 * tokens (unique) or 'D' digest[20] (duplicate); tokens = greedy LZSS over
 * FindMatch's output (a match of length >= 3 is a 2-byte token
 * (offset & 0xFFF) | (length - 3) << 12, else a literal), in groups of 8
 * behind a flag byte (bit set = literal). */

/* Encodes one batch: chunk k = data[starts[k], starts[k+1]) (the last ends
 * at nbytes; starts[0] == 0, increasing), digest[20k..] (row A4), is_dup[k]
 * (row A7/A8), match_len / match_off per byte (dedup_op_findmatch output,
 * copied to the host).  window must be 4096 and 3 <= max_coded <= 18 (the
 * 12 + 4 bit token).  Returns the bytes written to out, DEDUP_ENOMEM if
 * out_cap is too small, DEDUP_EINVAL on bad arguments. */
int64_t dedup_archive_encode(const uint8_t* data, uint64_t nbytes, const uint32_t* starts,
                             uint32_t n_chunks, const uint8_t* digest, const uint8_t* is_dup,
                             const uint8_t* match_len, const uint16_t* match_off,
                             uint32_t window, uint32_t max_coded, uint8_t* out,
                             uint64_t out_cap);

/* Decoder state across batches (the digest -> chunk map that 'D' records
 * refer to).  new returns NULL for a window other than 4096. */
typedef struct dedup_archive_decoder dedup_archive_decoder;
dedup_archive_decoder* dedup_archive_decoder_new(uint32_t window);
void dedup_archive_decoder_free(dedup_archive_decoder* d);

/* Decodes the records in[0, in_len) (whole records, in stream order) into
 * out; returns the bytes written, DEDUP_ENOMEM / DEDUP_EINVAL (malformed
 * input or a reference to an unknown digest). */
int64_t dedup_archive_decode(dedup_archive_decoder* d, const uint8_t* in, uint64_t in_len,
                             uint8_t* out, uint64_t out_cap);

/* ------------------------------------------------------------------------ */
/* 4. Multi-GPU wave pipeline (rows A5-A8 at G > 1), NCCL      */
/* ------------------------------------------------------------------------ */
/* One process (and one dedup_dist) per GPU.  In wave w every rank submits
 * one batch; its local rows (chunk, SHA-1, local combine, route by digest
 * owner) run on one of `depth` slots; when `depth` waves are in flight the
 * oldest completes: the 32-byte records are exchanged with grouped
 * ncclSend/ncclRecv (their per-owner counts were exchanged right behind the
 * wave's local rows, on a communicator split from the first, so the host
 * waits only for those; DEDUP_DIST_EARLY_COUNTS=0 exchanges them at
 * completion on the first one and must then be set alike on every rank,
 * as the split is collective), the owner inserts + looks up its shard (row
 * A7), the first ids come back (row A8) and the results are copied to
 * pinned host memory.  Every rank must make the same sequence of submit /
 * flush / end_stream calls (NCCL matches them in order). */
typedef struct dedup_dist dedup_dist;

/* A 128-byte NCCL unique id (rank 0 creates it, the others receive it). */
dedup_status dedup_nccl_unique_id(uint8_t out[128]);

/* cfg: the owner config of this rank (device, owner_rank = rank,
 * num_owners = nranks, table_capacity = this shard's expected distinct
 * digests; the chunker fields apply to every batch).  batch_bytes /
 * batch_items: the largest batch a wave may submit on this rank. */
dedup_status dedup_dist_create(const dedup_config* cfg, const uint8_t nccl_id[128], int nranks,
                               int rank, uint32_t depth, uint64_t batch_bytes,
                               uint32_t batch_items, dedup_dist** out);
void dedup_dist_destroy(dedup_dist* d);
const char* dedup_dist_last_error(const dedup_dist* d);

/* Submits this rank's batch of the next wave: d_bytes (device, 16-byte
 * aligned, after `producer`'s current work), item_off (host, n_items + 1
 * offsets, item_off[0] = 0, non-decreasing, item_off[n_items] = nbytes),
 * items get seq = first_seq + k.  Arguments are checked before anything is
 * enqueued (EINVAL).  If `depth` waves were in flight, the oldest completes
 * first and *completed = 1: read it with dedup_dist_result before the next
 * call.  A digest-table overflow of any owner shard (replies of ~0) makes
 * the completing call return the sticky DEDUP_ETABLEFULL; an NCCL error
 * (polled with ncclCommGetAsyncError while the host waits) aborts the
 * communicators and returns the sticky DEDUP_ENCCL. */
dedup_status dedup_dist_submit(dedup_dist* d, const uint8_t* d_bytes, uint64_t nbytes,
                               const uint64_t* item_off, uint32_t n_items, uint64_t first_seq,
                               void* producer, uint32_t* completed);
/* Completes the oldest wave in flight if any (*completed = 1). */
dedup_status dedup_dist_flush(dedup_dist* d, uint32_t* completed);
/* Makes `stream` (cudaStream_t as void*) wait for the results of every
 * completed wave (no host synchronisation); call after the flushes, e.g. to
 * bracket the pipeline with CUDA events. */
dedup_status dedup_dist_join(dedup_dist* d, void* stream);
/* New dedup stream (clears this rank's table shard).  With waves in flight
 * the reset is deferred: it is issued on the owner stream right before the
 * owner work of the next wave submitted, so the waves in flight still see
 * the old stream's table and the pipeline is not drained (every rank must
 * call it at the same wave). */
dedup_status dedup_dist_end_stream(dedup_dist* d);

typedef struct {
    uint64_t first_seq;
    uint32_t n_items, n_chunks;
    const uint64_t* item_off;          /* [n_items + 1] batch-relative */
    const uint32_t* item_first_chunk;  /* [n_items], 0xFFFFFFFF for empty items */
    const uint32_t* chunk_start;       /* [n_chunks] item-relative */
    const uint8_t* digest;             /* [n_chunks * 20] */
    const uint64_t* first_id;          /* [n_chunks] */
    const uint8_t* is_dup;             /* [n_chunks] */
} dedup_wave_result;
/* The last completed wave's results: waits until they are in host memory;
 * the views stay valid until that slot completes again (`depth`
 * completions later). */
dedup_status dedup_dist_result(const dedup_dist* d, dedup_wave_result* out);
/* The last completed wave's item count, chunk count and bytes, without
 * waiting for its results to reach host memory. */
dedup_status dedup_dist_last_counts(const dedup_dist* d, uint32_t* n_items, uint32_t* n_chunks,
                                    uint64_t* nbytes);

/* Kernels this rank's pipeline has launched so far. */
uint64_t dedup_dist_kernel_launches(const dedup_dist* d);
/* Bytes this rank has sent to OTHER ranks so far (32-byte records of row A6
 * and 8-byte replies of row A8, counted at completion). */
uint64_t dedup_dist_a2a_bytes(const dedup_dist* d);

/* Number of kernels this ctx has launched so far (all layers). */
uint64_t dedup_kernel_launches(const dedup_ctx* c);

/* ------------------------------------------------------------------------ */
/* 5. Measured roofline denominators ("Integer-op peak. Not in */
/*    MEASURED_PEAKS: microbenchmark LOP3/SHF/IADD3 throughput on B200")     */
/* ------------------------------------------------------------------------ */
typedef struct {
    /* thread-level integer ops per second (1e12) of one instruction kind on
     * the whole GPU: 8 independent chains per thread, 2 x 1024 threads per
     * SM.  lop3 / shf / iadd3 / prmt / lea_hi issue to the ALU pipe, imad /
     * imad_hi to the FMA pipe; mix_lop3_imad alternates LOP3 and IMAD (both
     * pipes, the issue-slot limit). */
    double lop3, shf, iadd3, imad, imad_hi, prmt, lea_hi, mix_lop3_imad;
    int32_t num_sms, clock_mhz_attr;
} dedup_int_rates;

/* Runs the probe kernels on `device` (about 1 s; device-wide, do not run
 * beside other work).  Errors: EINVAL (out NULL), ENOMEM, ECUDA. */
dedup_status dedup_probe_int_rates(int32_t device, dedup_int_rates* out);

#ifdef __cplusplus
}
#endif
#endif /* DEDUP_B200_H */
