// mg.h -- internal interface of the multi-GPU engine (mg.cpp) for api.cpp.
// Not part of the C ABI (include/dedup.h).
#pragma once
#include <stdint.h>

#include "dedup.h"

namespace dd {
namespace mg {

struct CtxEngine;  // the multi-GPU engine behind a dedup_ctx (num_devices >= 2)

// true iff cfg selects the multi-GPU engine
inline bool wanted(const dedup_config* cfg) {
    return cfg->num_devices >= 2 || cfg->transport != 0;
}

dedup_status create(const dedup_config* cfg, CtxEngine** out, const char** why);
void destroy(CtxEngine* e);
const char* last_error(const CtxEngine* e);
dedup_status submit_host(CtxEngine* e, uint32_t n_items, const uint8_t* const* item_ptr,
                         const uint64_t* item_len, uint64_t* first_seq_out);
dedup_status submit_device(CtxEngine* e, const uint8_t* d_bytes, uint64_t nbytes,
                           const uint64_t* item_off, uint32_t n_items, void* producer,
                           uint64_t* first_seq_out);
dedup_status join(CtxEngine* e, void* stream);
dedup_status end_stream(CtxEngine* e);
dedup_status drain(CtxEngine* e, uint32_t max_items, int32_t wait_ms, dedup_item_result* out,
                   uint32_t* n_out);
uint64_t pending(const CtxEngine* e);
dedup_status stats(const CtxEngine* e, dedup_stats_t* out);
uint64_t kernel_launches(const CtxEngine* e);
int32_t next_device(const CtxEngine* e);

}  // namespace mg
}  // namespace dd
