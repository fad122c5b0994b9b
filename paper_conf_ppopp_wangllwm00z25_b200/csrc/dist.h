// dist.h — multi-GPU (one process per GPU) phase-1 driver over NCCL (§4.3).
#pragma once
#include <cstdint>
#include "gala.h"

struct DistCtx;
void dist_run(DistCtx* d, double gamma, double tol, int max_levels);
gala_status dist_get_labels(DistCtx* d, int32_t* out, int64_t n, int64_t* k, bool device);
void dist_numerator(DistCtx* d, __int128* N, int64_t* W, int64_t* p, int64_t* q);
void dist_free(DistCtx* d);
void dist_set_option(DistCtx* d, const char* key, int64_t value);
int64_t dist_trace_count(DistCtx* d);
gala_status dist_trace_record(DistCtx* d, int64_t i, int64_t* out12);
gala_status dist_trace_labels(DistCtx* d, int64_t i, int32_t* out, int64_t n_level);
