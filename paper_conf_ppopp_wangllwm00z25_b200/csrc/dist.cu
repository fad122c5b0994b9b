// dist.cu — multi-GPU driver (placeholder until the NCCL path lands).
#include "dist.h"

struct DistCtx {
    int dummy;
};
void dist_run(DistCtx*, double, double, int) {}
gala_status dist_get_labels(DistCtx*, int32_t*, int64_t, int64_t*, bool) { return GALA_E_STATE; }
void dist_numerator(DistCtx*, __int128*, int64_t*, int64_t*, int64_t*) {}
void dist_free(DistCtx* d) { delete d; }
void dist_set_option(DistCtx*, const char*, int64_t) {}
int64_t dist_trace_count(DistCtx*) { return 0; }
gala_status dist_trace_record(DistCtx*, int64_t, int64_t*) { return GALA_E_STATE; }
gala_status dist_trace_labels(DistCtx*, int64_t, int32_t*, int64_t) { return GALA_E_STATE; }

extern "C" gala_status gala_nccl_unique_id(void*) { return GALA_E_NCCL; }
extern "C" gala_status gala_graph_from_csr_dist(const void*, int, int, int, int64_t, int64_t, int64_t, const int64_t*,
                                                const int32_t*, const int64_t*, uintptr_t, gala_graph*) {
    return GALA_E_NCCL;
}
