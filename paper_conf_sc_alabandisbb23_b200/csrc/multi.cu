// multi.cu -- multi-GPU layer (edge-partitioned single graph over NCCL).  Filled in below.
#include <string.h>

#include "driver.h"

using namespace eclscc;

extern "C" {

int ecl_scc_get_unique_id(uint8_t id[128]) {
    clear_err();
    if (!id) return fail(ECL_SCC_EINVAL, "NULL id");
    memset(id, 0, 128);
    return fail(ECL_SCC_EUNSUPPORTED, "partitioned mode not built yet");
}
int ecl_scc_comm_create(int32_t, int32_t, const uint8_t*, ecl_scc_comm_t*) {
    return fail(ECL_SCC_EUNSUPPORTED, "partitioned mode not built yet");
}
int ecl_scc_comm_destroy(ecl_scc_comm_t) { return ECL_SCC_OK; }
int ecl_scc_partitioned(ecl_scc_comm_t, int32_t, int32_t, int32_t, int64_t, const int32_t*, const int32_t*,
                        int32_t*, ecl_scc_stream_t, ecl_scc_stats*) {
    return fail(ECL_SCC_EUNSUPPORTED, "partitioned mode not built yet");
}
int ecl_scc_partitioned_emulated(int32_t, int32_t, int64_t, const int32_t*, const int32_t*, int32_t*,
                                 ecl_scc_stream_t, ecl_scc_stats*) {
    return fail(ECL_SCC_EUNSUPPORTED, "partitioned mode not built yet");
}
}
