// driver.h -- internal interface between the single-GPU driver and the multi-GPU layer.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "../../include/ecl_scc.h"
#include "common.cuh"

namespace eclscc {

// Workspace of one device.  All arrays are device memory.
struct Plan {
    uint32_t flags;
    int32_t n_cap;
    int64_t m_cap;
    int64_t nw_cap, bsum_cap;
    int32_t *sig_in, *sig_out;          // v_in / v_out (v_in may be the caller's labels_out)
    int32_t *kin, *kout;                // kept in/out degree (global-indexed), CSC cursor
    int32_t *act[2], *optr[2], *iptr[2];// double-buffered compacted working graph
    int32_t *oadj[2], *iadj[2];
    int4 *wsum, *wscan;                 // per-warp compaction counts and their prefix
    void* bsum;                         // scan block totals
    DevCounters* dc;                    // device counters
    DevCounters* hc;                    // pinned host mirror
    int32_t* u_rp;                      // batched: union CSR
    int32_t* u_ci;
    int64_t u_n_cap, u_m_cap;
};

int fail(int status, const char* fmt, ...);
void clear_err();
const char* last_err();
int plan_alloc(Plan* p, int32_t n_max, int64_t m_max);
void plan_free(Plan* p);
int run_graph(Plan* p, int32_t n, int64_t nnz, const int32_t* rp, const int32_t* ci, int32_t* vin,
              cudaStream_t s, ecl_scc_stats* st, int stop_iter, int32_t* dbg_in, int32_t* dbg_out);

}  // namespace eclscc
