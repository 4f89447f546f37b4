// driver.h -- internal interface between the single-GPU driver and the multi-GPU layer.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <vector>

#include "../../include/ecl_scc.h"
#include "common.cuh"
#include "halo.cuh"

namespace eclscc {

// Workspace of one device.  All arrays are device memory.
struct Plan {
    uint32_t flags;
    int32_t n_cap;
    int64_t m_cap;
    int64_t nw_cap, bsum_cap, chunk_cap;
    // double-buffered working graph in local numbering (kernels.cuh "Layout")
    int32_t *act[2], *cin[2], *cout[2];  // vertex IDs and signatures v_in / v_out
    int32_t *optr[2], *iptr[2];          // CSR / CSC offsets
    int32_t *oadj[2], *iadj[2];          // CSR / CSC adjacency
    int32_t *min_in[2], *min_out[2];     // ECL_SCC_FOUR_SIG: minimum signatures (mirrored), per buffer
    int32_t* t2;                         // ECL_SCC_TRIM2: Trim-2 partner per local vertex (-1: none)
    int32_t* hpos[2];                    // partitioned mode: halo position per local vertex, per buffer
    int32_t* slot;                       // ECL_SCC_COMPRESS / RAISE: priority -> local index
    int32_t lab_lo, lab_hi;              // label ownership: labels[v] written only for lab_lo <= v < lab_hi
    WGraph gk;                           // the graph of the compaction in progress (keep -> finish)
    int32_t *kin, *kout;                 // two n+1 int views (ingest histogram / cursor, relabel, levels)
    int2* kio;                           // the same memory as interleaved kept degrees {in, out} (compaction)
    int32_t* newidx;                     // old local -> new local (-1: leaves)
    int2* cnt;                           // per-vertex surviving (out, in) degree
    uint2* emask;                        // light rows: kept, then surviving, entries as bit masks
    int2* sig2;                          // power-law Phase 3: (v_in, v_out) interleaved copy
    int4 *wsum, *wscan;                  // per-warp compaction counts (alive, out, in, kept) and their prefix
    void* bsum;                          // scan block totals
    void* chunks;                        // long-row chunks, 2 x Chunk[chunk_cap] (current / next graph)
    int* chunk_cnt;                      // survivors per chunk of the current graph
    int2* hcnt;                          // survivors of a vertex's long rows
    int cb;                              // which chunk buffer belongs to the current graph
    int nchunks_cur;                     // chunks of the current graph
    DevCounters* dc;                     // device counters
    DevCounters* hc;                     // pinned host mirror
    int32_t* u_rp;                       // batched: union CSR and union labels
    int32_t* u_ci;
    int32_t* u_lab;
    int64_t u_n_cap, u_m_cap;
    void* u_desc;                        // batched: the per-graph table of the union kernels
    int u_desc_cap;
    uint8_t* dirty;                      // 2 x dirty_cap tile flags (Phase-2 skipping)
    int64_t dirty_cap;
    // storage reordering (reorder.cuh): permuted input CSR and the storage -> caller ID map
    int32_t *rp2, *ci2, *orig, *pos, *cellv, *fa, *fb, *cellbuf, *rcnt;
    const int32_t* orig_cur;             // orig when the current run is reordered, else null
    unsigned long long *pnin, *pnout;    // tile packs (pack.cuh): slot words per local vertex
    int2* ext;                           // tile packs: cut edges per tile
    bool pack_fused;                     // the last compaction's scatter wrote the tile pack
    int* ext_cnt;                        // tile packs: cut edges of each tile
    int* aq_state;                       // asynchronous Phase 2 (pack.cuh AsyncQ)
    uint8_t* aq_seen;
    unsigned long long* aq_ctr;
    int64_t aq_resident;                 // resident CTAs of k_prop_async (this plan's device)
    int device;                          // the device the plan was created on
    bool tile_attrs;                     // k_prop_tile / k_prop_pack attributes set on `device`
    // tuning knobs, read from the environment once when the plan is created (development
    // only; the defaults are the measured best): ECL_SCC_RUN, ECL_SCC_CLAIM,
    // ECL_SCC_CLAIM_DIV, ECL_SCC_CLAIM_MAX, ECL_SCC_ASYNC_CTAS
    int knob_run, knob_claim, knob_claim_div, knob_claim_max, knob_async_ctas, knob_lv_ctas;
    void* lv_ctl;                        // levels.cuh LvCtl (device)
    int32_t *h_rp, *h_ci, *h_lab;        // ecl_scc_host: device copies of the caller's host buffers
    int64_t h_n_cap, h_m_cap;
    int64_t hb_rp_cap, hb_ci_cap, hb_lab_cap;   // ecl_scc_batched_host: staging of a whole batch
    int32_t *hb_rp, *hb_ci, *hb_lab;
    int lv_resident;                     // co-resident CTAs of k_lv_run
    int64_t lk_resident;                 // resident CTAs of k_lk_run (levels, tile mode)
    bool kw;                             // compaction with 4-byte keep words (rows <= KW_DEG)
    int64_t launches;                    // kernels launched by the current call
    cudaEvent_t ev[6];                   // stage timing (ECL_SCC_TIME_STAGES)
    bool ev_ok;
    bool low_locality;                   // fewer than 25% of the input edges inside 2048-ID ranges
};

// all-reduce over the ranks of this process (1 with NCCL, P when emulated).  Every exchange
// is bracketed by CUDA events on the call's stream (stats->ms_comm: the communication
// share); the event pool is owned by the caller (a plan) and reused.
struct HaloRank;
struct Exchange {
    std::vector<cudaEvent_t>* ev = nullptr;   // pool of event pairs
    int used = 0;                             // pairs recorded by the current call
    int64_t bytes = 0;                        // bytes this rank contributed
    virtual ~Exchange() {}
    // op 0 = MAX, 1 = SUM; bufs[r] = rank r's buffer of `count` int32
    virtual int reduce(std::vector<int32_t*>& bufs, int64_t count, int op, cudaStream_t s) = 0;
    // partitioned (halo) mode: give every rank an exchange buffer of 2*entries int32 and the
    // push targets of the propagation kernel (R[r]->push)
    virtual int halo_buffers(std::vector<HaloRank*>& R, int64_t entries, cudaStream_t s) = 0;
    int allreduce(std::vector<int32_t*>& bufs, int64_t count, int op, cudaStream_t s);
    double ms() const;                        // after a stream synchronisation
};

// One rank of the edge-partitioned mode (halo.cuh): its rows, its local graph and the
// single-GPU workspace that runs it.
struct HaloRank {
    Plan p;                                   // workspace of the local graph
    int32_t n = 0, rb = 0, re = 0, nloc = 0, ng = 0;
    int64_t m = 0, m_cap = 0;
    const int32_t *rp = nullptr, *ci = nullptr;   // the caller's rows (global destination IDs)
    int32_t *lrp = nullptr, *lci = nullptr;   // local CSR (owned rows, then the ghosts' empty rows)
    int32_t* l2g = nullptr;                   // local -> global ID
    int32_t *gmark = nullptr, *gidx = nullptr;    // [n] ghost marks (then halo membership) / scans
    int32_t* lab = nullptr;                   // [n] encoded labels of the owned vertices
    int32_t* hbuf = nullptr;                  // [2*hcap] signature exchange buffer (in, out per entry)
    int32_t* hdeg = nullptr;                  // [2*hcap] kept-degree exchange buffer
    int64_t hcap = 0, H = 0;                  // capacity / current size of the halo
    bool hbuf_external = false;               // hbuf owned by the exchange (symmetric memory)
    int32_t* words = nullptr;                 // device: [0] injected, [1] live edges, [2] err
    HaloPush push{};                          // where k_prop_async pushes raised halo copies
    // loop state
    WGraph g{};
    int ob = 1;
    ~HaloRank();
};
int halo_rank_alloc(HaloRank* R, int32_t n, int32_t rb, int32_t re, int64_t m_cap, uint32_t flags);
int run_halo(std::vector<HaloRank*>& R, Exchange& X, int32_t n, uint32_t flags, int32_t* labels, cudaStream_t s,
             ecl_scc_stats* st);

int fail(int status, const char* fmt, ...);
void clear_err();
const char* last_err();
int plan_alloc(Plan* p, int32_t n_max, int64_t m_max);
void plan_free(Plan* p);
int run_graph(Plan* p, int32_t n, int64_t nnz, const int32_t* rp, const int32_t* ci, int32_t* labels,
              cudaStream_t s, ecl_scc_stats* st, int stop_iter, int32_t* dbg_in, int32_t* dbg_out);

}  // namespace eclscc
