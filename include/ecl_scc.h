/*
 * ecl_scc.h -- C ABI of the B200-native ECL-SCC hot path (libeclscc.so).
 *
 * Citation key: P:n = line n of the paper's text (Alabandi, Sands, Biros, Burtscher,
 * "A GPU Algorithm for Detecting Strongly Connected Components", SC'23).
 *
 * WHAT IS COMPUTED.  Input: "a directed graph G = (V, E) with unique vertex IDs" (P:116,
 * Alg. 1 "Input"); vertex IDs are CSR row indices 0..n-1 (reading 8).
 * Output: "for all v: v_in (and v_out) denotes to which SCC vertex v belongs" (P:156,
 * Alg. 1 "Output"); the signature of an SCC is its highest vertex ID (Sec. 3.2.1),
 * so labels_out[v] = max{ w : v and w are mutually reachable } -- a unique, schedule
 * independent answer, bit-exact against Tarjan.
 *
 * WHERE.  The graph is already on the GPU and the result is needed on the GPU;
 * every graph pointer below is a DEVICE pointer on the calling thread's current CUDA
 * device, unless marked "host".
 *
 * CONVENTIONS (all entry points).
 *  - Ownership: the caller owns every input and output buffer.  Inputs are never
 *    modified (the library compacts its own working copies).  The library owns its
 *    plan/workspace; passing a plan makes repeated calls allocation-free.
 *  - Errors: every call returns an ecl_scc_status and never aborts.  On error labels_out
 *    is unspecified; ecl_scc_last_error() returns a thread-local message.
 *      n == 0                                      -> ECL_SCC_OK, nothing written
 *      nnz == 0                                    -> labels[v] = v
 *      n < 0, nnz < 0, NULL pointer with n > 0     -> ECL_SCC_EINVAL
 *      row_ptr[0] != 0, row_ptr[n] != nnz, decreasing offsets, col_idx outside [0,n)
 *                                                  -> ECL_SCC_ERANGE (device validation
 *                                                     pass; skipped with ECL_SCC_NO_VALIDATE)
 *      nnz >= 2^31                                 -> ECL_SCC_EUNSUPPORTED (int32 offsets)
 *      workspace allocation failure                -> ECL_SCC_ENOMEM
 *      any CUDA runtime error                      -> ECL_SCC_ECUDA
 *  - Graph contents: self-loops and duplicate edges are accepted; they change no SCC
 *    (reading 9).
 *  - Synchrony: ecl_scc() returns after labels_out is written.  The _async form enqueues
 *    on `stream`; it waits on that stream only for the outer-loop convergence decision
 *    (one small device->host read per outer iteration), never on other streams.
 *  - Thread safety: distinct plans may be used concurrently from different host threads;
 *    a plan must not be used by two calls at once.
 */
#ifndef ECL_SCC_H
#define ECL_SCC_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct CUstream_st* ecl_scc_stream_t; /* == cudaStream_t; NULL = legacy default */

typedef enum {
    ECL_SCC_OK = 0,
    ECL_SCC_EINVAL = 1,
    ECL_SCC_ERANGE = 2,
    ECL_SCC_ENOMEM = 3,
    ECL_SCC_ECUDA = 4,
    ECL_SCC_ENCCL = 5,
    ECL_SCC_EUNSUPPORTED = 6
} ecl_scc_status;

/* plan flags (DESIGN.md "Readings" and "Kernels") */
#define ECL_SCC_NO_TRIM 0x1u      /* disable the Trim-1 round run with every edge removal */
#define ECL_SCC_COMPRESS 0x2u     /* variant: path compression (reading 4) -- a
                                     cut-edge pull takes max(in[u], in[in[u]]) (out likewise),
                                     through a priority -> local index map; two-signature method,
                                     single GPU */
#define ECL_SCC_NO_VALIDATE 0x4u  /* skip the device validation pass over row_ptr/col_idx */
#define ECL_SCC_SYNC_PASSES 0x8u  /* ablation: no block-local iteration, one Jacobi-like
                                     relaxation per global pass ("separate kernels") */
#define ECL_SCC_TIME_STAGES 0x10u /* record CUDA events around the stages (stats->ms_*) */
#define ECL_SCC_IDENTITY_IDS 0x20u /* propagate the raw vertex IDs instead of the internal
                                      priorities pi(v) (reading 16); labels are
                                      identical either way */
#define ECL_SCC_NO_DIRTY 0x40u    /* ablation: visit every tile in every Phase-2 pass */
/* 0x80u, 0x100u, 0x2000u: retired experimental variants (threshold stages, dependency-ordered
   sweeps, device-resident tail; measured negative) */
#define ECL_SCC_NO_REORDER 0x200u /* keep the caller's vertex numbering as the storage order
                                     (by default graphs without rows longer than 64 edges,
                                     n >= 16384 and fewer than 85% of the edges inside
                                     2048-ID ranges are renumbered into BFS-Voronoi cells) */
#define ECL_SCC_FORCE_REORDER 0x400u /* renumber into BFS-Voronoi cells whenever the graph has
                                        no row longer than 64 edges (tests, ablation) */
#define ECL_SCC_NO_PACK 0x800u    /* ablation: Phase 2 re-walks the CSR/CSC rows on every tile
                                     visit instead of reading per-iteration tile packs */
#define ECL_SCC_NO_ASYNC 0x1000u  /* ablation: Phase 2 as global passes (one launch each)
                                     instead of one persistent launch with a tile queue */
#define ECL_SCC_TRIM2 0x4000u     /* variant: Trim-2 in the same round as Trim-1 -- a pair
                                     u <-> w whose only kept in-edges (or only kept out-edges)
                                     are each other is an SCC of two (reading 17);
                                     EINVAL together with ECL_SCC_NO_TRIM */
#define ECL_SCC_HALO_ALLREDUCE 0x10000u /* partitioned mode, baseline exchange: combine the halo
                                     signatures with ncclAllReduce(MAX) after every local fixed
                                     point instead of the propagation kernel's peer pushes */
#define ECL_SCC_RAISE 0x20000u    /* variant: the sound form of the P:190 trick (DESIGN.md reading
                                     5) -- when v_in rises to t inside a tile, t is also offered to
                                     in[out[v]] (a descendant of v) if that vertex is in the same
                                     tile; v_out likewise to out[in[v]]; single GPU */
#define ECL_SCC_CLUSTER 0x40000u  /* variant: Phase 2 on thread-block-cluster pair tiles -- two
                                     CTAs share one 4096-vertex block-local fixed point through
                                     distributed shared memory (csrc/cluster.cuh); graphs
                                     without rows longer than 64 edges, single GPU */
#define ECL_SCC_NO_KW 0x80000u    /* ablation: the general compaction layout (8-byte kept degrees
                                     + 8-byte row masks per vertex) also for graphs whose rows
                                     have <= 8 entries, which otherwise use one 4-byte keep word */
#define ECL_SCC_FOUR_SIG 0x8000u  /* variant: the 4-signature method -- Phase 2 also
                                     propagates minimum ancestor / descendant IDs and Phase 3
                                     keeps an edge only if all four signatures agree; twice the
                                     signature memory and two Phase-2 fixed points per iteration */

#define ECL_SCC_TRACE_MAX 64

/* Per-run statistics (host struct, optional).  Index k = outer iteration k+1. */
typedef struct {
    int32_t iterations;                      /* outer iterations that ran Phase 2        */
    int32_t trace_len;                       /* min(iterations, ECL_SCC_TRACE_MAX)       */
    int64_t passes;                          /* global Phase-2 passes, all iterations; in
                                                the asynchronous mode (default for graphs
                                                without long rows): tile visits / tiles,
                                                rounded up, per iteration               */
    int64_t edges_in[ECL_SCC_TRACE_MAX];     /* live edges entering Phase 2 (after trim) */
    int64_t vertices_in[ECL_SCC_TRACE_MAX];  /* vertices with a live edge in Phase 2     */
    int64_t edges_kept[ECL_SCC_TRACE_MAX];   /* edges kept by Phase 3 (before next trim) */
    int64_t passes_iter[ECL_SCC_TRACE_MAX];  /* global passes of Phase 2, per iteration  */
    int64_t prop_bytes;                      /* algorithmic bytes of the Phase-2 work done
                                                (SURVEY 8(d) terms over the visited tiles) */
    int64_t kernel_launches;                 /* kernels this call launched                */
    /* device time per stage (CUDA events on the call's stream), only with
       ECL_SCC_TIME_STAGES; 0 otherwise */
    double ms_ingest;                        /* validation + CSC build                    */
    double ms_compact;                       /* Phase 3 + trim + compaction + Phase 1     */
    double ms_prop;                          /* Phase 2 (all passes)                      */
    double ms_prop_iter[ECL_SCC_TRACE_MAX];  /* Phase 2 of outer iteration k+1            */
    double ms_compact_iter[ECL_SCC_TRACE_MAX]; /* Phase 3 + compaction before iteration k+1 */
    /* multi-GPU (ecl_scc_partitioned): device time spent in the signature / degree / count
       exchanges (CUDA events around every collective on the call's stream), the bytes this
       rank contributed to them, and the number of exchanges; 0 for single-GPU calls */
    double ms_comm;
    int64_t comm_bytes;
    int64_t exchanges;
} ecl_scc_stats;

typedef struct ecl_scc_plan_s* ecl_scc_plan_t;

/* Workspace for graphs with n <= n_max, nnz <= nnz_max on the current device.
 * flags: ECL_SCC_* above.  Allocates device memory (about 24*n_max + 12*nnz_max bytes). */
int ecl_scc_plan_create(int32_t n_max, int64_t nnz_max, uint32_t flags, ecl_scc_plan_t* out);
int ecl_scc_plan_destroy(ecl_scc_plan_t plan);

/* Single graph, synchronous.  row_ptr: n+1 int32 offsets; col_idx: nnz int32 IDs;
 * labels_out: n int32 (written).  Uses a temporary plan with default flags. */
int ecl_scc(int32_t n, int64_t nnz, const int32_t* row_ptr, const int32_t* col_idx,
            int32_t* labels_out);

/* Single graph, on `stream`, with an optional plan (NULL: temporary) and optional host
 * stats (NULL: none).  Same arguments and layout as ecl_scc(). */
int ecl_scc_async(int32_t n, int64_t nnz, const int32_t* row_ptr, const int32_t* col_idx,
                  int32_t* labels_out, ecl_scc_stream_t stream, ecl_scc_plan_t plan,
                  ecl_scc_stats* stats);

/* Test/diagnostic entry: run until Phase 2 of outer iteration `stop_iter` (>= 1) has
 * reached its fixed point and write that iteration's signatures v_in -> sig_in[n] and
 * v_out -> sig_out[n] (device).  If the run terminates before stop_iter, both receive
 * the final labels.  Used for per-iteration parity against the oracle (DESIGN.md
 * reading 12: the state after each Phase 2 is schedule independent). */
int ecl_scc_debug_run(int32_t n, int64_t nnz, const int32_t* row_ptr, const int32_t* col_idx,
                      uint32_t flags, int32_t stop_iter, int32_t* sig_in, int32_t* sig_out,
                      ecl_scc_stream_t stream, ecl_scc_stats* stats);

/* Batch of G independent graphs on one GPU (one discrete ordinate each).
 * n, nnz: host arrays [G]; row_ptr, col_idx, labels_out: host arrays [G] of device
 * pointers.  Labels are per-graph LOCAL IDs (max local ID of the SCC).  The graphs are
 * solved together as one disjoint union (clusters never interact); a plan sized
 * for sum(n), sum(nnz) may be passed (NULL: temporary). */
int ecl_scc_batched(int32_t G, const int32_t* n, const int64_t* nnz,
                    const int32_t* const* row_ptr, const int32_t* const* col_idx,
                    int32_t* const* labels_out, ecl_scc_stream_t stream, ecl_scc_plan_t plan,
                    ecl_scc_stats* stats);

/* Same as ecl_scc_async, but row_ptr, col_idx and labels_out are HOST pointers (pinned
 * memory -- cudaMallocHost / cudaHostRegister -- gives full-speed copies).  The plan keeps
 * device copies (4*(n_max+1) + 4*nnz_max + 4*(n_max+1) bytes, allocated on first use); the
 * copies run on `stream`; returns after the labels are back on the host.  Errors as
 * ecl_scc_async (ERANGE from the device validation of the copied CSR). */
int ecl_scc_host(int32_t n, int64_t nnz, const int32_t* row_ptr, const int32_t* col_idx,
                 int32_t* labels_out, ecl_scc_stream_t stream, ecl_scc_plan_t plan,
                 ecl_scc_stats* stats);

/* ecl_scc_batched with HOST buffers: n, nnz, row_ptr, col_idx, labels_out as in
 * ecl_scc_batched, but row_ptr[g], col_idx[g] and labels_out[g] are HOST pointers (pinned
 * memory gives full-speed copies).  The plan (sized for the union: sum n, sum nnz) keeps
 * device staging copies of the whole batch (4*(sum n + G) + 4*sum nnz + 4*sum n bytes,
 * allocated on first use); the copies run on `stream`; returns after every graph's labels
 * are back on the host.  Errors as ecl_scc_batched. */
int ecl_scc_batched_host(int32_t G, const int32_t* n, const int64_t* nnz,
                         const int32_t* const* row_ptr, const int32_t* const* col_idx,
                         int32_t* const* labels_out, ecl_scc_stream_t stream, ecl_scc_plan_t plan,
                         ecl_scc_stats* stats);

/* ---- after SCC detection: the sweep schedule ------------------------------------ */
/* Levels of the SCC condensation (the step after SCC detection in the RTE application:
 * a transport sweep starts "from nodes with no incoming edges"; the paper tabulates
 * the condensation's "DAG depth" per mesh, Table 2).  levels_out[v] = length of the longest
 * path of the condensation DAG that ends in v's SCC (source SCCs: 0); SCCs of one level can
 * be swept concurrently.  *depth_out (host, nullable) = max level + 1 (0 for n == 0).
 * row_ptr/col_idx: the same device CSR given to ecl_scc(); labels: its device labels_out
 * (any labelling that gives every SCC, and only it, one value in [0, n)).  levels_out:
 * n int32, device, written.  Uses the plan's buffers as workspace (NULL: a temporary
 * plan).  Synchronous on `stream`.  Errors: EINVAL (arguments), ERANGE (a label outside
 * [0, n), or labels that induce a cyclic condensation, i.e. not the SCC partition). */
int ecl_scc_levels(int32_t n, int64_t nnz, const int32_t* row_ptr, const int32_t* col_idx,
                   const int32_t* labels, int32_t* levels_out, int32_t* depth_out,
                   ecl_scc_stream_t stream, ecl_scc_plan_t plan);

/* ---- multi-GPU: one large graph, edge-partitioned by source rows (SPMD) ---------- */
typedef struct ecl_scc_comm_s* ecl_scc_comm_t;

/* 128-byte NCCL unique id (rank 0 creates it; broadcast it out of band, e.g. over the
 * torch.distributed process group). */
int ecl_scc_get_unique_id(uint8_t id[128]);
/* Collective: every rank calls with the same id; binds to the current device. */
int ecl_scc_comm_create(int32_t nranks, int32_t rank, const uint8_t id[128], ecl_scc_comm_t* out);
int ecl_scc_comm_destroy(ecl_scc_comm_t comm);

/* Per-rank workspace of the partitioned mode (not collective): n global vertices, this
 * rank's source rows [row_begin, row_end), at most local_nnz_max local edges.  A plan makes
 * repeated ecl_scc_partitioned calls allocation-free.  flags: ECL_SCC_* (NO_TRIM,
 * NO_VALIDATE, IDENTITY_IDS are honoured). */
typedef struct ecl_scc_part_plan_s* ecl_scc_part_plan_t;
int ecl_scc_part_plan_create(int32_t n, int32_t row_begin, int32_t row_end, int64_t local_nnz_max,
                             uint32_t flags, ecl_scc_part_plan_t* out);
int ecl_scc_part_plan_destroy(ecl_scc_part_plan_t plan);

/* Collective over comm.  This rank owns source rows [row_begin, row_end) of the global
 * graph (n vertices): local_row_ptr has row_end-row_begin+1 offsets starting at 0,
 * local_col_idx holds local_nnz GLOBAL destination IDs.  Every rank runs the single-GPU path
 * on its rows (the owned vertices plus the destinations owned elsewhere, its ghosts); the
 * ranks exchange only the halo -- the vertices held by more than one rank (DESIGN.md section
 * 7): the kept degrees (Trim-1) once per outer iteration (ncclAllReduce SUM over the halo),
 * and in Phase 2 the signatures, pushed by the propagation kernel into every rank's halo
 * buffer (NCCL symmetric memory: NVLS multimem reduction or remote atomic max over NVLink)
 * with a one-word all-reduce as the barrier, until no rank's copy rises.
 * labels_out: n int32 on every rank (replicated result, one final ncclAllReduce).
 * plan: nullable (then a temporary workspace is allocated for this call).
 * Errors: invalid input on ANY rank makes every rank return ECL_SCC_ERANGE (the ranks agree
 * through the first exchange before any of them leaves); a CUDA or NCCL failure on one rank
 * leaves the communicator unusable (destroy it).  Trim-2 and the 4-signature variant are
 * not supported here (EUNSUPPORTED at plan creation).  stats->ms_comm / comm_bytes /
 * exchanges report the collectives of this rank (the fused pushes run inside the
 * propagation kernel and are not separately timed). */
int ecl_scc_partitioned(ecl_scc_comm_t comm, int32_t n, int32_t row_begin, int32_t row_end,
                        int64_t local_nnz, const int32_t* local_row_ptr,
                        const int32_t* local_col_idx, int32_t* labels_out,
                        ecl_scc_stream_t stream, ecl_scc_part_plan_t plan, ecl_scc_stats* stats);

/* Single-process emulation of the partitioned algorithm with P partitions on the
 * current device (P rank workspaces; the all-reduces are element-wise reductions over the P
 * buffers and the fused pushes target the P halo buffers of the same device).  Same
 * arithmetic and exchange protocol as ecl_scc_partitioned at P ranks; used to test the
 * partitioned path on one GPU.  Inputs as ecl_scc(); row ranges are chosen balanced by edge
 * count.  flags: as ecl_scc_part_plan_create (ECL_SCC_HALO_ALLREDUCE selects the baseline
 * exchange).  plan: nullable; from ecl_scc_emulated_plan_create for the same P, graph size
 * and flags (repeated calls without allocation). */
typedef struct ecl_scc_emulated_plan_s* ecl_scc_emulated_plan_t;
int ecl_scc_emulated_plan_create(int32_t P, int32_t n, int64_t nnz, const int32_t* row_ptr,
                                 uint32_t flags, ecl_scc_emulated_plan_t* out);
int ecl_scc_emulated_plan_destroy(ecl_scc_emulated_plan_t plan);
int ecl_scc_partitioned_emulated(int32_t P, int32_t n, int64_t nnz, const int32_t* row_ptr,
                                 const int32_t* col_idx, int32_t* labels_out, uint32_t flags,
                                 ecl_scc_stream_t stream, ecl_scc_emulated_plan_t plan,
                                 ecl_scc_stats* stats);

/* Diagnostics of a communicator: info[0] ranks, [1] this rank, [2] 1 if the NCCL device API
 * is in use for the fused halo exchange (peer pushes), [3] 1 if it uses NVLS multimem
 * reductions.  Filled after the first ecl_scc_partitioned call. */
int ecl_scc_comm_info(ecl_scc_comm_t comm, int32_t info[4]);

/* Diagnostics of the NVLS path of the fused halo exchange on the current device alone: a
 * one-device multicast object (cuMulticastCreate) bound to a buffer, the partitioned mode's
 * push kernel reducing into it through the multicast address with multimem.red.max, the
 * unicast view checked.  *checked = number of entries verified.  EUNSUPPORTED if the device
 * (or driver) has no multicast support. */
int ecl_scc_multimem_probe(int32_t* checked);

/* Host helper: split rows [0,n) into P contiguous ranges of about equal edge count
 * (binary search on the host row_ptr[n+1]); bounds_out[P+1] (host). */
int ecl_scc_partition_rows(int32_t P, int32_t n, const int32_t* row_ptr_host, int32_t* bounds_out);

/* Diagnostics: kernel event counters of the plan's last run (tile visits, block rounds,
 * warp drain iterations, vertex pushes, ...); all zero unless the library was built
 * with -DECL_PROF.  out: 8 host uint64. */
int ecl_scc_plan_counters(ecl_scc_plan_t plan, uint64_t out[8]);

const char* ecl_scc_status_string(int status);
const char* ecl_scc_last_error(void); /* thread-local, "" if none */
int ecl_scc_version(void);            /* 100 * major + minor */

#ifdef __cplusplus
}
#endif
#endif /* ECL_SCC_H */
