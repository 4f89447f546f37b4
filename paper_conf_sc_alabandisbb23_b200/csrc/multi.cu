// multi.cu -- multi-GPU layer: one large graph edge-partitioned by source rows (SPMD, one
// process per GPU), signatures combined with NCCL all-reduce(MAX) over NVLink/NVSwitch.
//
// Per outer iteration (same rule R2 and trace as the single-GPU path):
//   keep (Phase 3) on own rows and columns   -> kept degrees
//   all-reduce SUM of kept degrees (trim needs global degrees)
//   Trim-1 on own edges; all-reduce SUM of live edges   (termination, reading 2)
//   Phase 1 reset of the unfinished on the replica
//   Phase 2: repeat { local fixed point on own edges; all-reduce MAX of [in|out|changed] }
//            until no rank changed anything (a consistent global fixed point)
// The same driver runs P emulated ranks on one device (the all-reduce is an element-wise
// reduction over the P replicas), which is how the path is tested with one GPU.
#include <cuda_runtime.h>
#include <nccl.h>
#include <string.h>

#include <algorithm>
#include <memory>
#include <vector>

#include "driver.h"
#include "kernels.cuh"
#include "partition.cuh"
#include "scan.cuh"

namespace eclscc {

#define CKM(call)                                                                                     \
    do {                                                                                              \
        cudaError_t _e = (call);                                                                      \
        if (_e != cudaSuccess)                                                                        \
            return fail(ECL_SCC_ECUDA, "%s:%d %s: %s", __FILE__, __LINE__, #call, cudaGetErrorString(_e)); \
    } while (0)
#define CKN(call)                                                                                     \
    do {                                                                                              \
        ncclResult_t _r = (call);                                                                     \
        if (_r != ncclSuccess)                                                                        \
            return fail(ECL_SCC_ENCCL, "%s:%d %s: %s", __FILE__, __LINE__, #call, ncclGetErrorString(_r)); \
    } while (0)

static inline unsigned gridn(int64_t work, int t = 256) {
    int64_t g = (work + t - 1) / t;
    return (unsigned)std::max<int64_t>(1, std::min<int64_t>(g, 0x7FFFFFFF));
}

// One rank's share of the graph (device memory).
struct PRank {
    int32_t rb = 0, re = 0, nloc = 0;
    int64_t m = 0;
    const int32_t *rp = nullptr, *ci = nullptr;  // caller's local CSR (rows rb..re-1)
    int32_t *wci = nullptr, *odeg = nullptr;     // working rows (compacted in place)
    int32_t *cp = nullptr, *cr = nullptr, *ideg = nullptr;   // CSC of own edges, n columns
    int32_t* sig = nullptr;                      // [in(n) | out(n) | changed(1)] replica
    int32_t* kdeg = nullptr;                     // [kin(n) | kout(n)]
    int32_t* cnt = nullptr;                      // [live edges (int32 for the SUM), err, ring(RING), touched]
    unsigned long long* live = nullptr;
    void* bsum = nullptr;
    int32_t* grand = nullptr;
    ~PRank() {
        cudaFree(wci); cudaFree(odeg); cudaFree(cp); cudaFree(cr); cudaFree(ideg);
        cudaFree(sig); cudaFree(kdeg); cudaFree(cnt); cudaFree(live); cudaFree(bsum); cudaFree(grand);
    }
    int* ring() const { return cnt + 2; }
    int* touched() const { return cnt + 2 + RING; }
};

// all-reduce over the ranks of this process (1 with NCCL, P when emulated).  Every exchange
// is bracketed by CUDA events on the call's stream (stats->ms_comm: the communication
// share); the event pool is owned by the caller (a plan) and reused.
struct Exchange {
    std::vector<cudaEvent_t>* ev = nullptr;   // pool of event pairs
    int used = 0;                             // pairs recorded by the current call
    int64_t bytes = 0;                        // bytes this rank contributed
    virtual ~Exchange() {}
    // op 0 = MAX, 1 = SUM; bufs[r] = rank r's buffer of `count` int32
    virtual int reduce(std::vector<int32_t*>& bufs, int64_t count, int op, cudaStream_t s) = 0;
    int allreduce(std::vector<int32_t*>& bufs, int64_t count, int op, cudaStream_t s) {
        cudaEvent_t a = nullptr, b = nullptr;
        if (ev) {
            if ((size_t)(2 * used + 2) > ev->size()) {
                for (int k = 0; k < 2; k++) {
                    cudaEvent_t e;
                    CKM(cudaEventCreate(&e));
                    ev->push_back(e);
                }
            }
            a = (*ev)[2 * used];
            b = (*ev)[2 * used + 1];
            used++;
            CKM(cudaEventRecord(a, s));
        }
        if (int r = reduce(bufs, count, op, s)) return r;
        if (ev) CKM(cudaEventRecord(b, s));
        bytes += 4 * count;
        return ECL_SCC_OK;
    }
    double ms() const {                       // after a stream synchronisation
        double t = 0;
        for (int k = 0; ev && k < used; k++) {
            float x = 0.f;
            if (cudaEventElapsedTime(&x, (*ev)[2 * k], (*ev)[2 * k + 1]) == cudaSuccess) t += x;
            else cudaGetLastError();
        }
        return t;
    }
};

struct EmulatedExchange : Exchange {
    int32_t** dptrs = nullptr;
    int P = 0;
    explicit EmulatedExchange(int p) : P(p) {}
    ~EmulatedExchange() { cudaFree(dptrs); }
    int reduce(std::vector<int32_t*>& bufs, int64_t count, int op, cudaStream_t s) override {
        if (P == 1) return ECL_SCC_OK;
        if (!dptrs) CKM(cudaMalloc((void**)&dptrs, sizeof(int32_t*) * P));
        CKM(cudaMemcpyAsync(dptrs, bufs.data(), sizeof(int32_t*) * P, cudaMemcpyHostToDevice, s));
        part::k_reduce_replicas<<<std::min<unsigned>(gridn(count), 148 * 8), 256, 0, s>>>(P, dptrs, count, op);
        CKM(cudaGetLastError());
        return ECL_SCC_OK;
    }
};

struct NcclExchange : Exchange {
    ncclComm_t comm;
    explicit NcclExchange(ncclComm_t c) : comm(c) {}
    int reduce(std::vector<int32_t*>& bufs, int64_t count, int op, cudaStream_t s) override {
        CKN(ncclAllReduce(bufs[0], bufs[0], (size_t)count, ncclInt32, op == 0 ? ncclMax : ncclSum, comm, s));
        return ECL_SCC_OK;
    }
};

static int rank_alloc(PRank& R, int32_t n) {
    const size_t m = (size_t)std::max<int64_t>(R.m, 1), n1 = (size_t)n + 1;
    cudaError_t e = cudaSuccess;
    e = e ? e : cudaMalloc((void**)&R.wci, m * 4);
    e = e ? e : cudaMalloc((void**)&R.odeg, (size_t)std::max(R.nloc, 1) * 4);
    e = e ? e : cudaMalloc((void**)&R.cp, n1 * 4);
    e = e ? e : cudaMalloc((void**)&R.cr, m * 4);
    e = e ? e : cudaMalloc((void**)&R.ideg, n1 * 4);
    e = e ? e : cudaMalloc((void**)&R.sig, (2 * n1 + 1) * 4);
    e = e ? e : cudaMalloc((void**)&R.kdeg, 2 * n1 * 4);
    e = e ? e : cudaMalloc((void**)&R.cnt, (3 + RING) * 4);
    e = e ? e : cudaMalloc((void**)&R.live, 8);
    e = e ? e : cudaMalloc((void**)&R.bsum, ((n1 + SCAN_TILE - 1) / SCAN_TILE + 1) * sizeof(int4));
    e = e ? e : cudaMalloc((void**)&R.grand, 16);
    if (e != cudaSuccess) {
        cudaGetLastError();
        return fail(ECL_SCC_ENOMEM, "partition workspace: %s", cudaGetErrorString(e));
    }
    return ECL_SCC_OK;
}

__global__ void k_copy_flag(const int* __restrict__ touched, int32_t* __restrict__ dst, int err) {
    *dst = err ? err : *touched;
}
__global__ void k_live_to_i32(const unsigned long long* __restrict__ live, int32_t* __restrict__ dst) {
    *dst = (int32_t)*live;
}

// The partitioned driver over this process's ranks R (1 with NCCL, P when emulated).
// Every rank's graph pointers are device pointers on the current device.
static int run_partitioned(std::vector<PRank*>& R, Exchange& X, int32_t n, uint32_t flags, int32_t* labels,
                           cudaStream_t s, ecl_scc_stats* st) {
    const int P = (int)R.size();
    if (st) memset(st, 0, sizeof(*st));
    const Prio Pr = make_prio((uint32_t)n, (flags & ECL_SCC_IDENTITY_IDS) != 0);
    const bool trim = !(flags & ECL_SCC_NO_TRIM);
    std::vector<int32_t*> sigs(P), kdegs(P), cnts(P);
    int32_t hbuf[4];
    int64_t launches = 0;
    // ---- ingest: validation, working rows, CSC of own edges
    for (int r = 0; r < P; r++) {
        PRank& Q = *R[r];
        sigs[r] = Q.sig; kdegs[r] = Q.kdeg; cnts[r] = Q.cnt;
        CKM(cudaMemsetAsync(Q.cnt, 0, (3 + RING) * 4, s));
        if (!(flags & ECL_SCC_NO_VALIDATE) && Q.nloc > 0) {
            part::k_validate_part<<<std::min<unsigned>(gridn(std::max<int64_t>(Q.nloc, Q.m)), 148 * 16), 256, 0, s>>>(
                Q.nloc, Q.m, Q.rp, Q.ci, n, Q.cnt + 1);
            launches++;
        }
    }
    {   // every rank learns whether any rank's input is invalid, so all return together
        // instead of leaving the others blocked in the next collective
        std::vector<int32_t*> errs(P);
        for (int r = 0; r < P; r++) errs[r] = R[r]->cnt + 1;
        if (int e = X.allreduce(errs, 1, 0, s)) return e;
        CKM(cudaMemcpyAsync(hbuf, R[0]->cnt, 8, cudaMemcpyDeviceToHost, s));
        CKM(cudaStreamSynchronize(s));
        if (hbuf[1]) return fail(ECL_SCC_ERANGE, "partitioned: invalid local CSR on some rank");
    }
    for (int r = 0; r < P; r++) {
        PRank& Q = *R[r];
        if (Q.nloc > 0) {
            part::k_copy_rows<<<gridn(Q.nloc), 256, 0, s>>>(Q.nloc, Q.rb, Q.rp, Q.ci, Q.wci, Q.odeg);
            launches++;
        }
        CKM(cudaMemsetAsync(Q.ideg, 0, sizeof(int32_t) * (size_t)(n + 1), s));
        if (Q.nloc > 0) {
            part::k_indeg_rows<<<gridn(Q.nloc), 256, 0, s>>>(Q.nloc, Q.rp, Q.wci, Q.odeg, Q.ideg);
            launches++;
        }
        const int64_t nb = std::max<int64_t>((n + SCAN_TILE - 1) / SCAN_TILE, 1);
        k_scan_reduce<I1><<<(unsigned)nb, SCAN_THREADS, 0, s>>>((const I1*)Q.ideg, n, (I1*)Q.bsum);
        k_scan_top<I1><<<1, SCAN_THREADS, 0, s>>>((I1*)Q.bsum, nb, (I1*)Q.grand);
        k_scan_apply<I1><<<(unsigned)nb, SCAN_THREADS, 0, s>>>((const I1*)Q.ideg, n, (I1*)Q.bsum, (I1*)Q.cp,
                                                               (const I1*)Q.grand, 1);
        launches += 3;
        CKM(cudaMemsetAsync(Q.kdeg, 0, sizeof(int32_t) * (size_t)n, s));     // cursor
        if (Q.nloc > 0) {
            part::k_csc_rows<<<gridn(Q.nloc), 256, 0, s>>>(Q.nloc, Q.rb, Q.rp, Q.wci, Q.odeg, Q.cp, Q.kdeg, Q.cr);
            launches++;
        }
        part::k_init_prio<<<std::min<unsigned>(gridn(n), 148 * 16), 256, 0, s>>>(n, Q.sig, Q.sig + n, Pr);
        launches++;
        CKM(cudaGetLastError());
    }
    int iters = 0;
    int64_t passes_total = 0;
    for (int iter = 1;; iter++) {
        if (iter > n + 2) return fail(ECL_SCC_ECUDA, "internal: partitioned outer loop exceeded n+2 iterations");
        const int first = iter == 1;
        // ---- Phase 3 (keep) with kept degrees, summed over ranks
        for (int r = 0; r < P; r++) {
            PRank& Q = *R[r];
            CKM(cudaMemsetAsync(Q.kdeg, 0, sizeof(int32_t) * 2 * (size_t)n, s));
            if (Q.nloc > 0) {
                part::k_keep_rows<<<gridn(Q.nloc), 256, 0, s>>>(Q.nloc, Q.rb, Q.rp, Q.wci, Q.odeg, Q.sig, Q.sig + n,
                                                                first, Q.kdeg + n);
                launches++;
            }
            part::k_keep_cols<<<gridn(n), 256, 0, s>>>(n, Q.cp, Q.cr, Q.ideg, Q.sig, Q.sig + n, first, Q.kdeg);
            launches++;
        }
        if (int e = X.allreduce(kdegs, 2 * (int64_t)n, 1, s)) return e;
        // ---- Trim-1 with global degrees; live edges summed over ranks
        for (int r = 0; r < P; r++) {
            PRank& Q = *R[r];
            CKM(cudaMemsetAsync(Q.live, 0, 8, s));
            if (Q.nloc > 0) {
                part::k_trim_rows<<<gridn(Q.nloc), 256, 0, s>>>(Q.nloc, Q.rb, Q.rp, Q.wci, Q.odeg, Q.kdeg, Q.kdeg + n,
                                                                trim, Q.live);
                launches++;
            }
            part::k_trim_cols<<<gridn(n), 256, 0, s>>>(n, Q.cp, Q.cr, Q.ideg, Q.kdeg, Q.kdeg + n, trim);
            k_live_to_i32<<<1, 1, 0, s>>>(Q.live, Q.cnt);
            // ---- Phase 1 for the next Phase 2 (identical on every replica)
            part::k_reset_all<<<std::min<unsigned>(gridn(n), 148 * 16), 256, 0, s>>>(n, Q.sig, Q.sig + n, Pr);
            launches += 3;
        }
        if (int e = X.allreduce(cnts, 1, 1, s)) return e;
        CKM(cudaMemcpyAsync(hbuf, R[0]->cnt, 4, cudaMemcpyDeviceToHost, s));
        CKM(cudaStreamSynchronize(s));
        const int64_t live = hbuf[0];
        if (live == 0) break;
        if (st && iter - 1 < ECL_SCC_TRACE_MAX) st->edges_in[iter - 1] = live;
        if (st && iter >= 2 && iter - 2 < ECL_SCC_TRACE_MAX) st->edges_kept[iter - 2] = live;   // (after trim)
        // ---- Phase 2: local fixed points + all-reduce(MAX) until no rank changes
        int64_t passes_iter = 0;
        int local_err = 0;
        for (;;) {
            for (int r = 0; r < P; r++) {
                PRank& Q = *R[r];
                int* ring = Q.ring();
                CKM(cudaMemsetAsync(ring, 0, (RING + 1) * 4, s));      // ring words + touched
                int pass = 0, batch = 2;
                for (;;) {
                    for (int k = 0; k < batch; k++, pass++) {
                        part::k_prop_rows<<<gridn(std::max(Q.nloc, 1), 256 * part::PART_RPT), 256, 0, s>>>(
                            Q.nloc, Q.rb, Q.rp, Q.wci, Q.odeg, Q.sig + n, ring, pass, Q.touched());
                        part::k_prop_cols<<<gridn(n, 256 * part::PART_RPT), 256, 0, s>>>(n, Q.cp, Q.cr, Q.ideg, Q.sig,
                                                                                         ring, pass, Q.touched());
                        launches += 2;
                    }
                    CKM(cudaGetLastError());
                    CKM(cudaMemcpyAsync(hbuf, ring + ((pass - 1) & (RING - 1)), 4, cudaMemcpyDeviceToHost, s));
                    CKM(cudaStreamSynchronize(s));
                    if (hbuf[0] == 0) break;
                    if ((int64_t)pass > 4 * (int64_t)n + 1024) {
                        local_err = 1;             // reported through the exchange (all ranks stop)
                        break;
                    }
                    batch = std::min(batch * 2, RING / 2);
                }
                if (r == 0) passes_iter += pass;
                // did this rank change anything? (2: it failed; MAX makes every rank see it)
                k_copy_flag<<<1, 1, 0, s>>>(Q.touched(), Q.sig + 2 * (int64_t)n, local_err ? 2 : 0);
                launches++;
            }
            if (int e = X.allreduce(sigs, 2 * (int64_t)n + 1, 0, s)) return e;
            CKM(cudaMemcpyAsync(hbuf, R[0]->sig + 2 * (int64_t)n, 4, cudaMemcpyDeviceToHost, s));
            CKM(cudaStreamSynchronize(s));
            if (hbuf[0] == 2) return fail(ECL_SCC_ECUDA, "internal: local Phase 2 did not converge on some rank");
            if (hbuf[0] == 0) break;
        }
        iters = iter;
        passes_total += passes_iter;
        if (st && iter - 1 < ECL_SCC_TRACE_MAX) st->passes_iter[iter - 1] = passes_iter;
    }
    // ---- labels: all signatures are final on every replica (rank 0's is used)
    PRank& Q = *R[0];
    const unsigned gr = std::min<unsigned>(gridn(n), 148 * 16);
    part::k_encode_labels<<<gr, 256, 0, s>>>(n, Q.sig, labels, Pr.ids);
    launches++;
    if (!Pr.ids) {
        k_relabel_rep<<<gr, 256, 0, s>>>(n, labels, Q.kdeg, Pr);
        k_relabel_max<<<gr, 256, 0, s>>>(n, labels, Q.kdeg, Pr);
        k_relabel_apply<<<gr, 256, 0, s>>>(n, labels, Q.kdeg);
        launches += 3;
    }
    CKM(cudaGetLastError());
    CKM(cudaStreamSynchronize(s));
    if (st) {
        st->iterations = iters;
        st->trace_len = std::min(iters, ECL_SCC_TRACE_MAX);
        st->passes = passes_total;
        st->kernel_launches = launches;
        st->ms_comm = X.ms();
        st->comm_bytes = X.bytes;
        st->exchanges = X.used;
    }
    return ECL_SCC_OK;
}

}  // namespace eclscc

// =========================================================================== C ABI
using namespace eclscc;

struct ecl_scc_comm_s {
    ncclComm_t comm;
    int nranks, rank, device;
};

// per-rank workspace of the partitioned mode: allocated once, reused by every call
struct ecl_scc_part_plan_s {
    PRank R;
    uint32_t flags = 0;
    std::vector<cudaEvent_t> ev;              // exchange timing events
    ~ecl_scc_part_plan_s() {
        for (cudaEvent_t e : ev) cudaEventDestroy(e);
    }
};

extern "C" {

int ecl_scc_get_unique_id(uint8_t id[128]) {
    clear_err();
    if (!id) return fail(ECL_SCC_EINVAL, "NULL id");
    static_assert(sizeof(ncclUniqueId) == 128, "NCCL unique id size");
    ncclUniqueId u;
    CKN(ncclGetUniqueId(&u));
    memcpy(id, &u, 128);
    return ECL_SCC_OK;
}

int ecl_scc_comm_create(int32_t nranks, int32_t rank, const uint8_t id[128], ecl_scc_comm_t* out) {
    clear_err();
    if (!id || !out || nranks < 1 || rank < 0 || rank >= nranks) return fail(ECL_SCC_EINVAL, "comm_create: bad arguments");
    ncclUniqueId u;
    memcpy(&u, id, 128);
    ecl_scc_comm_s* c = new ecl_scc_comm_s();
    CKM(cudaGetDevice(&c->device));
    ncclResult_t r = ncclCommInitRank(&c->comm, nranks, u, rank);
    if (r != ncclSuccess) {
        delete c;
        return fail(ECL_SCC_ENCCL, "ncclCommInitRank: %s", ncclGetErrorString(r));
    }
    c->nranks = nranks;
    c->rank = rank;
    *out = c;
    return ECL_SCC_OK;
}

int ecl_scc_comm_destroy(ecl_scc_comm_t comm) {
    clear_err();
    if (!comm) return ECL_SCC_OK;
    ncclCommDestroy(comm->comm);
    delete comm;
    return ECL_SCC_OK;
}

int ecl_scc_part_plan_create(int32_t n, int32_t row_begin, int32_t row_end, int64_t local_nnz_max, uint32_t flags,
                             ecl_scc_part_plan_t* out) {
    clear_err();
    if (!out || n < 0 || row_begin < 0 || row_end < row_begin || row_end > n || local_nnz_max < 0)
        return fail(ECL_SCC_EINVAL, "part_plan_create: bad arguments");
    if (local_nnz_max >= (int64_t)INT32_MAX) return fail(ECL_SCC_EUNSUPPORTED, "local nnz >= 2^31");
    auto* h = new (std::nothrow) ecl_scc_part_plan_s();
    if (!h) return fail(ECL_SCC_ENOMEM, "host allocation");
    h->flags = flags;
    h->R.rb = row_begin; h->R.re = row_end; h->R.nloc = row_end - row_begin; h->R.m = local_nnz_max;
    if (int r = rank_alloc(h->R, n)) {
        delete h;
        return r;
    }
    *out = h;
    return ECL_SCC_OK;
}

int ecl_scc_part_plan_destroy(ecl_scc_part_plan_t plan) {
    clear_err();
    delete plan;
    return ECL_SCC_OK;
}

int ecl_scc_partitioned(ecl_scc_comm_t comm, int32_t n, int32_t row_begin, int32_t row_end, int64_t local_nnz,
                        const int32_t* local_row_ptr, const int32_t* local_col_idx, int32_t* labels_out,
                        ecl_scc_stream_t stream, ecl_scc_part_plan_t plan, ecl_scc_stats* stats) {
    clear_err();
    if (!comm || n < 0 || row_begin < 0 || row_end < row_begin || row_end > n || local_nnz < 0)
        return fail(ECL_SCC_EINVAL, "partitioned: bad arguments");
    if (n > 0 && (!labels_out || !local_row_ptr)) return fail(ECL_SCC_EINVAL, "partitioned: NULL pointer");
    if (local_nnz > 0 && !local_col_idx) return fail(ECL_SCC_EINVAL, "partitioned: NULL col_idx");
    if (local_nnz >= (int64_t)INT32_MAX) return fail(ECL_SCC_EUNSUPPORTED, "local nnz >= 2^31");
    if (n == 0) return ECL_SCC_OK;
    ecl_scc_part_plan_t tmp = nullptr;
    if (!plan) {
        if (int r = ecl_scc_part_plan_create(n, row_begin, row_end, local_nnz, 0, &tmp)) return r;
        plan = tmp;
    }
    int rc = ECL_SCC_OK;
    if (plan->R.rb != row_begin || plan->R.re != row_end || plan->R.m < local_nnz || (int64_t)plan->R.nloc < 0)
        rc = fail(ECL_SCC_EINVAL, "partitioned: the plan was made for other rows or fewer edges");
    if (!rc) {
        PRank& Q = plan->R;
        const int64_t cap = Q.m;
        Q.m = local_nnz;
        Q.rp = local_row_ptr;
        Q.ci = local_col_idx;
        std::vector<PRank*> R{&Q};
        NcclExchange X(comm->comm);
        X.ev = &plan->ev;
        rc = run_partitioned(R, X, n, plan->flags, labels_out, (cudaStream_t)stream, stats);
        Q.m = cap;
        Q.rp = Q.ci = nullptr;
    }
    if (tmp) ecl_scc_part_plan_destroy(tmp);
    return rc;
}

int ecl_scc_partitioned_emulated(int32_t P, int32_t n, int64_t nnz, const int32_t* row_ptr, const int32_t* col_idx,
                                 int32_t* labels_out, ecl_scc_stream_t stream, ecl_scc_stats* stats) {
    clear_err();
    if (P < 1 || P > 64 || n < 0 || nnz < 0) return fail(ECL_SCC_EINVAL, "partitioned_emulated: bad arguments");
    if (n > 0 && (!row_ptr || !labels_out)) return fail(ECL_SCC_EINVAL, "partitioned_emulated: NULL pointer");
    if (nnz > 0 && !col_idx) return fail(ECL_SCC_EINVAL, "partitioned_emulated: NULL col_idx");
    if (nnz >= (int64_t)INT32_MAX) return fail(ECL_SCC_EUNSUPPORTED, "nnz >= 2^31");
    if (n == 0) return ECL_SCC_OK;
    cudaStream_t s = (cudaStream_t)stream;
    // row ranges balanced by edge count, from the host copy of row_ptr
    std::vector<int32_t> hrp((size_t)n + 1), bounds((size_t)P + 1);
    CKM(cudaMemcpy(hrp.data(), row_ptr, sizeof(int32_t) * (size_t)(n + 1), cudaMemcpyDeviceToHost));
    if (hrp[0] != 0 || hrp[n] != nnz) return fail(ECL_SCC_ERANGE, "invalid CSR offsets");
    if (int r = ecl_scc_partition_rows(P, n, hrp.data(), bounds.data())) return r;
    // each emulated rank gets its own local CSR (rebased offsets), as a real rank would
    std::vector<std::unique_ptr<PRank>> own;
    std::vector<PRank*> R;
    std::vector<int32_t*> lrps;
    int rc = ECL_SCC_OK;
    for (int r = 0; r < P && rc == ECL_SCC_OK; r++) {
        auto Q = std::make_unique<PRank>();
        Q->rb = bounds[r]; Q->re = bounds[r + 1]; Q->nloc = Q->re - Q->rb;
        Q->m = (int64_t)hrp[Q->re] - hrp[Q->rb];
        std::vector<int32_t> lrp((size_t)Q->nloc + 1);
        for (int i = 0; i <= Q->nloc; i++) lrp[i] = hrp[Q->rb + i] - hrp[Q->rb];
        int32_t* d = nullptr;
        if (cudaMalloc((void**)&d, sizeof(int32_t) * lrp.size()) != cudaSuccess) {
            cudaGetLastError();
            rc = fail(ECL_SCC_ENOMEM, "emulated rank offsets");
            break;
        }
        lrps.push_back(d);
        if (cudaMemcpy(d, lrp.data(), sizeof(int32_t) * lrp.size(), cudaMemcpyHostToDevice) != cudaSuccess) {
            rc = fail(ECL_SCC_ECUDA, "emulated rank offsets copy");
            break;
        }
        Q->rp = d;
        Q->ci = col_idx + hrp[Q->rb];
        rc = rank_alloc(*Q, n);
        R.push_back(Q.get());
        own.push_back(std::move(Q));
    }
    if (rc == ECL_SCC_OK) {
        EmulatedExchange X(P);
        std::vector<cudaEvent_t> ev;
        X.ev = &ev;
        rc = run_partitioned(R, X, n, 0, labels_out, s, stats);
        cudaStreamSynchronize(s);
        for (cudaEvent_t e : ev) cudaEventDestroy(e);
    }
    cudaStreamSynchronize(s);
    own.clear();
    for (int32_t* d : lrps) cudaFree(d);
    return rc;
}

}  // extern "C"

