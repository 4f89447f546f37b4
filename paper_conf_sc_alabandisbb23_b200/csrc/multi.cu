// multi.cu -- multi-GPU layer: one large graph edge-partitioned by source rows,
// SPMD, one process per GPU.  The algorithm is run_halo (driver.cu, halo.cuh): every rank runs
// the single-GPU machinery on its local graph and the ranks exchange only the signatures of
// the halo (vertices held by more than one rank).
//
// Exchanges (Exchange, driver.h):
//   * NcclExchange -- degree / count / label all-reduces with NCCL; the signature exchange of
//     Phase 2 is FUSED into the propagation kernel (f1): the halo buffer is NCCL symmetric
//     memory (ncclMemAlloc + ncclCommWindowRegister), and k_prop_async pushes every raised
//     halo copy straight into every peer's buffer -- one multimem.red.max through the
//     NVSwitch when the communicator has NVLS multicast (ncclGetLsaMultimemPointer), else
//     remote atomicMax over NVLink peer pointers (ncclGetLsaPointer); a one-word all-reduce
//     is the barrier.  Without the device API (or with ECL_SCC_HALO_ALLREDUCE) the halo
//     buffer is combined by ncclAllReduce(MAX) instead (the baseline).
//   * EmulatedExchange -- P ranks in one process on one device (tests): reductions over the
//     P buffers, pushes into the P buffers of the same device.
#include <cuda.h>
#include <cuda_runtime.h>
#include <nccl.h>
#include <nccl_device.h>
#include <string.h>

#include <algorithm>
#include <memory>
#include <new>
#include <vector>

#include "driver.h"
#include "kernels.cuh"
#include "partition.cuh"

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

struct EmulatedExchange : Exchange {
    int32_t** dptrs = nullptr;
    int P = 0;
    bool fused = true;                    // pushes into the P buffers (else: all-reduce exchange)
    EmulatedExchange(int p, bool f) : P(p), fused(f) {}
    ~EmulatedExchange() { cudaFree(dptrs); }
    int reduce(std::vector<int32_t*>& bufs, int64_t count, int op, cudaStream_t s) override {
        if (P == 1) return ECL_SCC_OK;
        if (!dptrs) CKM(cudaMalloc((void**)&dptrs, sizeof(int32_t*) * P));
        CKM(cudaMemcpyAsync(dptrs, bufs.data(), sizeof(int32_t*) * P, cudaMemcpyHostToDevice, s));
        part::k_reduce_replicas<<<std::min<unsigned>(gridn(count), 148 * 8), 256, 0, s>>>(P, dptrs, count, op);
        CKM(cudaGetLastError());
        return ECL_SCC_OK;
    }
    // every rank pushes into all P buffers (same device: plain atomics)
    int halo_buffers(std::vector<HaloRank*>& R, int64_t entries, cudaStream_t) override {
        for (HaloRank* Q : R) {
            if (!Q->hbuf_external) cudaFree(Q->hbuf);
            Q->hbuf = nullptr;
            Q->hbuf_external = false;
            if (cudaMalloc((void**)&Q->hbuf, sizeof(int32_t) * 2 * (size_t)entries) != cudaSuccess) {
                cudaGetLastError();
                return fail(ECL_SCC_ENOMEM, "halo exchange buffer");
            }
        }
        for (HaloRank* Q : R) {
            Q->push = HaloPush{};
            if (!fused || P > HALO_MAX_PEERS) continue;   // (then: the all-reduce exchange)
            Q->push.np = P;
            for (int k = 0; k < P; k++) Q->push.peer[k] = R[k]->hbuf;
        }
        return ECL_SCC_OK;
    }
};

}  // namespace eclscc

using namespace eclscc;

// one NCCL communicator plus the device-side state of the fused halo exchange
struct ecl_scc_comm_s {
    ncclComm_t comm;
    int nranks, rank, device;
    bool dev_tried = false;
    bool dev_ok = false;                 // ncclDevCommCreate succeeded
    bool multimem = false;               // its LSA team has NVLS multicast
    ncclDevComm dcomm{};
    ncclWindow_t win = nullptr;          // the registered halo buffer
    void* wbuf = nullptr;                // ncclMemAlloc'd halo buffer
    int32_t** dptr = nullptr;            // device scratch: peer / multicast pointers
};

namespace eclscc {

static __global__ void k_lsa_pointers(ncclWindow_t w, int np, int32_t** out) {
    for (int p = 0; p < np; p++) out[p] = (int32_t*)ncclGetLsaPointer(w, 0, p);
}
static __global__ void k_lsa_multimem(ncclWindow_t w, ncclDevComm dc, int32_t** out) {
    out[0] = (int32_t*)ncclGetLsaMultimemPointer(w, 0, dc);
}

struct NcclExchange : Exchange {
    ecl_scc_comm_s* c;
    bool allow_fused;
    NcclExchange(ecl_scc_comm_s* cc, bool fused) : c(cc), allow_fused(fused) {}
    int reduce(std::vector<int32_t*>& bufs, int64_t count, int op, cudaStream_t s) override {
        CKN(ncclAllReduce(bufs[0], bufs[0], (size_t)count, ncclInt32, op == 0 ? ncclMax : ncclSum, c->comm, s));
        return ECL_SCC_OK;
    }
    // collective: the halo buffer in symmetric memory, registered as a window; push targets
    // from the device API (multicast, or every LSA peer); plain memory + all-reduce otherwise
    int halo_buffers(std::vector<HaloRank*>& R, int64_t entries, cudaStream_t s) override {
        HaloRank* Q = R[0];
        const size_t bytes = sizeof(int32_t) * 2 * (size_t)entries;
        if (!Q->hbuf_external) cudaFree(Q->hbuf);
        Q->hbuf = nullptr;
        Q->hbuf_external = false;
        Q->push = HaloPush{};
        if (c->win) {
            ncclCommWindowDeregister(c->comm, c->win);
            c->win = nullptr;
        }
        if (c->wbuf) {
            ncclMemFree(c->wbuf);
            c->wbuf = nullptr;
        }
        bool fused = false;
        if (allow_fused && c->nranks <= HALO_MAX_PEERS) {
            const size_t wb = (bytes + NCCL_WIN_REQUIRED_ALIGNMENT - 1) / NCCL_WIN_REQUIRED_ALIGNMENT *
                              NCCL_WIN_REQUIRED_ALIGNMENT;
            if (ncclMemAlloc(&c->wbuf, wb) == ncclSuccess &&
                ncclCommWindowRegister(c->comm, c->wbuf, wb, &c->win, NCCL_WIN_COLL_SYMMETRIC) == ncclSuccess) {
                if (!c->dev_tried) {
                    c->dev_tried = true;
                    ncclDevCommRequirements req = {};
                    req.lsaMultimem = true;
                    c->multimem = ncclDevCommCreate(c->comm, &req, &c->dcomm) == ncclSuccess;
                    if (!c->multimem) {
                        req.lsaMultimem = false;
                        c->dev_ok = ncclDevCommCreate(c->comm, &req, &c->dcomm) == ncclSuccess;
                    } else {
                        c->dev_ok = true;
                    }
                }
                const ncclTeam_t lsa = ncclTeamLsa(c->comm);
                if (c->dev_ok && lsa.nRanks == c->nranks) {       // every rank reachable by load/store
                    if (!c->dptr) CKM(cudaMalloc((void**)&c->dptr, sizeof(int32_t*) * (HALO_MAX_PEERS + 1)));
                    int32_t* h[HALO_MAX_PEERS + 1] = {};
                    k_lsa_pointers<<<1, 1, 0, s>>>(c->win, c->nranks, c->dptr);
                    if (c->multimem) k_lsa_multimem<<<1, 1, 0, s>>>(c->win, c->dcomm, c->dptr + HALO_MAX_PEERS);
                    CKM(cudaGetLastError());
                    CKM(cudaMemcpyAsync(h, c->dptr, sizeof(h), cudaMemcpyDeviceToHost, s));
                    CKM(cudaStreamSynchronize(s));
                    Q->push.np = c->nranks;
                    for (int k = 0; k < c->nranks; k++) Q->push.peer[k] = h[k];
                    Q->push.mc = c->multimem ? h[HALO_MAX_PEERS] : nullptr;
                    Q->push.sys = 1;
                    Q->hbuf = h[lsa.rank];                    // this rank's own copy (symmetric memory)
                    Q->hbuf_external = true;
                    fused = Q->hbuf != nullptr;
                }
            } else {
                cudaGetLastError();
            }
        }
        if (!fused) {                                   // the baseline: ncclAllReduce(MAX) of the buffer
            Q->push = HaloPush{};
            Q->hbuf_external = false;
            if (cudaMalloc((void**)&Q->hbuf, bytes) != cudaSuccess) {
                cudaGetLastError();
                return fail(ECL_SCC_ENOMEM, "halo exchange buffer");
            }
        }
        return ECL_SCC_OK;
    }
};

}  // namespace eclscc

// P emulated ranks on one device (tests, development): their workspaces and row offsets
struct ecl_scc_emulated_plan_s {
    int P = 0;
    int32_t n = 0;
    int64_t nnz = 0;
    uint32_t flags = 0;
    std::vector<std::unique_ptr<HaloRank>> R;
    std::vector<int32_t*> lrps;               // per rank: rebased row offsets (device)
    std::vector<int64_t> coff;                // per rank: offset of its rows in col_idx
    std::vector<cudaEvent_t> ev;
    ~ecl_scc_emulated_plan_s() {
        R.clear();
        for (int32_t* d : lrps) cudaFree(d);
        for (cudaEvent_t e : ev) cudaEventDestroy(e);
    }
};

// driver-API entry points through the runtime (no link-time dependency on libcuda)
template <typename F>
static F drv(const char* name) {
    void* fn = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint(name, &fn, cudaEnableDefault, &q) != cudaSuccess || q != cudaDriverEntryPointSuccess) {
        cudaGetLastError();
        return nullptr;
    }
    return (F)fn;
}
#define ECL_DRV(name) auto name = drv<decltype(&::name)>(#name)

// per-rank workspace of the partitioned mode: allocated once, reused by every call
struct ecl_scc_part_plan_s {
    HaloRank R;
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
    if (comm->win) ncclCommWindowDeregister(comm->comm, comm->win);
    if (comm->wbuf) ncclMemFree(comm->wbuf);
    if (comm->dev_ok) ncclDevCommDestroy(comm->comm, &comm->dcomm);
    cudaFree(comm->dptr);
    ncclCommDestroy(comm->comm);
    delete comm;
    return ECL_SCC_OK;
}

int ecl_scc_comm_info(ecl_scc_comm_t comm, int32_t info[4]) {
    clear_err();
    if (!comm || !info) return fail(ECL_SCC_EINVAL, "comm_info: bad arguments");
    info[0] = comm->nranks;
    info[1] = comm->rank;
    info[2] = comm->dev_ok ? 1 : 0;
    info[3] = comm->multimem ? 1 : 0;
    return ECL_SCC_OK;
}

// One-device multicast object bound to a buffer; k_halo_push (the partitioned mode's push
// code) reduces into it through the multicast address with multimem.red.max, and the unicast
// view is checked.  Exercises the NVLS path of the fused halo exchange on a single GPU.
int ecl_scc_multimem_probe(int32_t* checked) {
    clear_err();
    if (checked) *checked = 0;
    int dev = 0;
    CKM(cudaGetDevice(&dev));
    CKM(cudaFree(nullptr));                                   // a current context
    ECL_DRV(cuDeviceGetAttribute);
    ECL_DRV(cuMulticastGetGranularity);
    ECL_DRV(cuMulticastCreate);
    ECL_DRV(cuMulticastAddDevice);
    ECL_DRV(cuMemCreate);
    ECL_DRV(cuMulticastBindMem);
    ECL_DRV(cuMemAddressReserve);
    ECL_DRV(cuMemMap);
    ECL_DRV(cuMemSetAccess);
    ECL_DRV(cuMemUnmap);
    ECL_DRV(cuMemAddressFree);
    ECL_DRV(cuMulticastUnbind);
    ECL_DRV(cuMemRelease);
    if (!cuDeviceGetAttribute || !cuMulticastGetGranularity || !cuMulticastCreate || !cuMulticastAddDevice ||
        !cuMemCreate || !cuMulticastBindMem || !cuMemAddressReserve || !cuMemMap || !cuMemSetAccess || !cuMemUnmap ||
        !cuMemAddressFree || !cuMulticastUnbind || !cuMemRelease)
        return fail(ECL_SCC_EUNSUPPORTED, "multimem_probe: driver entry points unavailable");
    int mc_ok = 0;
    if (cuDeviceGetAttribute(&mc_ok, CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, dev) != CUDA_SUCCESS || !mc_ok)
        return fail(ECL_SCC_EUNSUPPORTED, "multimem_probe: the device has no multicast support");
    constexpr int H = 1 << 16;                                // halo entries (2 ints each)
    CUmulticastObjectProp mp = {};
    mp.numDevices = 1;
    mp.handleTypes = CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR;
    size_t gran = 0;
    mp.size = 2 * H * sizeof(int32_t);
    if (cuMulticastGetGranularity(&gran, &mp, CU_MULTICAST_GRANULARITY_RECOMMENDED) != CUDA_SUCCESS)
        return fail(ECL_SCC_EUNSUPPORTED, "multimem_probe: cuMulticastGetGranularity failed");
    const size_t size = (mp.size + gran - 1) / gran * gran;
    mp.size = size;
    CUmemGenericAllocationHandle mc = 0, mem = 0;
    CUdeviceptr uc_ptr = 0, mc_ptr = 0;
    int rc = ECL_SCC_OK;
    CUmemAllocationProp ap = {};
    ap.type = CU_MEM_ALLOCATION_TYPE_PINNED;
    ap.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
    ap.location.id = dev;
    ap.requestedHandleTypes = CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR;
    CUmemAccessDesc acc = {};
    acc.location = ap.location;
    acc.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
    int32_t *hpos = nullptr, *cin = nullptr, *cout = nullptr;
    std::vector<int32_t> h(2 * (size_t)H);
    {
        int step = 0;
        CUresult cr = CUDA_SUCCESS;
        auto ok = [&](CUresult r) { step++; cr = r; return r == CUDA_SUCCESS; };
        // the exportable handle type a multicast object accepts depends on the platform: try
        // none, a POSIX file descriptor, then a fabric handle
        const CUmemAllocationHandleType types[3] = {CU_MEM_HANDLE_TYPE_NONE, CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR,
                                                    CU_MEM_HANDLE_TYPE_FABRIC};
        for (int k = 0; k < 3 && mc == 0; k++) {
            mp.handleTypes = types[k];
            ap.requestedHandleTypes = types[k];
            if (cuMulticastCreate(&mc, &mp) != CUDA_SUCCESS) mc = 0;
        }
        if (!(ok(mc ? CUDA_SUCCESS : CUDA_ERROR_NOT_SUPPORTED) && ok(cuMulticastAddDevice(mc, dev)) && ok(cuMemCreate(&mem, size, &ap, 0)) &&
              ok(cuMulticastBindMem(mc, 0, mem, 0, size, 0)) && ok(cuMemAddressReserve(&uc_ptr, size, gran, 0, 0)) &&
              ok(cuMemMap(uc_ptr, size, 0, mem, 0)) && ok(cuMemSetAccess(uc_ptr, size, &acc, 1)) &&
              ok(cuMemAddressReserve(&mc_ptr, size, gran, 0, 0)) && ok(cuMemMap(mc_ptr, size, 0, mc, 0)) &&
              ok(cuMemSetAccess(mc_ptr, size, &acc, 1))))
            rc = fail(ECL_SCC_EUNSUPPORTED, "multimem_probe: multicast setup step %d failed (CUresult %d; size %zu, granularity %zu)",
                      step, (int)cr, size, gran);
    }
    if (!rc && (cudaMalloc((void**)&hpos, H * 4) != cudaSuccess || cudaMalloc((void**)&cin, H * 4) != cudaSuccess ||
                cudaMalloc((void**)&cout, H * 4) != cudaSuccess))
        rc = fail(ECL_SCC_ENOMEM, "multimem_probe: buffers");
    if (!rc) {
        // entry p receives max(in) = 3p + 1 over two pushes (3p, then 3p + 1) and out = 5p + 2
        std::vector<int32_t> hp(H), a(H), b(H);
        for (int p = 0; p < H; p++) hp[p] = H - 1 - p;       // local vertex i -> halo position H-1-i
        cudaMemcpy(hpos, hp.data(), H * 4, cudaMemcpyHostToDevice);
        cudaMemset((void*)uc_ptr, 0, size);
        HaloPush P{};
        P.hpos = hpos;
        P.mc = (int32_t*)mc_ptr;
        P.sys = 1;
        for (int round = 0; round < 2 && !rc; round++) {
            for (int i = 0; i < H; i++) {
                const int p = hp[i];
                a[i] = round ? 3 * p + 1 : 3 * p;
                b[i] = round ? 5 * p : 5 * p + 2;
            }
            cudaMemcpy(cin, a.data(), H * 4, cudaMemcpyHostToDevice);
            cudaMemcpy(cout, b.data(), H * 4, cudaMemcpyHostToDevice);
            k_halo_push<<<(H + 255) / 256, 256>>>(H, cin, cout, P);
            if (cudaDeviceSynchronize() != cudaSuccess) rc = fail(ECL_SCC_ECUDA, "multimem_probe: push kernel failed");
        }
        if (!rc) {
            cudaMemcpy(h.data(), (void*)uc_ptr, 2 * (size_t)H * 4, cudaMemcpyDeviceToHost);
            for (int p = 0; p < H && !rc; p++)
                if (h[2 * (size_t)p] != 3 * p + 1 || h[2 * (size_t)p + 1] != 5 * p + 2)
                    rc = fail(ECL_SCC_ECUDA, "multimem_probe: entry %d holds (%d, %d), expected (%d, %d)", p,
                              h[2 * (size_t)p], h[2 * (size_t)p + 1], 3 * p + 1, 5 * p + 2);
            if (!rc && checked) *checked = H;
        }
    }
    cudaFree(hpos); cudaFree(cin); cudaFree(cout);
    if (mc_ptr) { cuMemUnmap(mc_ptr, size); cuMemAddressFree(mc_ptr, size); }
    if (uc_ptr) { cuMemUnmap(uc_ptr, size); cuMemAddressFree(uc_ptr, size); }
    if (mc) { cuMulticastUnbind(mc, dev, 0, size); cuMemRelease(mc); }
    if (mem) cuMemRelease(mem);
    cudaGetLastError();
    return rc;
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
    if (int r = halo_rank_alloc(&h->R, n, row_begin, row_end, local_nnz_max, flags)) {
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
    HaloRank& Q = plan->R;
    if (Q.n != n || Q.rb != row_begin || Q.re != row_end || Q.m_cap < local_nnz)
        rc = fail(ECL_SCC_EINVAL, "partitioned: the plan was made for another graph, other rows or fewer edges");
    if (!rc) {
        Q.m = local_nnz;
        Q.rp = local_row_ptr;
        Q.ci = local_col_idx;
        std::vector<HaloRank*> R{&Q};
        NcclExchange X(comm, !(plan->flags & ECL_SCC_HALO_ALLREDUCE));
        X.ev = &plan->ev;
        rc = run_halo(R, X, n, plan->flags, labels_out, (cudaStream_t)stream, stats);
        Q.rp = Q.ci = nullptr;
    }
    if (tmp) ecl_scc_part_plan_destroy(tmp);
    return rc;
}

int ecl_scc_emulated_plan_destroy(ecl_scc_emulated_plan_t plan) {
    clear_err();
    delete plan;
    return ECL_SCC_OK;
}

int ecl_scc_emulated_plan_create(int32_t P, int32_t n, int64_t nnz, const int32_t* row_ptr, uint32_t flags,
                                 ecl_scc_emulated_plan_t* out) {
    clear_err();
    if (!out || P < 1 || P > 64 || n < 1 || nnz < 0 || !row_ptr) return fail(ECL_SCC_EINVAL, "emulated_plan_create: bad arguments");
    if (nnz >= (int64_t)INT32_MAX) return fail(ECL_SCC_EUNSUPPORTED, "nnz >= 2^31");
    // row ranges balanced by edge count, from the host copy of row_ptr
    std::vector<int32_t> hrp((size_t)n + 1), bounds((size_t)P + 1);
    CKM(cudaMemcpy(hrp.data(), row_ptr, sizeof(int32_t) * (size_t)(n + 1), cudaMemcpyDeviceToHost));
    if (hrp[0] != 0 || hrp[n] != nnz) return fail(ECL_SCC_ERANGE, "invalid CSR offsets");
    if (int r = ecl_scc_partition_rows(P, n, hrp.data(), bounds.data())) return r;
    auto* h = new (std::nothrow) ecl_scc_emulated_plan_s();
    if (!h) return fail(ECL_SCC_ENOMEM, "host allocation");
    h->P = P; h->n = n; h->nnz = nnz; h->flags = flags;
    // each emulated rank gets its own local CSR (rebased offsets), as a real rank would
    for (int r = 0; r < P; r++) {
        auto Q = std::make_unique<HaloRank>();
        const int32_t rb = bounds[r], re = bounds[r + 1];
        const int64_t m = (int64_t)hrp[re] - hrp[rb];
        std::vector<int32_t> lrp((size_t)(re - rb) + 1);
        for (int i = 0; i <= re - rb; i++) lrp[i] = hrp[rb + i] - hrp[rb];
        int32_t* d = nullptr;
        int rc = ECL_SCC_OK;
        if (cudaMalloc((void**)&d, sizeof(int32_t) * lrp.size()) != cudaSuccess) {
            cudaGetLastError();
            rc = fail(ECL_SCC_ENOMEM, "emulated rank offsets");
        } else {
            h->lrps.push_back(d);
            if (cudaMemcpy(d, lrp.data(), sizeof(int32_t) * lrp.size(), cudaMemcpyHostToDevice) != cudaSuccess)
                rc = fail(ECL_SCC_ECUDA, "emulated rank offsets copy");
        }
        if (!rc) rc = halo_rank_alloc(Q.get(), n, rb, re, m, flags);
        if (rc) {
            delete h;
            return rc;
        }
        Q->m = m;
        Q->rp = d;
        h->coff.push_back(hrp[rb]);
        h->R.push_back(std::move(Q));
    }
    *out = h;
    return ECL_SCC_OK;
}

int ecl_scc_partitioned_emulated(int32_t P, int32_t n, int64_t nnz, const int32_t* row_ptr, const int32_t* col_idx,
                                 int32_t* labels_out, uint32_t flags, ecl_scc_stream_t stream,
                                 ecl_scc_emulated_plan_t plan, ecl_scc_stats* stats) {
    clear_err();
    if (P < 1 || P > 64 || n < 0 || nnz < 0) return fail(ECL_SCC_EINVAL, "partitioned_emulated: bad arguments");
    if (n > 0 && (!row_ptr || !labels_out)) return fail(ECL_SCC_EINVAL, "partitioned_emulated: NULL pointer");
    if (nnz > 0 && !col_idx) return fail(ECL_SCC_EINVAL, "partitioned_emulated: NULL col_idx");
    if (nnz >= (int64_t)INT32_MAX) return fail(ECL_SCC_EUNSUPPORTED, "nnz >= 2^31");
    if (n == 0) return ECL_SCC_OK;
    cudaStream_t s = (cudaStream_t)stream;
    ecl_scc_emulated_plan_t tmp = nullptr;
    if (!plan) {
        if (int r = ecl_scc_emulated_plan_create(P, n, nnz, row_ptr, flags, &tmp)) return r;
        plan = tmp;
    }
    int rc = ECL_SCC_OK;
    if (plan->P != P || plan->n != n || plan->nnz != nnz || plan->flags != flags)
        rc = fail(ECL_SCC_EINVAL, "partitioned_emulated: the plan was made for another graph, P or flags");
    if (!rc) {
        std::vector<HaloRank*> R;
        for (int r = 0; r < P; r++) {
            plan->R[r]->ci = col_idx + plan->coff[r];
            R.push_back(plan->R[r].get());
        }
        EmulatedExchange X(P, !(flags & ECL_SCC_HALO_ALLREDUCE));
        X.ev = &plan->ev;
        rc = run_halo(R, X, n, flags, labels_out, s, stats);
    }
    cudaStreamSynchronize(s);
    if (tmp) ecl_scc_emulated_plan_destroy(tmp);
    return rc;
}

}  // extern "C"
