// scan_multi.cu -- the single-box multi-GPU layer of the C-ABI (include/scan_b200.h).
//
// Case 1 (PAPER.md:191-193 [§4]): problems are spread over the GPUs, each rank scans its
// own problems -- no communication at all (SCAN_SHARD_PROBLEMS).
// Case 2, Multi-GPU Problem Scattering (PAPER.md:195-205 [§4.1, Figs. 6-7]): every problem
// is split into rank-ordered contiguous portions (SCAN_SHARD_ELEMENTS):
//   Stage 1+2 on the local portion   scan_shard_totals  (chunk aggregates + portion totals)
//   exchange                         ncclAllGather of the G portion totals of every rank
//                                    over NVLink/NVSwitch (replaces the paper's P2P writes
//                                    to a master GPU and MPI_Gather/MPI_Scatter, PAPER.md:199,
//                                    207; every rank folds the totals of ranks < r itself, so
//                                    there is no master and no scatter)
//   Stage 3 on the local portion     scan_shard_scan    (carry = ranks < r, then chunks)
// All three steps are stream-ordered on the caller's stream; no host synchronisation.
//
// NCCL is loaded with dlopen at communicator creation (the process normally already has
// torch's libnccl.so.2 mapped), so the library itself loads on machines without NCCL.
#include <cuda_runtime.h>
#include <dlfcn.h>

#include <cstdint>
#include <cstring>
#include <mutex>

#include "scan_b200.h"

namespace {

struct NcclUniqueId { char internal[128]; };
typedef int (*AllGatherFn)(const void*, void*, size_t, int, void*, cudaStream_t);
typedef int (*CommInitRankFn)(void**, int, NcclUniqueId, int);
typedef int (*CommDestroyFn)(void*);
typedef int (*GetUniqueIdFn)(NcclUniqueId*);
constexpr int kNcclUint64 = 5;

struct NcclApi {
    bool ok = false;
    AllGatherFn all_gather = nullptr;
    CommInitRankFn init_rank = nullptr;
    CommDestroyFn destroy = nullptr;
    GetUniqueIdFn unique_id = nullptr;
};

NcclApi& nccl() {
    static NcclApi api;
    static std::once_flag once;
    std::call_once(once, [] {
        void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL | RTLD_NOLOAD);
        if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
        if (!h) return;
        api.all_gather = (AllGatherFn)dlsym(h, "ncclAllGather");
        api.init_rank = (CommInitRankFn)dlsym(h, "ncclCommInitRank");
        api.destroy = (CommDestroyFn)dlsym(h, "ncclCommDestroy");
        api.unique_id = (GetUniqueIdFn)dlsym(h, "ncclGetUniqueId");
        api.ok = api.all_gather && api.init_rank && api.destroy && api.unique_id;
    });
    return api;
}

}  // namespace

struct scan_comm_s {
    void* nccl_comm = nullptr;     // ncclComm_t
    bool owned = false;
    int rank = 0;
    int ngpu = 1;
    int device = 0;
    void* totals = nullptr;        // [G] this rank's portion totals
    void* all_totals = nullptr;    // [ngpu][G]
    int64_t cap_g = 0;
    void* ws = nullptr;            // three-stage workspace (chunk aggregates) kept between steps
    size_t ws_bytes = 0;
};

extern "C" {

scan_status scan_comm_create_nccl(void* nccl_comm, int rank, int ngpu, scan_comm_t* out) {
    if (!nccl_comm || !out || ngpu < 1 || rank < 0 || rank >= ngpu) return SCAN_ERR_INVALID_ARG;
    if (!nccl().ok) return SCAN_ERR_NCCL;
    scan_comm_s* c = new scan_comm_s();
    c->nccl_comm = nccl_comm;
    c->owned = false;
    c->rank = rank;
    c->ngpu = ngpu;
    cudaGetDevice(&c->device);
    *out = c;
    return SCAN_OK;
}

scan_status scan_comm_get_unique_id(void* id_out_128) {
    if (!id_out_128) return SCAN_ERR_INVALID_ARG;
    if (!nccl().ok) return SCAN_ERR_NCCL;
    NcclUniqueId id;
    if (nccl().unique_id(&id) != 0) return SCAN_ERR_NCCL;
    std::memcpy(id_out_128, &id, sizeof(id));
    return SCAN_OK;
}

scan_status scan_comm_init_rank(const void* nccl_unique_id, int rank, int ngpu, scan_comm_t* out) {
    if (!nccl_unique_id || !out || ngpu < 1 || rank < 0 || rank >= ngpu) return SCAN_ERR_INVALID_ARG;
    if (!nccl().ok) return SCAN_ERR_NCCL;
    NcclUniqueId id;
    std::memcpy(&id, nccl_unique_id, sizeof(id));
    void* comm = nullptr;
    if (nccl().init_rank(&comm, ngpu, id, rank) != 0) return SCAN_ERR_NCCL;
    scan_comm_s* c = new scan_comm_s();
    c->nccl_comm = comm;
    c->owned = true;
    c->rank = rank;
    c->ngpu = ngpu;
    cudaGetDevice(&c->device);
    *out = c;
    return SCAN_OK;
}

scan_status scan_comm_destroy(scan_comm_t c) {
    if (!c) return SCAN_ERR_INVALID_ARG;
    cudaDeviceSynchronize();
    if (c->totals) cudaFree(c->totals);
    if (c->all_totals) cudaFree(c->all_totals);
    if (c->ws) cudaFree(c->ws);
    scan_status st = SCAN_OK;
    if (c->owned && c->nccl_comm && nccl().destroy(c->nccl_comm) != 0) st = SCAN_ERR_NCCL;
    delete c;
    return st;
}

scan_status scan_batch_multi(const void* in_local, void* out_local, int64_t N_local, int64_t G, scan_op op,
                             scan_dtype dtype, scan_kind kind, void* stream, int ngpu, scan_comm_t comm,
                             scan_shard mode) {
    if (mode == SCAN_SHARD_PROBLEMS)          // Case 1: each rank scans its own problems
        return scan_batch(in_local, out_local, N_local, G, op, dtype, kind, stream);
    if (mode != SCAN_SHARD_ELEMENTS) return SCAN_ERR_UNSUPPORTED;
    if (!comm || ngpu != comm->ngpu || N_local < 0 || G < 0) return SCAN_ERR_INVALID_ARG;
    if (G == 0) return SCAN_OK;
    cudaStream_t s = (cudaStream_t)stream;
    // buffers owned by the communicator (grown on demand; host-synchronous only then)
    if (comm->cap_g < G) {
        cudaStreamSynchronize(s);
        if (comm->totals) cudaFree(comm->totals);
        if (comm->all_totals) cudaFree(comm->all_totals);
        comm->totals = comm->all_totals = nullptr;
        if (cudaMalloc(&comm->totals, G * 8) != cudaSuccess ||
            cudaMalloc(&comm->all_totals, (size_t)G * 8 * comm->ngpu) != cudaSuccess) {
            cudaGetLastError();
            comm->cap_g = 0;
            return SCAN_ERR_NO_MEMORY;
        }
        comm->cap_g = G;
    }
    const size_t need = scan_shard_workspace_bytes(N_local, G);
    if (comm->ws_bytes < need) {
        cudaStreamSynchronize(s);
        if (comm->ws) cudaFree(comm->ws);
        comm->ws = nullptr;
        if (cudaMalloc(&comm->ws, need) != cudaSuccess) { cudaGetLastError(); comm->ws_bytes = 0; return SCAN_ERR_NO_MEMORY; }
        cudaMemset(comm->ws, 0, need);
        comm->ws_bytes = need;
    }
    scan_status st = scan_shard_totals(in_local, N_local, G, op, dtype, comm->totals, comm->ws, comm->ws_bytes, stream);
    if (st != SCAN_OK) return st;
    if (nccl().all_gather(comm->totals, comm->all_totals, (size_t)G, kNcclUint64, comm->nccl_comm, s) != 0)
        return SCAN_ERR_NCCL;
    return scan_shard_scan(in_local, out_local, N_local, G, op, dtype, kind, comm->all_totals, comm->rank,
                           comm->ngpu, comm->ws, comm->ws_bytes, stream);
}

}  // extern "C"
