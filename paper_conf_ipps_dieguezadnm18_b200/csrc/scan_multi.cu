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
//
// Fused exchange (scan_comm_create_peer): instead of the host-launched all-gather, the
// Stage 2 kernel of every rank stores its G totals straight into the mailboxes of the
// ranks after it (one-sided stores over NVLink into peer HBM mapped with CUDA IPC) and
// release-stores a flag; the Stage 3 kernel acquire-spins on its own flags and folds the
// rows.  No collective call, no host involvement after setup (scan_internal.h, PeerParams).
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <unistd.h>

#include <cstdint>
#include <cstring>
#include <mutex>

#include "scan_b200.h"
#include "scan_internal.h"

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

// Mailbox of one rank (in its own HBM, written by peers):
//   [0, 64)     flags[kMaxPeers]  flags[q] = last epoch whose totals rank q pushed here
//   [64, 128)   acks[kMaxPeers]   acks[q]  = last epoch in which rank q read this rank's rows
//   [128, 136)  counters[2]       last-CTA counters of Stage 2 / Stage 3 (local use)
//   [256, ...)  totals[2][ngpu][G_cap] 8-byte slots; half = epoch & 1, row = pushing rank
constexpr size_t kMbFlags = 0, kMbAcks = 64, kMbCounters = 128, kMbTotals = 256;
constexpr uint32_t kPeerMagic = 0x53434e50u;   // "SCNP"
struct PeerHandle {                            // the SCAN_PEER_HANDLE_BYTES blob
    uint32_t magic;
    int32_t device;
    int64_t pid;
    uint64_t dptr;
    uint64_t bytes;
    cudaIpcMemHandle_t ipc;
};
static_assert(sizeof(PeerHandle) <= SCAN_PEER_HANDLE_BYTES, "peer handle blob too small");

struct scan_comm_s {
    enum Backend { NCCL = 0, PEER = 1 } backend = NCCL;
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
    // PEER backend
    char* mailbox = nullptr;       // own mailbox (cudaMalloc, IPC-exported)
    size_t mb_bytes = 0;
    int64_t peer_gcap = 0;         // G capacity of every mailbox (fixed at creation)
    char* peer_base[scanb200::kMaxPeers] = {};   // every rank's mailbox in this address space
    bool peer_ipc[scanb200::kMaxPeers] = {};     // opened with cudaIpcOpenMemHandle
    bool peers_open = false;
    uint64_t epoch = 0;            // calls made on this communicator
};

namespace {
scan_status grow_buffers(scan_comm_s* comm, int64_t N_local, int64_t G, cudaStream_t s, bool all_totals) {
    if (comm->cap_g < G) {
        cudaStreamSynchronize(s);
        if (comm->totals) cudaFree(comm->totals);
        if (comm->all_totals) cudaFree(comm->all_totals);
        comm->totals = comm->all_totals = nullptr;
        if (cudaMalloc(&comm->totals, G * 8) != cudaSuccess ||
            (all_totals && cudaMalloc(&comm->all_totals, (size_t)G * 8 * comm->ngpu) != cudaSuccess)) {
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
    return SCAN_OK;
}
}  // namespace

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

scan_status scan_comm_create_peer(int rank, int ngpu, int64_t max_G, scan_comm_t* out) {
    if (!out || ngpu < 1 || rank < 0 || rank >= ngpu || max_G < 1) return SCAN_ERR_INVALID_ARG;
    if (ngpu > scanb200::kMaxPeers) return SCAN_ERR_UNSUPPORTED;
    if (max_G > (int64_t(1) << 40)) return SCAN_ERR_INVALID_ARG;
    scan_comm_s* c = new scan_comm_s();
    c->backend = scan_comm_s::PEER;
    c->rank = rank;
    c->ngpu = ngpu;
    cudaGetDevice(&c->device);
    c->peer_gcap = max_G;
    c->mb_bytes = kMbTotals + (size_t)2 * ngpu * max_G * 8;
    void* mb = nullptr;
    if (cudaMalloc(&mb, c->mb_bytes) != cudaSuccess) { cudaGetLastError(); delete c; return SCAN_ERR_NO_MEMORY; }
    c->mailbox = (char*)mb;
    if (cudaMemset(mb, 0, c->mb_bytes) != cudaSuccess || cudaDeviceSynchronize() != cudaSuccess) {
        cudaGetLastError(); cudaFree(mb); delete c; return SCAN_ERR_CUDA;
    }
    c->peer_base[rank] = c->mailbox;
    *out = c;
    return SCAN_OK;
}

scan_status scan_comm_peer_handle(scan_comm_t c, void* handle_out) {
    if (!c || !handle_out || c->backend != scan_comm_s::PEER) return SCAN_ERR_INVALID_ARG;
    PeerHandle h;
    std::memset(&h, 0, sizeof(h));
    h.magic = kPeerMagic;
    h.device = c->device;
    h.pid = (int64_t)getpid();
    h.dptr = (uint64_t)(uintptr_t)c->mailbox;
    h.bytes = c->mb_bytes;
    if (cudaIpcGetMemHandle(&h.ipc, c->mailbox) != cudaSuccess) { cudaGetLastError(); return SCAN_ERR_CUDA; }
    std::memset(handle_out, 0, SCAN_PEER_HANDLE_BYTES);
    std::memcpy(handle_out, &h, sizeof(h));
    return SCAN_OK;
}

scan_status scan_comm_peer_open(scan_comm_t c, const void* handles) {
    if (!c || !handles || c->backend != scan_comm_s::PEER || c->peers_open) return SCAN_ERR_INVALID_ARG;
    const char* blob = (const char*)handles;
    for (int q = 0; q < c->ngpu; ++q) {
        PeerHandle h;
        std::memcpy(&h, blob + (size_t)q * SCAN_PEER_HANDLE_BYTES, sizeof(h));
        if (h.magic != kPeerMagic || h.bytes != c->mb_bytes) return SCAN_ERR_INVALID_ARG;   // same ngpu, max_G
        if (q == c->rank) continue;
        if (h.pid == (int64_t)getpid()) {          // same process: the pointer is already valid
            if (h.device != c->device) {
                cudaError_t e = cudaDeviceEnablePeerAccess(h.device, 0);
                if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled) { cudaGetLastError(); return SCAN_ERR_CUDA; }
                cudaGetLastError();
            }
            c->peer_base[q] = (char*)(uintptr_t)h.dptr;
        } else {
            void* p = nullptr;
            if (cudaIpcOpenMemHandle(&p, h.ipc, cudaIpcMemLazyEnablePeerAccess) != cudaSuccess) {
                cudaGetLastError();
                return SCAN_ERR_CUDA;
            }
            c->peer_base[q] = (char*)p;
            c->peer_ipc[q] = true;
        }
    }
    c->peers_open = true;
    return SCAN_OK;
}

scan_status scan_comm_destroy(scan_comm_t c) {
    if (!c) return SCAN_ERR_INVALID_ARG;
    cudaDeviceSynchronize();
    for (int q = 0; q < scanb200::kMaxPeers; ++q)
        if (c->peer_ipc[q]) cudaIpcCloseMemHandle(c->peer_base[q]);
    if (c->mailbox) cudaFree(c->mailbox);
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
    scanb200::NvtxRange nvtx_range("scan_batch_multi");
    if (mode == SCAN_SHARD_PROBLEMS)          // Case 1: each rank scans its own problems
        return scan_batch(in_local, out_local, N_local, G, op, dtype, kind, stream);
    if (mode != SCAN_SHARD_ELEMENTS) return SCAN_ERR_UNSUPPORTED;
    if (!comm || ngpu != comm->ngpu || N_local < 0 || G < 0) return SCAN_ERR_INVALID_ARG;
    if (G == 0) return SCAN_OK;
    cudaStream_t s = (cudaStream_t)stream;
    if (comm->backend == scan_comm_s::PEER) {
        if (!comm->peers_open) return SCAN_ERR_INVALID_ARG;
        if (G > comm->peer_gcap) return SCAN_ERR_INVALID_ARG;
        scan_status st = grow_buffers(comm, N_local, G, s, false);
        if (st != SCAN_OK) return st;
        const uint64_t epoch = ++comm->epoch;
        const size_t half = (size_t)(epoch & 1) * comm->ngpu * comm->peer_gcap;
        scanb200::PeerParams pp{};
        pp.on = true;
        pp.rank = comm->rank;
        pp.ngpu = comm->ngpu;
        pp.epoch = epoch;
        pp.my_flags = (const uint64_t*)(comm->mailbox + kMbFlags);
        pp.my_acks = (const uint64_t*)(comm->mailbox + kMbAcks);
        pp.counters = (uint32_t*)(comm->mailbox + kMbCounters);
        for (int q = 0; q < comm->ngpu; ++q) {
            char* b = comm->peer_base[q];
            pp.push_totals[q] = (uint64_t*)(b + kMbTotals) + half + (size_t)comm->rank * comm->peer_gcap;
            pp.push_flag[q] = (uint64_t*)(b + kMbFlags) + comm->rank;
            pp.push_ack[q] = (uint64_t*)(b + kMbAcks) + comm->rank;
        }
        const uint64_t* rows = (const uint64_t*)(comm->mailbox + kMbTotals) + half;
        st = scanb200::shard_run_peer(in_local, out_local, N_local, G, op, dtype, kind, comm->ws, comm->ws_bytes,
                                      (uint64_t*)comm->totals, rows, comm->peer_gcap, pp, s);
        // argument errors are found before any launch: the call did not happen, so the
        // epoch is not consumed (every rank must see the same sequence of epochs)
        if (st == SCAN_ERR_INVALID_ARG || st == SCAN_ERR_NO_MEMORY) --comm->epoch;
        return st;
    }
    if (!comm->nccl_comm) return SCAN_ERR_INVALID_ARG;
    scan_status gst = grow_buffers(comm, N_local, G, s, true);
    if (gst != SCAN_OK) return gst;
    scan_status st = scan_shard_totals(in_local, N_local, G, op, dtype, comm->totals, comm->ws, comm->ws_bytes, stream);
    if (st != SCAN_OK) return st;
    if (nccl().all_gather(comm->totals, comm->all_totals, (size_t)G, kNcclUint64, comm->nccl_comm, s) != 0)
        return SCAN_ERR_NCCL;
    return scan_shard_scan(in_local, out_local, N_local, G, op, dtype, kind, comm->all_totals, comm->rank,
                           comm->ngpu, comm->ws, comm->ws_bytes, stream);
}

}  // extern "C"
