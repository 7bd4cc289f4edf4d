// scan_internal.h -- host-side interface between the C-ABI (scan_api.cu) and the kernels.
// Not installed, not part of the public boundary (include/scan_b200.h is).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

#include "scan_b200.h"

#include <nvtx3/nvToolsExt.h>

namespace scanb200 {

// NVTX range around a library call or phase (visible in Nsight Systems / Compute; a
// no-op costing a few ns when no tool is attached).  Names mirror the paper's phases.
struct NvtxRange {
    explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
    ~NvtxRange() { nvtxRangePop(); }
    NvtxRange(const NvtxRange&) = delete;
    NvtxRange& operator=(const NvtxRange&) = delete;
};

// ---------------------------------------------------------------- launch facts (scan_launch.cu)
// SM count of the current device, and per (device, kernel): the dynamic shared memory /
// non-portable cluster opt-ins plus the occupancy -- cached per device, thread-safe.
cudaError_t current_device_sms(int* sms);
cudaError_t kernel_prepare(const void* func, int threads, size_t dyn_smem, bool nonportable_cluster, int* occ);
// Persistent grid of min(occupancy x SMs, tiles) CTAs launched COOPERATIVELY (the whole
// grid co-resident, as the static round-robin tile schedules require), optionally as a
// programmatic dependent of the stream's previous kernel.
cudaError_t launch_persistent(const void* func, void** args, int64_t tiles, int threads, size_t dyn_smem,
                              bool pdl, cudaStream_t s);

enum class OpCode : int { AddU32 = 0, MaxI32 = 1, MaxU32 = 2, MaxF32 = 3, AddF32 = 4 };

// ---------------------------------------------------------------- single-pass look-back
struct LookbackParams {
    const void* in;
    void* out;
    int64_t N;          // elements per problem (> 0)
    int64_t total;      // G * N
    uint32_t* ctl;      // [0] (unused, kept 0), [1] CTAs that read this launch's tag,
                        // [2] epoch   (zero-initialised once)
    uint64_t* desc;     // descriptors: value<<32|tag<<2|status (two such words per tile for fp64)
    int64_t capacity;   // 16-byte descriptor slots of the workspace (>= tiles of any call)
    uint64_t* trace;    // debug: 4 %globaltimer stamps per tile (NULL in normal use)
    int64_t trace_tiles;
    bool vec;           // in and out are 16-byte aligned
    bool exclusive;
    bool pdl_first;     // cross-call programmatic launch (L2-staged kernel): CTAs may be
                        // scheduled while the stream's previous kernel drains and execute
                        // griddepcontrol.wait before their first global memory access
    int lb_mode;        // L2-staged kernel: 0 = round-1 speculative serialized look-back
                        // (A/B only), otherwise the lazy round-robin look-back
    bool keep_last;     // L2-staged kernel: each CTA's last tile is scanned from the read-1
                        // ring slot (no second read on the kernel's critical tail)
    uint32_t poll_ns;   // first back-off of a failed look-back poll (look_back_par / _rr)
    bool early_read2;   // L2-staged kernel: read 2 at the tile's aggregate, not its carry
};
// u64 words per look-back descriptor slot.  A descriptor needs 1 (32-bit carries) or 2
// (fp64 carries) words; one descriptor per 64-byte slot puts only two tiles on a 128-byte
// L2 line, i.e. few concurrent publishers and pollers per line.  Measured on one 2^30
// problem: packed 8-byte descriptors ~80 % of copy, 16-byte slots ~90 %, 32/64-byte ~99 %
// (the look-back round trip under full HBM load was dominated by line contention).
constexpr int kDescWords = 8;
int64_t lookback_tile_elems(int variant);      // 0 for an unknown variant
bool lookback_variant_valid(int variant);
cudaError_t launch_lookback(OpCode op, const LookbackParams& p, int variant, cudaStream_t s);

// ---------------------------------------------------------------- fused peer exchange
// The exchange step of the sharded path done by the kernels themselves over peer memory
// (Stage 1 results of every GPU reach the GPUs that need them; here by
// one-sided NVLink stores instead of P2P copies to a master GPU).  Every rank owns a
// mailbox in its own HBM (layout in scan_multi.cu); peers write into it, it only reads it.
//   Stage 2 (aux_scan)  waits until every rank p > rank acknowledged call epoch-2 (the
//                       mailbox parity it is about to overwrite), stores its G portion
//                       totals into row `rank` of every peer p > rank, and the last CTA
//                       release-stores `epoch` into flag[rank] of those peers.
//   Stage 3 (chunk_scan) acquire-spins on its own flags of ranks < rank, folds their rows
//                       into the carry, and the last CTA release-stores `epoch` into
//                       ack[rank] of every peer p < rank.
constexpr int kMaxPeers = 8;
struct PeerParams {
    uint64_t* push_totals[kMaxPeers];   // peer p's mailbox row `rank` of this call's parity
    uint64_t* push_flag[kMaxPeers];     // &flags[rank] in peer p's mailbox
    uint64_t* push_ack[kMaxPeers];      // &acks[rank] in peer p's mailbox
    const uint64_t* my_flags;           // own mailbox flags[kMaxPeers] (written by ranks < rank)
    const uint64_t* my_acks;            // own mailbox acks[kMaxPeers]  (written by ranks > rank)
    uint32_t* counters;                 // own mailbox: [0] Stage 2, [1] Stage 3 CTAs done
    uint64_t epoch;                     // this call's number (>= 1), identical on every rank
    int rank, ngpu;
    bool on;
};

// ---------------------------------------------------------------- cascade / three-stage
// Chunked per-problem kernels.  Problem g is cut into Bx chunks of `chunk` elements
// (chunk = K * tile, the paper's cascade depth K).
struct ChunkParams {
    const void* in;
    void* out;
    int64_t N;              // elements per problem (local shard length in sharded mode)
    int64_t G;
    int64_t chunk;          // elements per chunk (multiple of the tile)
    int64_t Bx;             // chunks per problem
    uint64_t* aux;          // [G][Bx] 8-byte slots: chunk reductions, then exclusive prefixes
    uint64_t* totals;       // [G] problem totals (Stage 2 output)
    const uint64_t* carry_src;  // [carry_rows][G] slots folded into every problem's carry
    int carry_rows;
    int64_t carry_stride;   // elements between carry rows (0 means G)
    bool vec;
    bool exclusive;
    bool aux_raw;           // aux holds the RAW chunk reductions (Stage 2 skipped): every
                            // Stage 3 CTA folds those of the chunks before it itself
    bool pdl_first;         // cross-call programmatic launch: the kernel may start while the
                            // stream's previous kernel (any kernel) finishes, and waits for it
                            // (griddepcontrol.wait) before its FIRST memory access
    bool pdl;               // launch as a programmatic dependent of the previous kernel of
                            // this library call (Stage 2 after Stage 1, Stage 3 after Stage 2)
    PeerParams peer;        // fused exchange (peer.on) -- sharded path only
    int64_t pf_ctas;        // Stage 1 with pdl_first: CTAs below this index (the first wave,
                            // the ones that can start while the previous kernel drains)
                            // L2-prefetch their first tiles before griddepcontrol.wait
};
int64_t chunk_tile_elems();
int64_t warp_tile_elems();
// Stage 1: aux[g][c] = reduction of chunk c of problem g
cudaError_t launch_chunk_reduce(OpCode op, const ChunkParams& p, cudaStream_t s);
// Stage 2: exclusive scan of aux[g][*] in place, totals[g] = full reduction (L_y > 1
// problems per block)
cudaError_t launch_aux_scan(OpCode op, const ChunkParams& p, cudaStream_t s);
// Stage 3: scan of every chunk + carry (carry_src rows, then aux prefix when aux != null).
// With Bx == 1 and aux == null this is the CTA-per-problem cascade.
cudaError_t launch_chunk_scan(OpCode op, const ChunkParams& p, cudaStream_t s);
// Warp-per-problem cascade (L_y = warps per block problems per CTA).
cudaError_t launch_warp_cascade(OpCode op, const ChunkParams& p, cudaStream_t s);
// sharded path with short portions (Bx == 1): Stage 1 / Stage 3 with one warp per problem
cudaError_t launch_warp_reduce(OpCode op, const ChunkParams& p, cudaStream_t s);
cudaError_t launch_warp_shard_scan(OpCode op, const ChunkParams& p, cudaStream_t s);
// Packed short problems: p.chunk = k whole problems per warp span (k*N % 4 == 0 when
// p.vec), segmented scan, no carry between spans (L_x < 32).
cudaError_t launch_packed_warp(OpCode op, const ChunkParams& p, cudaStream_t s);
// Cluster per problem (scan_cluster.cu): G clusters of csize CTAs (power of two <= 16);
// the CTAs of one problem exchange their tile aggregates through distributed shared
// memory (one cluster barrier per round of csize tiles).  variant 0/1/2 = 8192/4096/16384-
// element tiles.
constexpr int kMaxClusterCtas = 16;
int64_t cluster_tile_elems(int variant);
cudaError_t launch_cluster_scan(OpCode op, const ChunkParams& p, int variant, int csize, cudaStream_t s);
// ---------------------------------------------------------------- fused three stages
// scan_fused.cu: Stage 1 -> grid barrier -> Stage 2 fold -> Stage 3 in ONE cooperative
// launch, one 8192-element tile per CTA held in registers (latency-bound totals).
struct FusedParams {
    const void* in;
    void* out;
    int64_t total;              // G * N
    int64_t tiles_per_problem;  // N / tile when N is a multiple of the tile, else (G == 1) all tiles
    uint64_t* aux;              // [tiles] 8-byte aggregate slots
    bool vec;
    bool exclusive;
    bool pdl_first;
};
int64_t fused_tile_elems();
int64_t fused_max_tiles(OpCode op);  // co-resident CTAs on the current device (0 on error)
cudaError_t launch_fused(OpCode op, const FusedParams& p, cudaStream_t s);

// Fused exchange with an empty local portion (no Stage 3 CTAs): one CTA waits for the
// flags of ranks < rank and acknowledges them, so peers never wait on this rank.
cudaError_t launch_peer_ack(const PeerParams& pp, cudaStream_t s);

// Host side of the fused exchange (scan_api.cu): Stage 1+2 with the push, Stage 3 with
// the wait and the acknowledgement, on one stream.  `ws` must be sized by
// three_stage_bytes(N_local, G, 0) (scan_shard_workspace_bytes).
scan_status shard_run_peer(const void* in, void* out, int64_t N_local, int64_t G, scan_op op, scan_dtype dt,
                           scan_kind kind, void* ws, size_t ws_bytes, uint64_t* totals,
                           const uint64_t* mailbox_rows, int64_t row_stride, const PeerParams& peer,
                           cudaStream_t s);

}  // namespace scanb200
