// scan_api.cu -- the C-ABI of libscanb200.so (declared in include/scan_b200.h):
// argument checks, workspace management, kernel selection, the host-buffer pipeline and
// the sharded-mode steps.  Every computation is a launch of this library's kernels.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <map>
#include <tuple>
#include <mutex>
#include <utility>
#include <vector>

#include "scan_b200.h"
#include "scan_internal.h"

using namespace scanb200;

namespace {

constexpr size_t kCtlBytes = 256;          // [0] ticket [1] done [2] epoch (look-back)
constexpr int kTargetCtas = 148 * 8;       // chunk count target of the three-stage path
constexpr int64_t kMaxChunkTiles = 16;     // longest three-stage chunk (tiles of 4096)
constexpr int64_t kFuse2MaxChunks = 256;   // Stage 2 folded into Stage 3 up to this many chunks

size_t align_up(size_t v, size_t a) { return (v + a - 1) / a * a; }

bool valid_enums(scan_op op, scan_dtype dt, scan_kind kind) {
    return (op == SCAN_OP_ADD || op == SCAN_OP_MAX) &&
           (dt == SCAN_I32 || dt == SCAN_U32 || dt == SCAN_F32) &&
           (kind == SCAN_INCLUSIVE || kind == SCAN_EXCLUSIVE);
}

OpCode opcode(scan_op op, scan_dtype dt) {
    if (op == SCAN_OP_ADD) return dt == SCAN_F32 ? OpCode::AddF32 : OpCode::AddU32;
    if (dt == SCAN_I32) return OpCode::MaxI32;
    if (dt == SCAN_U32) return OpCode::MaxU32;
    return OpCode::MaxF32;
}

bool split_desc(scan_op op, scan_dtype dt) { return op == SCAN_OP_ADD && dt == SCAN_F32; }

// ---------------------------------------------------------------- dispatch
// The analogue of the paper's empirical K search: the regions below come
// from on-box sweeps recorded in profiles/ (bench.py --sweep, tools/*_probe.py, and the
// scan_autotune grid r01_autotune_probe.jsonl); scan_autotune overrides them per shape.
//   many problems of moderate N (rows 16-byte aligned): the paper's own batch mapping wins
//     on B200 -- one CTA per problem (cascade, L_y = 1) for N > 4096, one warp per problem
//     (L_y = 8) for 768 <= N <= 4096: no inter-CTA traffic at all, ~6.3-6.8 TB/s measured;
//   few short / medium problems (latency bound): one CTA per problem (G <= 148, N <= 8192),
//     one thread-block cluster per problem (N <= 2^15), then the paper's
//     three-stage form (G <= 64, G*N <= 2^23; two launches while <= 256 chunks);
//   a few hundred to a few thousand problems up to 2^16: CTA / warp per problem again
//     (1.1-4.8x over the flat look-back);
//   short rows (N < 1024, 16-byte aligned base pointers, large totals): several whole
//     problems per warp (packed_warp; power-of-two N <= 512 at ~104 % of copy);
//   everything else (few large problems, unaligned pointers): single-pass look-back
//     (L2-staged variant for G*N >= 2^22, one-tile-per-CTA for short unaligned rows).
//   (boundary re-measured with 64-byte descriptor slots, profiles/r01_boundary.txt: the
//    look-back matches or beats the CTA cascade up to G = 2048 for N >= 2^17; the cascade
//    wins from G = 4096, where every SM holds many whole problems)
// `aligned` = both base pointers 16-byte aligned.
scan_algo choose_algo(int64_t N, int64_t G, bool aligned) {
    const bool rows_aligned = aligned && (N % 4 == 0);
    // (N = 4096 exactly: one warp per problem 102 % vs one CTA 93 % of copy at G = 2^16,
    //  tools/n12_probe.py)
    if (rows_aligned && G >= 4096 && N > 4096) return SCAN_ALGO_CASCADE_CTA;
    // hundreds to thousands of problems just above 2^16 elements, and a few thousand up to
    // ~2^18: one CTA per problem beats the flat look-back there, by 3-44 % where problem
    // starts fall inside look-back tiles (N not a multiple of 8192: every problem's first
    // tile needs its own look-back, the CTAs fall out of step and the round-robin
    // look-backs re-poll), ~equal on tile-aligned N (tools/cascade_boundary_probe.py,
    // profiles/r02_cascade_boundary.jsonl, re-measured after the segmented-scan fix); from
    // 2^18 on at G < 2400 the look-back wins; elsewhere the two are within ~3 %
    if (rows_aligned && N > 65536 &&
        ((G >= 300 && N <= 81920) || (G >= 1024 && N <= 131072) ||
         (G >= 2048 && (G >= 2400 || N < 262144))))
        return SCAN_ALGO_CASCADE_CTA;
    if (rows_aligned && G >= 1184 && N >= 768 && N <= 4096) return SCAN_ALGO_CASCADE_WARP;
    // few short / medium problems (latency bound, tools/cluster_probe.py on B200,
    // profiles/r01_cluster_probe.jsonl): one CTA per problem up to 8192 elements
    // (~2.5-3.3 us per call against 5-12 us for three-stage / look-back), one thread-block
    // cluster per problem (DSMEM aggregates) up to 2^15: ~3.3-3.9 us
    if (G <= 148 && N <= 8192) return SCAN_ALGO_CASCADE_CTA;
    // ... and for 64 < G <= 148 up to ~20K elements (G = 80-140, N = 9220-16388: 0.18-0.33 of
    // copy against 0.10-0.21 for the look-back; profiles/r02_mid_batch_dispatch.jsonl)
    if (rows_aligned && G > 64 && G <= 148 && N > 8192 && N < 20480) return SCAN_ALGO_CASCADE_CTA;
    // G just under the SM count: one CTA per problem is one full wave (G = 148, N = 20484-32772:
    // 0.53-0.62 of copy against 0.42-0.53 three-stage; G = 140: a tie)
    if (rows_aligned && G > 140 && G <= 148 && N > 8192 && N < 36864) return SCAN_ALGO_CASCADE_CTA;
    // (2^15 < N <= 2^16 at G = 1: the two-launch chain 3.6 us vs the cluster 3.9-4.0 us once
    //  both use programmatic launch, profiles/r01_g1_probe_cluster_boundary.jsonl)
    if (G <= 64 && N <= 32768) return SCAN_ALGO_CLUSTER;
    // one problem of 2.5 M .. ~4.8 M elements (as many 8192-element tiles as CTAs fit at once):
    // the three stages fused into one cooperative launch with every tile held in registers
    // across one grid barrier -- one read instead of two, one launch instead of two or three
    // (4.7 M: 8.6 vs 13.3 us three-stage, 11.7 us look-back; 2^22: 8.4 vs 9.5 us;
    // profiles/r02_fused_probe.jsonl); below 2.5 M the two-launch chain is faster
    if (G == 1 && N > (int64_t(5) << 19) && N <= fused_max_tiles(OpCode::AddF32) * fused_tile_elems())
        return SCAN_ALGO_FUSED;
    // three-stage up to 2^22 elements (two launches: the second read of the input still
    // hits L2); above, the three-launch form loses to the lazy look-back (5 x 2^20: 12.3 /
    // 13.2 us against 12.5 / 12.5 us i32 / f32; 7 x 2^20: 15.5 against 14.2 / 15.0 us;
    // profiles/r02_fused_probe_tpc2_REVERTED.jsonl)
    if (G <= 64 && N * G <= (int64_t(1) << 22) && N >= 4096) return SCAN_ALGO_THREE_STAGE;
    // tens to a few hundred problems of up to ~80K elements, 2^22 < G*N <= 2^24, problem
    // starts inside look-back tiles: the latency-bound middle, where the three-stage form
    // (its second read still hits L2) beats both the look-back and one CTA per problem
    // (G = 100, N = 65540: 0.59 vs 0.53 / 0.43 of copy; G = 160, N = 32772: 0.54 vs 0.43 /
    // 0.44).  Tile-aligned or longer rows stay on the look-back since its session-3 changes
    // (G = 200, N = 65536: 0.83 vs 0.71; tools/shape_probe.py, profiles/r02_mid_batch_shapes.jsonl)
    if (rows_aligned && G > 64 && G < 300 && N >= 4096 && N <= 81920 && N % 8192 != 0 &&
        N * G > (int64_t(1) << 22) && N * G <= (int64_t(1) << 24))
        return SCAN_ALGO_THREE_STAGE;
    // the same below 2^22 elements for 64 < G <= 148, tile-aligned or not (G = 70 / 100 / 128,
    // N = 20484-40964: 0.25-0.47 of copy against 0.18-0.42 for the look-back; 100 x 32768:
    // 0.50 vs 0.36; profiles/r02_mid_batch_dispatch.jsonl)
    if (rows_aligned && G > 64 && G <= 148 && N >= 20480 && N * G <= (int64_t(1) << 22))
        return SCAN_ALGO_THREE_STAGE;
    // tile-aligned rows of 40960-65536 elements, 148 < G <= 600: the look-back (every problem
    // starts on a tile) beats one CTA per problem (G = 200, N = 65536: 0.81 vs 0.63; G = 500:
    // 0.92 vs 0.79); from G = 800 the cascade wins again (profiles/r02_mid_batch_dispatch.jsonl)
    if (rows_aligned && G > 148 && G <= 600 && N >= 40960 && N <= 65536 && N % 8192 == 0)
        return SCAN_ALGO_LOOKBACK;
    // a few hundred to a few thousand problems of moderate length (scan_autotune over a
    // G x N grid, profiles/r01_autotune_probe.jsonl): whole problems per warp / per CTA
    // beat the flat look-back 1.1-4.8x there (e.g. G = 1024, N = 4096: 5.9 us vs 28 us)
    if (G > 148 && N <= 1024 && N * G <= (int64_t(1) << 20)) return SCAN_ALGO_CASCADE_WARP;
    if (G > 148 && N > 1024 && N <= 65536) return SCAN_ALGO_CASCADE_CTA;
    // short rows: several whole problems per warp (power-of-two N <= 512 flag-free)
    if (aligned && N < 1024) return SCAN_ALGO_PACKED_WARP;
    return SCAN_ALGO_LOOKBACK;
}
int choose_lookback_variant(int64_t N, int64_t G) {
    const int64_t total = N * G;
    if (N < 1024 && G > 1) return 2;
    return total >= (int64_t(1) << 22) ? 3 : 1;
}

// cluster family: param = 32 * variant + csize (csize a power of two <= 16), < 0 = auto:
// 4096-element tiles (variant 1), the smallest cluster that covers the problem in one
// round (<= 16) -- the measured best for 2^13 < N <= 2^16 at G = 1..16
void cluster_config(int64_t N, int64_t param, int* variant, int* csize) {
    if (param >= 0) {
        *variant = (int)((param / 32) % 3);
        int c = (int)(param % 32);
        int q = 1;
        while (q < c && q < kMaxClusterCtas) q <<= 1;
        *csize = q;
        return;
    }
    *variant = 1;
    const int64_t tiles = (N + cluster_tile_elems(1) - 1) / cluster_tile_elems(1);
    int q = 1;
    while (q < tiles && q < kMaxClusterCtas) q <<= 1;
    *csize = q;
}

int64_t three_stage_chunk(int64_t N, int64_t G, int64_t K) {
    const int64_t tile = chunk_tile_elems();
    if (K > 0) return K * tile;
    // latency-bound totals: one tile per chunk up to 2^19 elements (G = 1: 4.9-5.1 us
    // against 5.6-5.7 us at K = 2), two tiles up to 2^22 (configs[0], 2^20: 5.5 us against
    // 5.7 us at K = 1); tools/g1_probe.py, profiles/r01_g1_probe.jsonl
    if (N * G <= (int64_t(1) << 19)) return tile;
    // up to 2^22: at least two tiles, and few enough chunks (<= kFuse2MaxChunks) that Stage
    // 2 folds into Stage 3 (2^22: 10.3 us against 11.9 us as three launches,
    // profiles/r01_mid_probe.jsonl)
    if (N * G <= (int64_t(1) << 22)) {
        const int64_t c = (N + kFuse2MaxChunks - 1) / kFuse2MaxChunks;
        return std::max<int64_t>(2 * tile, (c + tile - 1) / tile * tile);
    }
    int64_t bx = std::max<int64_t>(1, (kTargetCtas + G - 1) / G);
    int64_t chunk = (N + bx - 1) / bx;
    chunk = std::max<int64_t>(tile, (chunk + tile - 1) / tile * tile);
    // Long portions: chunks of at most kMaxChunkTiles tiles, i.e. many short-lived CTAs in
    // blockIdx order, so the CTAs running at any time stream NEIGHBOURING memory (as the
    // batch kernels do).  ~1184 long chunks spread the concurrent streams ~29 MB apart at
    // 2^33 elements and Stage 3 ran at ~92 % of copy (measured).
    return std::min<int64_t>(chunk, kMaxChunkTiles * tile);
}

// problems per warp span of the packed kernel.  A span is walked in 1024-element windows,
// so a span of k*N elements wastes the unused tail of its last window; k is a multiple of
// q = 4/gcd(N,4) so every span starts 16-byte aligned.  `target` > 0: the largest such k
// with k*N <= target (at least q).  Default: among spans of 2048..8192 elements the one
// whose windows are best used (ties: the shortest) -- measured on B200 (tools/short_probe.py):
// ~4096-element spans beat 1024-element ones by 3-9 % for ragged N, and a half-empty last
// window costs its full latency.
constexpr int64_t kPackedMaxN = int64_t(1) << 24;
constexpr int64_t kPackedWindow = 1024;
int64_t packed_span_problems(int64_t N, int64_t target) {
    N = std::max<int64_t>(N, 1);
    const int64_t q = (N % 4 == 0) ? 1 : (N % 2 == 0) ? 2 : 4;
    if (target > 0) return std::max<int64_t>(target / N / q * q, q);
    int64_t best = q;
    double best_u = -1.0;
    for (int64_t k = q; k == q || k * N <= 8192; k += q) {
        const int64_t span = k * N;
        if (span < 2048 && (k + q) * N <= 8192) continue;
        const double u = (double)span / (double)(((span + kPackedWindow - 1) / kPackedWindow) * kPackedWindow);
        if (u > best_u + 1e-9) { best_u = u; best = k; }
    }
    return best;
}

// Look-back workspace: ctl | desc[C] (16-byte slots).  The layout depends only on the
// workspace size (capacity C), never on the call; every descriptor word carries the tag
// of the launch that wrote it, so 8-byte (32-bit carries) and 16-byte (fp64 carries)
// uses of the same bytes can never be confused.
constexpr size_t kLbSlotBytes = 8 * kDescWords;
size_t lookback_bytes(int64_t total, int variant, bool split) {
    (void)split;
    int64_t tile = lookback_tile_elems(variant);
    int64_t tiles = (total + tile - 1) / tile;
    return kCtlBytes + kLbSlotBytes * (size_t)tiles;
}
size_t fused_bytes(int64_t N, int64_t G) {
    const int64_t tile = fused_tile_elems();
    return kCtlBytes + align_up((size_t)((N * G + tile - 1) / tile) * 8, 256);
}
size_t three_stage_bytes(int64_t N, int64_t G, int64_t K) {
    int64_t chunk = three_stage_chunk(N, G, K);
    int64_t bx = (N + chunk - 1) / chunk;
    return kCtlBytes + align_up(G * bx * 8, 256) + align_up(G * 8, 256);
}

// ---------------------------------------------------------------- workspace cache
struct Ws { void* ptr = nullptr; size_t bytes = 0; };
std::mutex g_ws_mu;
// one cache per (device, stream, family): the look-back descriptors must never share
// bytes with another family's scratch values, and the chunk prefixes that
// scan_shard_totals leaves for scan_shard_scan (FAM_SHARD) must survive any scan_batch
// call the caller issues on the same stream between the two steps
enum Family { FAM_LOOKBACK = 0, FAM_CHUNKED = 1, FAM_SHARD = 2 };
std::map<std::tuple<int, cudaStream_t, int>, Ws> g_ws;

scan_status cached_workspace(cudaStream_t s, int fam, size_t need, void** out, size_t* out_bytes) {
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) return SCAN_ERR_NO_DEVICE;
    std::lock_guard<std::mutex> lk(g_ws_mu);
    Ws& w = g_ws[std::make_tuple(dev, s, fam)];
    if (w.bytes < need) {
        size_t nb = std::max(need, w.bytes * 2);
        if (w.ptr) cudaFreeAsync(w.ptr, s);
        w.ptr = nullptr; w.bytes = 0;
        if (cudaMallocAsync(&w.ptr, nb, s) != cudaSuccess) { cudaGetLastError(); return SCAN_ERR_NO_MEMORY; }
        if (cudaMemsetAsync(w.ptr, 0, nb, s) != cudaSuccess) return SCAN_ERR_CUDA;
        w.bytes = nb;
    }
    *out = w.ptr;
    *out_bytes = w.bytes;
    return SCAN_OK;
}

scan_status resolve_ws(void* ws, size_t ws_bytes, size_t need, cudaStream_t s, int fam, void** out,
                       size_t* out_bytes) {
    if (ws) {
        if (ws_bytes < need) return SCAN_ERR_NO_MEMORY;
        if (((uintptr_t)ws) % 256) return SCAN_ERR_INVALID_ARG;
        *out = ws;
        *out_bytes = ws_bytes;
        return SCAN_OK;
    }
    return cached_workspace(s, fam, need, out, out_bytes);
}

// cross-call programmatic dependent launch of the CTA cascade (SCANB200_NO_PDL=1 disables
// it, for A/B measurements)
const bool g_cross_pdl = std::getenv("SCANB200_NO_PDL") == nullptr;

// look-back options, A/B switches for on-box measurements (round 2):
// SCANB200_LB_MODE=0 restores the round-1 speculative serialized look-back of the L2-staged
// kernel, SCANB200_NO_KEEP_LAST=1 re-reads its last tiles, SCANB200_POLL_NS sets the first
// back-off of a failed window poll
const int g_lb_mode = std::getenv("SCANB200_LB_MODE") ? std::atoi(std::getenv("SCANB200_LB_MODE")) : 1;
const bool g_keep_last = std::getenv("SCANB200_NO_KEEP_LAST") == nullptr;
// sharded path: warp-per-problem Stage 1 / Stage 3 for short portions (SCANB200_NO_WARP_SHARD=1: A/B)
const bool g_warp_shard = std::getenv("SCANB200_NO_WARP_SHARD") == nullptr;
// the L2-staged kernel's read 2 at the tile's aggregate instead of its carry: 3-7 % faster
// up to 2^28 elements, a wash (+-2 %) above (profiles/r02_lb_early_read2_ab.txt);
// SCANB200_EARLY_READ2=1 / SCANB200_LATE_READ2=1 force either form at every size (A/B)
const bool g_early_read2_all = std::getenv("SCANB200_EARLY_READ2") != nullptr;
const bool g_late_read2_all = std::getenv("SCANB200_LATE_READ2") != nullptr;
const uint32_t g_poll_ns = (uint32_t)std::atoi(std::getenv("SCANB200_POLL_NS") ? std::getenv("SCANB200_POLL_NS") : "64");

// debug timeline buffer for the look-back kernels (scan_debug_trace)
uint64_t* g_trace = nullptr;
int64_t g_trace_tiles = 0;

// ---------------------------------------------------------------- argument checks
bool device_accessible(const void* p) {
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, p) != cudaSuccess) { cudaGetLastError(); return false; }
    return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

scan_status check_buffers(const void* in, const void* out, int64_t total, bool check_device) {
    if (!in || !out) return SCAN_ERR_INVALID_ARG;
    if (((uintptr_t)in) % 4 || ((uintptr_t)out) % 4) return SCAN_ERR_INVALID_ARG;
    uintptr_t a = (uintptr_t)in, b = (uintptr_t)out, n = (uintptr_t)total * 4;
    if (a != b && a < b + n && b < a + n) return SCAN_ERR_INVALID_ARG;     // partial overlap
    if (check_device && (!device_accessible(in) || !device_accessible(out))) return SCAN_ERR_INVALID_ARG;
    return SCAN_OK;
}

scan_status check_shape(int64_t N, int64_t G, int64_t* total) {
    if (N < 0 || G < 0) return SCAN_ERR_INVALID_ARG;
    if (N > 0 && G > (int64_t(1) << 62) / N) return SCAN_ERR_INVALID_ARG;
    *total = N * G;
    return SCAN_OK;
}

scan_status from_cuda(cudaError_t e) { return e == cudaSuccess ? SCAN_OK : SCAN_ERR_CUDA; }

// ---------------------------------------------------------------- kernel families
scan_status run_lookback(const void* in, void* out, int64_t N, int64_t G, scan_op op, scan_dtype dt,
                         scan_kind kind, int variant, void* ws, size_t ws_bytes, cudaStream_t s) {
    const int64_t total = N * G;
    const int64_t cap = (int64_t)((ws_bytes - kCtlBytes) / kLbSlotBytes);
    LookbackParams p{};
    p.in = in; p.out = out; p.N = N; p.total = total;
    char* base = (char*)ws;
    p.ctl = (uint32_t*)base;
    p.desc = (uint64_t*)(base + kCtlBytes);
    p.capacity = cap;
    p.trace = g_trace;
    p.trace_tiles = g_trace_tiles;
    p.vec = (((uintptr_t)in) % 16 == 0) && (((uintptr_t)out) % 16 == 0);
    p.exclusive = kind == SCAN_EXCLUSIVE;
    p.pdl_first = g_cross_pdl;
    p.lb_mode = g_lb_mode;
    p.keep_last = g_keep_last;
    p.poll_ns = g_poll_ns;
    p.early_read2 = !g_late_read2_all && (g_early_read2_all || total <= (int64_t(1) << 28));
    return from_cuda(launch_lookback(opcode(op, dt), p, variant, s));
}

ChunkParams chunk_params(const void* in, void* out, int64_t N, int64_t G, scan_kind kind) {
    ChunkParams p{};
    p.in = in; p.out = out; p.N = N; p.G = G;
    p.vec = (((uintptr_t)in) % 16 == 0) && (((uintptr_t)out) % 16 == 0) && (N % 4 == 0);
    p.exclusive = kind == SCAN_EXCLUSIVE;
    // the first wave of Stage 1 (~4 CTAs per SM) prefetches its first tiles while it waits
    // for the previous kernel (later CTAs never wait); profiles/r02_pdl_prefetch_ab.txt
    int sms = 0;
    p.pf_ctas = current_device_sms(&sms) == cudaSuccess ? 4 * (int64_t)sms : 0;
    return p;
}

scan_status run_three_stage(const void* in, void* out, int64_t N, int64_t G, scan_op op, scan_dtype dt,
                            scan_kind kind, int64_t K, void* ws, const uint64_t* carry_src,
                            int carry_rows, cudaStream_t s, bool stages12, bool stage3,
                            uint64_t* totals_out, const PeerParams* peer = nullptr,
                            int64_t carry_stride = 0, bool pdl3 = false) {
    ChunkParams p = chunk_params(in, out, N, G, kind);
    if (peer) p.peer = *peer;
    p.carry_stride = carry_stride;
    p.chunk = three_stage_chunk(N, G, K);
    p.Bx = (N + p.chunk - 1) / p.chunk;
    char* base = (char*)ws + kCtlBytes;
    p.aux = (uint64_t*)base;
    p.totals = totals_out ? totals_out : (uint64_t*)(base + align_up(G * p.Bx * 8, 256));
    p.carry_src = carry_src;
    p.carry_rows = carry_rows;
    const OpCode oc = opcode(op, dt);
    if (stages12 && stage3 && !totals_out && !peer && p.Bx <= kFuse2MaxChunks) {
        // few chunks per problem and nobody needs the totals: Stage 2 is folded into
        // Stage 3's prologue (two launches instead of three; latency-bound totals).
        // Stage 1 is itself a cross-call programmatic launch (waits before reading).
        p.pdl = p.pdl_first = g_cross_pdl;
        cudaError_t e = launch_chunk_reduce(oc, p, s);
        p.pdl_first = false;
        if (e != cudaSuccess) return SCAN_ERR_CUDA;
        p.aux_raw = true;
        p.pdl = true;                                        // Stage 3 overlaps Stage 1's tail
        return from_cuda(launch_chunk_scan(oc, p, s));
    }
    // many short portions (one chunk per problem): Stage 1 and Stage 3 with one warp per
    // problem (profiles/r02_mps_phases_W1.jsonl: one CTA per problem idled at N <= 2048);
    // Stage 2 is folded into Stage 1 there (one chunk per problem: only the totals move)
    const bool warp_path = p.Bx == 1 && N <= 4096 && G >= 1184 && g_warp_shard;
    if (stages12 && warp_path) {
        // Stages 1+2 in one launch (the warp stores and pushes its problem's total)
        if (launch_warp_reduce(oc, p, s) != cudaSuccess) return SCAN_ERR_CUDA;
    } else if (stages12) {
        cudaError_t e = launch_chunk_reduce(oc, p, s);       // normal launch: waits for the caller's work
        if (e != cudaSuccess) return SCAN_ERR_CUDA;
        p.pdl = true;                                        // Stage 2 overlaps Stage 1's tail
        e = launch_aux_scan(oc, p, s);
        if (e != cudaSuccess) return SCAN_ERR_CUDA;
    }
    // Stage 3 directly after this library's Stage 2 (same call, or the fused-exchange
    // path) starts early and loads its first tile while Stage 2 finishes
    p.pdl = stages12 || pdl3;
    if (stage3) return from_cuda(warp_path ? launch_warp_shard_scan(oc, p, s) : launch_chunk_scan(oc, p, s));
    return SCAN_OK;
}

// ---------------------------------------------------------------- tuned choices
// Filled by scan_autotune (the automated form of the paper's empirical K search,
// PAPER.md:183): exact problem (device, N, G, base-pointer alignment, op, dtype, kind) ->
// measured fastest family and parameter.  SCAN_ALGO_AUTO consults it before the static
// rules.  op / dtype / kind are part of the key because the cost differs (fp64 carries of
// f32 add, the exclusive form), and the device because a process may drive several GPUs.
using TuneKey = std::tuple<int, int64_t, int64_t, bool, int, int, int>;
std::mutex g_tune_mu;
std::map<TuneKey, std::pair<scan_algo, int64_t>> g_tuned;

TuneKey tune_key(int64_t N, int64_t G, bool aligned, scan_op op, scan_dtype dt, scan_kind kind) {
    int dev = -1;
    if (cudaGetDevice(&dev) != cudaSuccess) { cudaGetLastError(); dev = -1; }
    return TuneKey(dev, N, G, aligned, (int)op, (int)dt, (int)kind);
}

bool tuned_choice(const TuneKey& key, scan_algo* algo, int64_t* param) {
    std::lock_guard<std::mutex> lk(g_tune_mu);
    auto it = g_tuned.find(key);
    if (it == g_tuned.end()) return false;
    *algo = it->second.first;
    *param = it->second.second;
    return true;
}

scan_status run_algo(const void* in, void* out, int64_t N, int64_t G, scan_op op, scan_dtype dt,
                     scan_kind kind, scan_algo algo, int64_t param, void* ws, size_t ws_bytes,
                     cudaStream_t s) {
    if (algo == SCAN_ALGO_AUTO) {
        const bool aligned = (((uintptr_t)in) % 16 == 0) && (((uintptr_t)out) % 16 == 0);
        // a caller workspace is sized for the static choice (scan_workspace_bytes(AUTO)),
        // so tuned choices apply only with the library's own workspace
        if (ws || !tuned_choice(tune_key(N, G, aligned, op, dt, kind), &algo, &param)) {
            algo = choose_algo(N, G, aligned);
            // a caller workspace is sized and laid out for the look-back family
            // (scan_workspace_bytes(AUTO)); never let AUTO put three-stage or fused scratch
            // (untagged values the look-back could misread) into it
            if (ws && (algo == SCAN_ALGO_THREE_STAGE || algo == SCAN_ALGO_FUSED)) algo = SCAN_ALGO_LOOKBACK;
            param = -1;
        }
    }
    switch (algo) {
    case SCAN_ALGO_LOOKBACK: {
        if (param >= 0 && !lookback_variant_valid((int)param)) return SCAN_ERR_UNSUPPORTED;
        int variant = param >= 0 ? (int)param : choose_lookback_variant(N, G);
        void* w = nullptr;
        size_t wb = 0;
        scan_status st = resolve_ws(ws, ws_bytes, lookback_bytes(N * G, variant, split_desc(op, dt)), s,
                                    FAM_LOOKBACK, &w, &wb);
        if (st != SCAN_OK) return st;
        return run_lookback(in, out, N, G, op, dt, kind, variant, w, wb, s);
    }
    case SCAN_ALGO_CASCADE_CTA: {
        ChunkParams p = chunk_params(in, out, N, G, kind);
        p.chunk = std::max<int64_t>(N, 1); p.Bx = 1;
        // programmatic launch behind the stream's previous kernel: the CTAs are scheduled
        // into the SMs its last wave frees and wait there (griddepcontrol.wait) before
        // their first access, so back-to-back calls lose no launch gap
        p.pdl = p.pdl_first = g_cross_pdl;
        return from_cuda(launch_chunk_scan(opcode(op, dt), p, s));
    }
    case SCAN_ALGO_CASCADE_WARP: {
        ChunkParams p = chunk_params(in, out, N, G, kind);
        p.chunk = std::max<int64_t>(N, 1); p.Bx = 1;
        p.pdl = p.pdl_first = g_cross_pdl;
        return from_cuda(launch_warp_cascade(opcode(op, dt), p, s));
    }
    case SCAN_ALGO_PACKED_WARP: {
        if (N > kPackedMaxN) return SCAN_ERR_UNSUPPORTED;
        ChunkParams p = chunk_params(in, out, N, G, kind);
        p.vec = (((uintptr_t)in) % 16 == 0) && (((uintptr_t)out) % 16 == 0);
        p.chunk = packed_span_problems(N, param); p.Bx = 1;
        p.pdl = p.pdl_first = g_cross_pdl;
        return from_cuda(launch_packed_warp(opcode(op, dt), p, s));
    }
    case SCAN_ALGO_CLUSTER: {
        int variant = 0, csize = 0;
        cluster_config(N, param, &variant, &csize);
        if ((int64_t)G * csize > 0x7FFFFFFFll) return SCAN_ERR_UNSUPPORTED;
        ChunkParams p = chunk_params(in, out, N, G, kind);
        p.pdl_first = g_cross_pdl;
        return from_cuda(launch_cluster_scan(opcode(op, dt), p, variant, csize, s));
    }
    case SCAN_ALGO_FUSED: {
        const int64_t tile = fused_tile_elems();
        const int64_t tiles = (N * G + tile - 1) / tile;
        if (!(G == 1 || N % tile == 0)) return SCAN_ERR_UNSUPPORTED;
        if (tiles > fused_max_tiles(opcode(op, dt))) return SCAN_ERR_UNSUPPORTED;
        void* w = nullptr;
        size_t wb = 0;
        scan_status st = resolve_ws(ws, ws_bytes, fused_bytes(N, G), s, FAM_CHUNKED, &w, &wb);
        if (st != SCAN_OK) return st;
        FusedParams p{};
        p.in = in; p.out = out; p.total = N * G;
        p.tiles_per_problem = G == 1 ? tiles : N / tile;
        p.aux = (uint64_t*)((char*)w + kCtlBytes);
        p.vec = (((uintptr_t)in) % 16 == 0) && (((uintptr_t)out) % 16 == 0);
        p.exclusive = kind == SCAN_EXCLUSIVE;
        p.pdl_first = g_cross_pdl;
        return from_cuda(launch_fused(opcode(op, dt), p, s));
    }
    case SCAN_ALGO_THREE_STAGE: {
        void* w = nullptr;
        size_t wb = 0;
        scan_status st = resolve_ws(ws, ws_bytes, three_stage_bytes(N, G, param), s, FAM_CHUNKED, &w, &wb);
        if (st != SCAN_OK) return st;
        return run_three_stage(in, out, N, G, op, dt, kind, param, w, nullptr, 0, s, true, true, nullptr);
    }
    default:
        return SCAN_ERR_UNSUPPORTED;
    }
}

// ---------------------------------------------------------------- host-buffer pipeline
// Three streams per device: copy-in, compute, copy-out; S staging slots of kPiece
// elements rotate through them so the H2D copy of unit u+1, the scan of unit u and the
// D2H copy of unit u-1 overlap (both copy engines busy: PCIe is full duplex).
// Staging granularity: small enough that the first copy-in and the last copy-out (which
// cannot overlap anything) are short, large enough to amortise per-copy costs.  Defaults
// from the on-box e2e sweep; SCANB200_HOST_PIECE / SCANB200_HOST_SLOTS override them.
constexpr int kMaxSlots = 8;

int64_t env_i64(const char* name, int64_t dflt, int64_t lo, int64_t hi) {
    const char* s = std::getenv(name);
    if (!s) return dflt;
    const long long v = std::atoll(s);
    return v < lo ? lo : v > hi ? hi : v;
}
int64_t host_piece() {                               // elements per staging slot
    static const int64_t v = env_i64("SCANB200_HOST_PIECE", int64_t(1) << 22, int64_t(1) << 16, int64_t(1) << 26);
    return v;
}
int host_slots() {
    static const int v = (int)env_i64("SCANB200_HOST_SLOTS", 4, 2, kMaxSlots);
    return v;
}

struct HostCtx {
    bool init = false;
    cudaStream_t h2d = nullptr, comp = nullptr, d2h = nullptr;
    void* slot[kMaxSlots] = {};
    cudaEvent_t ev_in[kMaxSlots] = {}, ev_scan[kMaxSlots] = {}, ev_out[kMaxSlots] = {};
    uint64_t* piece_totals = nullptr;
    int64_t piece_cap = 0;
};
std::mutex g_host_mu;
std::map<int, HostCtx> g_host;

scan_status host_ctx(int dev, HostCtx** out) {
    HostCtx& c = g_host[dev];
    if (!c.init) {
        if (cudaStreamCreateWithFlags(&c.h2d, cudaStreamNonBlocking) != cudaSuccess ||
            cudaStreamCreateWithFlags(&c.comp, cudaStreamNonBlocking) != cudaSuccess ||
            cudaStreamCreateWithFlags(&c.d2h, cudaStreamNonBlocking) != cudaSuccess)
            return SCAN_ERR_CUDA;
        for (int k = 0; k < host_slots(); ++k) {
            if (cudaMalloc(&c.slot[k], host_piece() * 4) != cudaSuccess) { cudaGetLastError(); return SCAN_ERR_NO_MEMORY; }
            if (cudaEventCreateWithFlags(&c.ev_in[k], cudaEventDisableTiming) != cudaSuccess ||
                cudaEventCreateWithFlags(&c.ev_scan[k], cudaEventDisableTiming) != cudaSuccess ||
                cudaEventCreateWithFlags(&c.ev_out[k], cudaEventDisableTiming) != cudaSuccess)
                return SCAN_ERR_CUDA;
        }
        c.init = true;
    }
    *out = &c;
    return SCAN_OK;
}

// One staging unit: elements [off, off + n) of the flat batch = problems [g0, g0 + ng)
// (whole problems, N <= piece) or piece j of problem g0 (long problems).
struct HostUnit { int64_t off, n, g0, ng, j; };

// Units of at most `piece` elements with a short RAMP at both ends of the call: the first
// host->device copy and the last device->host copy cannot overlap anything (the pipeline
// fills and drains), so they are made short -- piece/16, piece/4, then full pieces, then
// piece/4, piece/16 (e2e).  Whole problems per unit when N <= piece; pieces
// of one problem otherwise (a piece never spans two problems).
std::vector<HostUnit> host_units(int64_t N, int64_t G, int64_t piece) {
    std::vector<HostUnit> u;
    const int64_t total = N * G;
    const bool ramp = total > 2 * piece;
    const int64_t r1 = std::max<int64_t>(piece / 16, 1), r2 = std::max<int64_t>(piece / 4, 1);
    int64_t g = 0, e = 0, done = 0, j = 0;
    while (done < total) {
        const int64_t rem = total - done;
        int64_t b = piece;
        if (ramp) {
            if (u.size() == 0) b = r1;
            else if (u.size() == 1) b = r2;
            else if (rem <= r1) b = rem;
            else if (rem <= r1 + r2) b = rem - r1;
            else if (rem <= piece + r1 + r2) b = rem - r1 - r2;
        }
        b = std::min(b, piece);
        HostUnit h{};
        if (N <= piece) {
            const int64_t ng = std::min<int64_t>(std::max<int64_t>(b / N, 1), G - g);
            h = HostUnit{g * N, ng * N, g, ng, 0};
            g += ng;
        } else {
            const int64_t n = std::min<int64_t>(std::max<int64_t>(b, 1), N - e);
            h = HostUnit{g * N + e, n, g, 1, j};
            e += n;
            ++j;
            if (e == N) { e = 0; j = 0; ++g; }
        }
        done += h.n;
        u.push_back(h);
    }
    return u;
}

scan_status host_pipeline(const void* in_host, void* out_host, int64_t N, int64_t G, scan_op op,
                          scan_dtype dt, scan_kind kind) {
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) return SCAN_ERR_NO_DEVICE;
    std::lock_guard<std::mutex> lk(g_host_mu);
    HostCtx* c = nullptr;
    scan_status st = host_ctx(dev, &c);
    if (st != SCAN_OK) return st;
    const int64_t kPiece = host_piece();
    const int kSlots = host_slots();
    const bool pieces = N > kPiece;
    const std::vector<HostUnit> units = host_units(N, G, kPiece);
    int64_t npieces = 0;
    for (const HostUnit& h : units) npieces = std::max<int64_t>(npieces, h.j + 1);
    if (pieces && c->piece_cap < npieces) {
        if (c->piece_totals) cudaFree(c->piece_totals);
        c->piece_totals = nullptr;
        if (cudaMalloc(&c->piece_totals, npieces * 8) != cudaSuccess) { cudaGetLastError(); return SCAN_ERR_NO_MEMORY; }
        c->piece_cap = npieces;
    }
    const char* src = (const char*)in_host;
    char* dst = (char*)out_host;
    for (size_t u = 0; u < units.size(); ++u) {
        const int k = (int)(u % kSlots);
        const HostUnit& h = units[u];
        if (u >= (size_t)kSlots && cudaStreamWaitEvent(c->h2d, c->ev_out[k], 0) != cudaSuccess) return SCAN_ERR_CUDA;
        if (cudaMemcpyAsync(c->slot[k], src + h.off * 4, h.n * 4, cudaMemcpyHostToDevice, c->h2d) != cudaSuccess)
            return SCAN_ERR_CUDA;
        if (cudaEventRecord(c->ev_in[k], c->h2d) != cudaSuccess) return SCAN_ERR_CUDA;
        if (cudaStreamWaitEvent(c->comp, c->ev_in[k], 0) != cudaSuccess) return SCAN_ERR_CUDA;
        if (pieces) {
            // piece j of a problem: three-stage scan whose carry folds the totals of pieces 0..j-1
            void* w = nullptr; size_t wb = 0;
            st = cached_workspace(c->comp, FAM_CHUNKED, three_stage_bytes(h.n, 1, 0), &w, &wb);
            if (st != SCAN_OK) return st;
            st = run_three_stage(c->slot[k], c->slot[k], h.n, 1, op, dt, kind, 0, w, c->piece_totals,
                                 (int)h.j, c->comp, true, true, c->piece_totals + h.j);
        } else {
            st = run_algo(c->slot[k], c->slot[k], N, h.ng, op, dt, kind, SCAN_ALGO_AUTO, -1, nullptr, 0, c->comp);
        }
        if (st != SCAN_OK) return st;
        if (cudaEventRecord(c->ev_scan[k], c->comp) != cudaSuccess) return SCAN_ERR_CUDA;
        if (cudaStreamWaitEvent(c->d2h, c->ev_scan[k], 0) != cudaSuccess) return SCAN_ERR_CUDA;
        if (cudaMemcpyAsync(dst + h.off * 4, c->slot[k], h.n * 4, cudaMemcpyDeviceToHost, c->d2h) != cudaSuccess)
            return SCAN_ERR_CUDA;
        if (cudaEventRecord(c->ev_out[k], c->d2h) != cudaSuccess) return SCAN_ERR_CUDA;
    }
    return from_cuda(cudaStreamSynchronize(c->d2h));
}

}  // namespace

// =================================================================== exported C-ABI
extern "C" {

const char* scan_status_string(scan_status s) {
    switch (s) {
    case SCAN_OK: return "SCAN_OK";
    case SCAN_ERR_INVALID_ARG: return "SCAN_ERR_INVALID_ARG";
    case SCAN_ERR_UNSUPPORTED: return "SCAN_ERR_UNSUPPORTED";
    case SCAN_ERR_CUDA: return "SCAN_ERR_CUDA";
    case SCAN_ERR_NCCL: return "SCAN_ERR_NCCL";
    case SCAN_ERR_NO_MEMORY: return "SCAN_ERR_NO_MEMORY";
    case SCAN_ERR_NO_DEVICE: return "SCAN_ERR_NO_DEVICE";
    }
    return "SCAN_ERR_UNKNOWN";
}

int scan_abi_version(void) { return SCAN_B200_ABI_VERSION; }

scan_status scan_debug_trace(void* device_buf, int64_t tiles) {
    if (tiles < 0 || (tiles > 0 && !device_buf)) return SCAN_ERR_INVALID_ARG;
    g_trace = tiles ? (uint64_t*)device_buf : nullptr;
    g_trace_tiles = tiles;
    return SCAN_OK;
}

scan_status scan_plan_ex(int64_t N, int64_t G, scan_op op, scan_dtype dtype, scan_kind kind, const void* in,
                         const void* out, int* algo, int64_t* param) {
    if (!algo || !param || N < 0 || G < 0 || !valid_enums(op, dtype, kind)) return SCAN_ERR_INVALID_ARG;
    const bool aligned = (((uintptr_t)in) % 16 == 0) && (((uintptr_t)out) % 16 == 0);
    scan_algo ta;
    int64_t tp;
    if (tuned_choice(tune_key(N, G, aligned, op, dtype, kind), &ta, &tp)) {
        *algo = (int)ta;
        *param = tp;
        return SCAN_OK;
    }
    const scan_algo a = choose_algo(N, G, aligned);
    *algo = (int)a;
    *param = a == SCAN_ALGO_LOOKBACK ? choose_lookback_variant(N, G) : -1;
    return SCAN_OK;
}

scan_status scan_plan(int64_t N, int64_t G, const void* in, const void* out, int* algo, int64_t* param) {
    return scan_plan_ex(N, G, SCAN_OP_ADD, SCAN_I32, SCAN_INCLUSIVE, in, out, algo, param);
}

size_t scan_workspace_bytes(int64_t N, int64_t G, scan_op op, scan_dtype dtype, scan_algo algo, int64_t param) {
    if (N <= 0 || G <= 0) return kCtlBytes;
    if (algo == SCAN_ALGO_AUTO) {
        // pointer alignment is unknown here: cover the look-back choice (the only one that
        // needs workspace) with its largest descriptor array (8192-element tiles)
        return lookback_bytes(N * G, 1, split_desc(op, dtype));
    }
    if (algo == SCAN_ALGO_LOOKBACK) {
        if (param >= 0 && !lookback_variant_valid((int)param)) return kCtlBytes;
        int variant = param >= 0 ? (int)param : choose_lookback_variant(N, G);
        return lookback_bytes(N * G, variant, split_desc(op, dtype));
    }
    if (algo == SCAN_ALGO_THREE_STAGE) return three_stage_bytes(N, G, param);
    if (algo == SCAN_ALGO_FUSED) return fused_bytes(N, G);
    return kCtlBytes;
}

scan_status scan_batch_ex(const void* in, void* out, int64_t N, int64_t G, scan_op op, scan_dtype dtype,
                          scan_kind kind, scan_algo algo, int64_t param, void* workspace,
                          size_t workspace_bytes, void* stream) {
    NvtxRange nvtx_range("scan_batch");
    if (!valid_enums(op, dtype, kind)) return SCAN_ERR_INVALID_ARG;
    if (algo < SCAN_ALGO_AUTO || algo > SCAN_ALGO_FUSED) return SCAN_ERR_UNSUPPORTED;
    int64_t total = 0;
    scan_status st = check_shape(N, G, &total);
    if (st != SCAN_OK) return st;
    if (total == 0) return SCAN_OK;
    st = check_buffers(in, out, total, true);
    if (st != SCAN_OK) return st;
    if (algo == SCAN_ALGO_THREE_STAGE && param < 0) param = 0;          // auto K
    return run_algo(in, out, N, G, op, dtype, kind, algo, param, workspace, workspace_bytes,
                    (cudaStream_t)stream);
}

scan_status scan_batch(const void* in, void* out, int64_t N, int64_t G, scan_op op, scan_dtype dtype,
                       scan_kind kind, void* stream) {
    return scan_batch_ex(in, out, N, G, op, dtype, kind, SCAN_ALGO_AUTO, -1, nullptr, 0, stream);
}

scan_status scan_autotune(const void* in, void* out, int64_t N, int64_t G, scan_op op, scan_dtype dtype,
                          scan_kind kind, void* stream, int* algo_out, int64_t* param_out, float* us_out) {
    NvtxRange nvtx_range("scan_autotune");
    if (!valid_enums(op, dtype, kind)) return SCAN_ERR_INVALID_ARG;
    int64_t total = 0;
    scan_status st = check_shape(N, G, &total);
    if (st != SCAN_OK) return st;
    if (total == 0) return SCAN_ERR_INVALID_ARG;
    st = check_buffers(in, out, total, true);
    if (st != SCAN_OK) return st;
    if (in == out) return SCAN_ERR_INVALID_ARG;          // timing runs would rescan the output
    cudaStream_t s = (cudaStream_t)stream;
    const bool aligned = (((uintptr_t)in) % 16 == 0) && (((uintptr_t)out) % 16 == 0);
    // candidates: every family that takes this shape at a sane cost (a single CTA or warp
    // per problem is excluded for few long problems: it would run for seconds)
    std::vector<std::pair<scan_algo, int64_t>> cand;
    for (int v : {0, 1, 2, 3, 10}) cand.push_back({SCAN_ALGO_LOOKBACK, v});
    for (int k : {0, 1, 2, 4}) cand.push_back({SCAN_ALGO_THREE_STAGE, k});
    if (G >= 64 || N <= (int64_t(1) << 16)) cand.push_back({SCAN_ALGO_CASCADE_CTA, -1});
    if (G >= 256 && N <= (int64_t(1) << 16)) cand.push_back({SCAN_ALGO_CASCADE_WARP, -1});
    if (aligned && N < 1024) cand.push_back({SCAN_ALGO_PACKED_WARP, -1});
    cand.push_back({SCAN_ALGO_FUSED, -1});                   // rejects ineligible shapes itself
    if (N <= (int64_t(1) << 20) && G * kMaxClusterCtas <= 0x7FFFFFFFll)
        for (int v = 0; v < 3; ++v)
            for (int c : {2, 4, 8, 16}) cand.push_back({SCAN_ALGO_CLUSTER, 32 * v + c});
    // Device time per call, measured like the on-box sweeps: `reps` calls captured into a
    // CUDA graph on the library's tuning stream and replayed between two events, so host
    // launch overhead does not pick the winner of small, latency-bound shapes.
    cudaStream_t ts = nullptr;
    {
        int dev = 0;
        if (cudaGetDevice(&dev) != cudaSuccess) return SCAN_ERR_NO_DEVICE;
        static std::map<int, cudaStream_t> streams;          // one per device, kept (its
        std::lock_guard<std::mutex> lk(g_tune_mu);            // workspaces are cached)
        auto it = streams.find(dev);
        if (it == streams.end()) {
            if (cudaStreamCreateWithFlags(&ts, cudaStreamNonBlocking) != cudaSuccess) return SCAN_ERR_CUDA;
            streams[dev] = ts;
        } else {
            ts = it->second;
        }
    }
    if (cudaStreamSynchronize(s) != cudaSuccess) return SCAN_ERR_CUDA;     // the caller's inputs
    cudaEvent_t e0, e1;
    if (cudaEventCreate(&e0) != cudaSuccess) return SCAN_ERR_CUDA;
    if (cudaEventCreate(&e1) != cudaSuccess) { cudaEventDestroy(e0); return SCAN_ERR_CUDA; }
    float best = -1.0f;
    std::pair<scan_algo, int64_t> win{SCAN_ALGO_AUTO, -1};
    st = SCAN_OK;
    for (const auto& c : cand) {
        // warm-up call outside any capture (workspace growth, first-launch attributes); a
        // family that rejects the shape is skipped
        if (run_algo(in, out, N, G, op, dtype, kind, c.first, c.second, nullptr, 0, ts) != SCAN_OK ||
            cudaStreamSynchronize(ts) != cudaSuccess) {
            cudaGetLastError();
            continue;
        }
        float ms1 = 0.0f;
        if (cudaEventRecord(e0, ts) != cudaSuccess) { st = SCAN_ERR_CUDA; break; }
        run_algo(in, out, N, G, op, dtype, kind, c.first, c.second, nullptr, 0, ts);
        if (cudaEventRecord(e1, ts) != cudaSuccess || cudaEventSynchronize(e1) != cudaSuccess ||
            cudaEventElapsedTime(&ms1, e0, e1) != cudaSuccess) { st = SCAN_ERR_CUDA; break; }
        if (best > 0.0f && ms1 > 20.0f * best) continue;          // far off: not worth more reps
        const int reps = (int)std::min(20.0f, std::max(2.0f, 1.0f / std::max(ms1, 1e-3f)));
        cudaGraph_t graph = nullptr;
        cudaGraphExec_t exec = nullptr;
        if (cudaStreamBeginCapture(ts, cudaStreamCaptureModeThreadLocal) != cudaSuccess) { st = SCAN_ERR_CUDA; break; }
        bool ok = true;
        for (int r = 0; r < reps && ok; ++r)
            ok = run_algo(in, out, N, G, op, dtype, kind, c.first, c.second, nullptr, 0, ts) == SCAN_OK;
        if (cudaStreamEndCapture(ts, &graph) != cudaSuccess) ok = false;
        if (ok && cudaGraphInstantiate(&exec, graph, 0) != cudaSuccess) ok = false;
        float ms = 0.0f;
        if (ok) ok = cudaGraphLaunch(exec, ts) == cudaSuccess && cudaEventRecord(e0, ts) == cudaSuccess &&
                     cudaGraphLaunch(exec, ts) == cudaSuccess && cudaEventRecord(e1, ts) == cudaSuccess &&
                     cudaEventSynchronize(e1) == cudaSuccess && cudaEventElapsedTime(&ms, e0, e1) == cudaSuccess;
        if (exec) cudaGraphExecDestroy(exec);
        if (graph) cudaGraphDestroy(graph);
        if (!ok) {                     // not capturable / failed: this candidate is skipped
            cudaGetLastError();
            cudaStreamSynchronize(ts);
            continue;
        }
        ms /= reps;
        if (best < 0.0f || ms < best) { best = ms; win = c; }
    }
    cudaStreamSynchronize(ts);
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    if (st != SCAN_OK) return st;
    if (best < 0.0f) return SCAN_ERR_UNSUPPORTED;
    {
        std::lock_guard<std::mutex> lk(g_tune_mu);
        g_tuned[tune_key(N, G, aligned, op, dtype, kind)] = win;
    }
    if (algo_out) *algo_out = (int)win.first;
    if (param_out) *param_out = win.second;
    if (us_out) *us_out = best * 1e3f;
    return SCAN_OK;
}

scan_status scan_autotune_clear(void) {
    std::lock_guard<std::mutex> lk(g_tune_mu);
    g_tuned.clear();
    return SCAN_OK;
}

scan_status scan_batch_host(const void* in_host, void* out_host, int64_t N, int64_t G, scan_op op,
                            scan_dtype dtype, scan_kind kind) {
    NvtxRange nvtx_range("scan_batch_host");
    if (!valid_enums(op, dtype, kind)) return SCAN_ERR_INVALID_ARG;
    int64_t total = 0;
    scan_status st = check_shape(N, G, &total);
    if (st != SCAN_OK) return st;
    if (total == 0) return SCAN_OK;
    st = check_buffers(in_host, out_host, total, false);
    if (st != SCAN_OK) return st;
    if (N > (int64_t(1) << 54)) return SCAN_ERR_UNSUPPORTED;      // piece count must fit an int
    return host_pipeline(in_host, out_host, N, G, op, dtype, kind);
}

// ---------------------------------------------------------------- sharded problems
size_t scan_shard_workspace_bytes(int64_t N_local, int64_t G) {
    if (N_local < 0 || G <= 0) return kCtlBytes;
    return three_stage_bytes(N_local, G, 0);      // an empty portion still needs its G totals
}

scan_status scan_shard_totals(const void* in_local, int64_t N_local, int64_t G, scan_op op, scan_dtype dtype,
                              void* totals_dev, void* workspace, size_t workspace_bytes, void* stream) {
    NvtxRange nvtx_range("stage1+2 (chunk reduce, totals)");
    if (!valid_enums(op, dtype, SCAN_INCLUSIVE)) return SCAN_ERR_INVALID_ARG;
    int64_t total = 0;
    scan_status st = check_shape(N_local, G, &total);
    if (st != SCAN_OK) return st;
    if (G == 0) return SCAN_OK;
    if (!totals_dev || ((uintptr_t)totals_dev) % 8) return SCAN_ERR_INVALID_ARG;
    cudaStream_t s = (cudaStream_t)stream;
    if (total > 0) {            // an empty portion still writes the identity totals (Stage 2 only)
        st = check_buffers(in_local, in_local, total, true);
        if (st != SCAN_OK) return st;
    }
    void* w = nullptr;
    size_t wb = 0;
    st = resolve_ws(workspace, workspace_bytes, three_stage_bytes(N_local, G, 0), s, FAM_SHARD, &w, &wb);
    if (st != SCAN_OK) return st;
    return run_three_stage(in_local, nullptr, N_local, G, op, dtype, SCAN_INCLUSIVE, 0, w, nullptr, 0, s,
                           true, false, (uint64_t*)totals_dev);
}

scan_status scan_shard_scan(const void* in_local, void* out_local, int64_t N_local, int64_t G, scan_op op,
                            scan_dtype dtype, scan_kind kind, const void* all_totals_dev, int rank, int ngpu,
                            void* workspace, size_t workspace_bytes, void* stream) {
    NvtxRange nvtx_range("stage3 (scan + carry)");
    if (!valid_enums(op, dtype, kind)) return SCAN_ERR_INVALID_ARG;
    if (ngpu < 1 || rank < 0 || rank >= ngpu) return SCAN_ERR_INVALID_ARG;
    int64_t total = 0;
    scan_status st = check_shape(N_local, G, &total);
    if (st != SCAN_OK) return st;
    if (total == 0) return SCAN_OK;
    if (rank > 0 && (!all_totals_dev || ((uintptr_t)all_totals_dev) % 8)) return SCAN_ERR_INVALID_ARG;
    st = check_buffers(in_local, out_local, total, true);
    if (st != SCAN_OK) return st;
    cudaStream_t s = (cudaStream_t)stream;
    void* w = nullptr;
    size_t wb = 0;
    st = resolve_ws(workspace, workspace_bytes, three_stage_bytes(N_local, G, 0), s, FAM_SHARD, &w, &wb);
    if (st != SCAN_OK) return st;
    return run_three_stage(in_local, out_local, N_local, G, op, dtype, kind, 0, w,
                           (const uint64_t*)all_totals_dev, rank, s, false, true, nullptr);
}

}  // extern "C"

// ---------------------------------------------------------------- fused peer exchange
// Both halves of one rank's sharded call with the exchange done by the kernels over peer
// memory (scan_multi.cu owns the mailboxes).  carry rows = ranks < rank of the mailbox.
scan_status scanb200::shard_run_peer(const void* in, void* out, int64_t N_local, int64_t G, scan_op op,
                                     scan_dtype dt, scan_kind kind, void* ws, size_t ws_bytes,
                                     uint64_t* totals, const uint64_t* mailbox_rows, int64_t row_stride,
                                     const PeerParams& peer, cudaStream_t s) {
    if (!valid_enums(op, dt, kind)) return SCAN_ERR_INVALID_ARG;
    int64_t total = 0;
    scan_status st = check_shape(N_local, G, &total);
    if (st != SCAN_OK) return st;
    if (G == 0) return SCAN_OK;
    if (total > 0) {
        st = check_buffers(in, out, total, true);
        if (st != SCAN_OK) return st;
    }
    if (ws_bytes < three_stage_bytes(N_local, G, 0)) return SCAN_ERR_NO_MEMORY;
    st = run_three_stage(in, out, N_local, G, op, dt, kind, 0, ws, mailbox_rows, peer.rank, s, true, false,
                         totals, &peer, row_stride);
    if (st != SCAN_OK) return st;
    if (total == 0) return from_cuda(launch_peer_ack(peer, s));
    return run_three_stage(in, out, N_local, G, op, dt, kind, 0, ws, mailbox_rows, peer.rank, s, false, true,
                           totals, &peer, row_stride, true);
}
