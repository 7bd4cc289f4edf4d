// scan_chunked.cu -- per-problem chunked kernels: the paper's cascade (PAPER.md:126 [§3.1,
// Fig. 5]) and three-stage reduce-then-scan (PAPER.md:110-118 [§3.1, Fig. 3]), on sm_100a.
//
//   chunk_reduce  (Stage 1, "Chunk Reduce")      one CTA per (problem, chunk); the CTA walks
//                                                the chunk tile by tile (cascade, K tiles)
//                                                and writes one value per chunk to aux.
//   aux_scan      (Stage 2, "Intermediate Scan") one WARP per problem (L_y^2 = warps per
//                                                block problems per CTA);
//                                                exclusive scan of the Bx chunk values in
//                                                place + the problem total.
//   chunk_scan    (Stage 3, "Scan+Addition")     one CTA per (problem, chunk); carry =
//                                                (rank carry rows) . aux prefix, then a
//                                                cascade over the chunk's tiles.  With one
//                                                chunk per problem and no aux this is the
//                                                CTA-per-problem batch kernel (L_y = 1).
//   warp_cascade                                  one WARP per problem, cascade over
//                                                V*128-element windows (small/medium N).
//   packed_warp                                   k whole SHORT problems per warp (one
//                                                span of k*N elements, segmented scan).
//
// Aux, totals and carry slots are 8 bytes: the 32-bit value in the low half, or the fp64
// carry of f32 add.  All problem-local indices are 64-bit (N*G reaches 2^36).
#include "scan_common.cuh"
#include "scan_internal.h"

namespace scanb200 {

namespace {

constexpr int CH_WARPS = 8, CH_V = 4;           // chunk kernels: 4096-element tiles
constexpr int WC_WARPS = 8, WC_V = 8;           // warp cascade: 1024-element windows per warp

template <class C> __device__ __forceinline__ C slot_get(uint64_t s);
template <> __device__ __forceinline__ uint32_t slot_get<uint32_t>(uint64_t s) { return (uint32_t)s; }
template <> __device__ __forceinline__ int32_t slot_get<int32_t>(uint64_t s) { return (int32_t)(uint32_t)s; }
template <> __device__ __forceinline__ float slot_get<float>(uint64_t s) { return __uint_as_float((uint32_t)s); }
template <> __device__ __forceinline__ double slot_get<double>(uint64_t s) { return __longlong_as_double((long long)s); }
__device__ __forceinline__ uint64_t slot_put(uint32_t v) { return v; }
__device__ __forceinline__ uint64_t slot_put(int32_t v) { return (uint32_t)v; }
__device__ __forceinline__ uint64_t slot_put(float v) { return __float_as_uint(v); }
__device__ __forceinline__ uint64_t slot_put(double v) { return (uint64_t)__double_as_longlong(v); }

template <class C> __device__ __forceinline__ C shfl_up_c(C v, int d) {
    if constexpr (sizeof(C) == 8) return __shfl_up_sync(FULL, v, d);
    else return from_bits<C>(__shfl_up_sync(FULL, to_bits<C>(v), d));
}
template <class C> __device__ __forceinline__ C shfl_idx_c(C v, int s) {
    if constexpr (sizeof(C) == 8) return __shfl_sync(FULL, v, s);
    else return from_bits<C>(__shfl_sync(FULL, to_bits<C>(v), s));
}

// ------------------------------------------------------------------ Stage 1
template <class Op, int WARPS, int V>
__global__ void __launch_bounds__(WARPS * 32) chunk_reduce_kernel(ChunkParams p) {
    using T = typename Op::T;
    using C = typename Op::Carry;
    constexpr int TILE = WARPS * 32 * V * 4, WCH = V * 128;
    __shared__ __align__(16) C s_part[(WARPS + 3) & ~3];
    const int warp = threadIdx.x >> 5, lane = lane_id();
    const int64_t g = (int64_t)blockIdx.x / p.Bx, c = (int64_t)blockIdx.x % p.Bx;
    const int64_t row = g * p.N;
    const int64_t start = c * p.chunk;
    const int64_t end = (start + p.chunk < p.N) ? start + p.chunk : p.N;
    const T* in = (const T*)p.in;
    // Ordering rule of the library: a kernel may touch memory before its own
    // griddepcontrol.wait only if its primary executed the wait BEFORE it triggered.  The
    // fused Stage 3 (aux_raw) loads its first input tile before waiting, so when this
    // Stage 1 is itself a cross-call programmatic dependent (pdl_first) it waits for the
    // stream's previous kernel -- which may trigger at entry and still be writing our
    // input -- before letting Stage 3 launch.  Otherwise Stage 1 was a normal launch and
    // everything before it is complete: trigger at once.
    if (p.pdl_first && threadIdx.x == 0 && (int64_t)blockIdx.x < p.pf_ctas)
        prefetch_l2_span(in + row + start, min(end - start, (int64_t)2 * TILE));
    if (p.pdl_first) grid_dep_wait();      // cross-call programmatic launch (ChunkParams)
    grid_dep_launch();          // Stage 2 / fused Stage 3 may be scheduled now

    C acc = Op::cidentity();
    // two tiles per iteration: both tiles' rows are in flight before either is reduced
    // (one memory latency per 2 tiles; rows past the chunk end load as the identity)
    for (int64_t off = start + warp * WCH; off < end; off += 2 * TILE) {
        Row4<T> x[2 * V];
#pragma unroll
        for (int j = 0; j < V; ++j) x[j] = load_row<Op>(in, row + off + j * 128 + lane * 4, row + end, p.vec);
#pragma unroll
        for (int j = 0; j < V; ++j)
            x[V + j] = load_row<Op>(in, row + off + TILE + j * 128 + lane * 4, row + end, p.vec);
#pragma unroll
        for (int h = 0; h < 2; ++h) {
            T t = Op::identity();
#pragma unroll
            for (int j = 0; j < V; ++j)
#pragma unroll
                for (int k = 0; k < 4; ++k) t = Op::apply(t, x[h * V + j].v[k]);
            acc = Op::capply(acc, Op::to_carry(t));
        }
    }
    acc = warp_reduce_carry<Op>(acc);
    if (lane == 0) s_part[warp] = acc;
    __syncthreads();
    if (threadIdx.x == 0) {
        C tot = Op::cidentity();
#pragma unroll
        for (int w = 0; w < WARPS; ++w) tot = Op::capply(tot, s_part[w]);
        p.aux[g * p.Bx + c] = slot_put(tot);
    }
}

// ------------------------------------------------------------------ fused peer exchange
// Spin helpers of the peer protocol (scan_internal.h, PeerParams).  One thread per CTA
// spins; the result is published to the CTA by the caller's __syncthreads.
// A peer that never arrives (a rank that crashed, or calls issued out of order) must not
// hang the device forever: after kPeerTimeoutNs the kernel traps, which surfaces as a CUDA
// error at the caller's next synchronisation ("fail loudly").
constexpr uint64_t kPeerTimeoutNs = 120ull * 1000000000ull;
__device__ __forceinline__ uint64_t global_ns() {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
__device__ __forceinline__ void peer_wait_ge(const uint64_t* slot, uint64_t want) {
    if (ld_acquire_sys_u64(slot) >= want) return;
    const uint64_t t0 = global_ns();
    uint32_t n = 0;
    while (ld_acquire_sys_u64(slot) < want) {
        __nanosleep(64);
        if ((++n & 1023u) == 0u && global_ns() - t0 > kPeerTimeoutNs) __trap();
    }
}
// "Last CTA done" (fence, count, the last one to arrive releases): returns true in
// exactly one CTA per launch, after every CTA's prior stores are visible system-wide.
// The counter resets itself for the next launch (stream-ordered after this one).
__device__ __forceinline__ bool peer_last_cta(uint32_t* counter) {
    __threadfence_system();
    const uint32_t n = gridDim.x;
    if (atomicAdd(counter, 1u) != n - 1) return false;
    *counter = 0;
    __threadfence_system();
    return true;
}

// ------------------------------------------------------------------ Stage 2
// A round of AUX_ITEMS consecutive chunk values per lane: all loads of a round are issued
// together (one memory latency per 32*AUX_ITEMS values instead of per 32), scanned
// serially in registers, then across lanes with shuffles (the tile engine's structure).
constexpr int AUX_ITEMS = 8;

template <class Op>
__device__ __forceinline__ void aux_scan_problem(const ChunkParams& p, int64_t g, int lane, bool push) {
    using C = typename Op::Carry;
    uint64_t* a = p.aux + g * p.Bx;
    C run = Op::cidentity();
    for (int64_t b = 0; b < p.Bx; b += 32 * AUX_ITEMS) {
        const int64_t i0 = b + (int64_t)lane * AUX_ITEMS;
        C v[AUX_ITEMS];
#pragma unroll
        for (int k = 0; k < AUX_ITEMS; ++k) v[k] = i0 + k < p.Bx ? slot_get<C>(a[i0 + k]) : Op::cidentity();
        C t = Op::cidentity();
#pragma unroll
        for (int k = 0; k < AUX_ITEMS; ++k) t = Op::capply(t, v[k]);
        C incl = t;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            C y = shfl_up_c<C>(incl, d);
            if (lane >= d) incl = Op::capply(y, incl);
        }
        C ex = shfl_up_c<C>(incl, 1);
        if (lane == 0) ex = Op::cidentity();
        C r = Op::capply(run, ex);
#pragma unroll
        for (int k = 0; k < AUX_ITEMS; ++k) {
            if (i0 + k < p.Bx) a[i0 + k] = slot_put(r);
            r = Op::capply(r, v[k]);
        }
        run = Op::capply(run, shfl_idx_c<C>(incl, 31));
    }
    if (lane == 0) {
        p.totals[g] = slot_put(run);
        if (push)       // one-sided stores over NVLink into every later rank's mailbox
            for (int q = p.peer.rank + 1; q < p.peer.ngpu; ++q) st_relaxed_sys_u64(p.peer.push_totals[q] + g, slot_put(run));
    }
}

// One CTA per problem, for many chunks per problem (large portions cut into short chunks
// so that concurrently running Stage 1/3 CTAs touch neighbouring memory): the Bx chunk
// values are scanned 32*WARPS at a time (warp shuffles + one smem slot per warp, the same
// block combine as the tile kernels).
template <class Op, int WARPS>
__global__ void __launch_bounds__(WARPS * 32) aux_scan_cta_kernel(ChunkParams p) {
    using C = typename Op::Carry;
    __shared__ __align__(16) C s_w[(WARPS + 3) & ~3];
    const int warp = threadIdx.x >> 5, lane = lane_id();
    const int64_t g = blockIdx.x;
    const PeerParams& pp = p.peer;
    const bool push = pp.on && pp.rank + 1 < pp.ngpu;
    grid_dep_launch();
    grid_dep_wait();
    if (push) {
        if (threadIdx.x == 0 && pp.epoch > 2)
            for (int q = pp.rank + 1; q < pp.ngpu; ++q) peer_wait_ge(pp.my_acks + q, pp.epoch - 2);
        __syncthreads();
    }
    uint64_t* a = p.aux + g * p.Bx;
    C run = Op::cidentity();
    for (int64_t b = 0; b < p.Bx; b += WARPS * 32 * AUX_ITEMS) {
        const int64_t i0 = b + (int64_t)threadIdx.x * AUX_ITEMS;
        C v[AUX_ITEMS];
#pragma unroll
        for (int k = 0; k < AUX_ITEMS; ++k) v[k] = i0 + k < p.Bx ? slot_get<C>(a[i0 + k]) : Op::cidentity();
        C t = Op::cidentity();
#pragma unroll
        for (int k = 0; k < AUX_ITEMS; ++k) t = Op::capply(t, v[k]);
        C incl = t;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            C y = shfl_up_c<C>(incl, d);
            if (lane >= d) incl = Op::capply(y, incl);
        }
        if (lane == 31) s_w[warp] = incl;
        __syncthreads();
        C wp = Op::cidentity(), btot = Op::cidentity();
#pragma unroll 4
        for (int w = 0; w < WARPS; ++w) {
            const C tw = s_w[w];
            if (w < warp) wp = Op::capply(wp, tw);
            btot = Op::capply(btot, tw);
        }
        C ex = shfl_up_c<C>(incl, 1);
        if (lane == 0) ex = Op::cidentity();
        C r = Op::capply(Op::capply(run, wp), ex);
#pragma unroll
        for (int k = 0; k < AUX_ITEMS; ++k) {
            if (i0 + k < p.Bx) a[i0 + k] = slot_put(r);
            r = Op::capply(r, v[k]);
        }
        run = Op::capply(run, btot);
        __syncthreads();
    }
    if (threadIdx.x == 0) {
        p.totals[g] = slot_put(run);
        if (push)
            for (int q = pp.rank + 1; q < pp.ngpu; ++q) st_relaxed_sys_u64(pp.push_totals[q] + g, slot_put(run));
        if (push && peer_last_cta(pp.counters + 0))
            for (int q = pp.rank + 1; q < pp.ngpu; ++q) st_release_sys_u64(pp.push_flag[q], pp.epoch);
    }
}

template <class Op, int WARPS>
__global__ void __launch_bounds__(WARPS * 32) aux_scan_kernel(ChunkParams p) {
    const int warp = threadIdx.x >> 5, lane = lane_id();
    const int64_t g = (int64_t)blockIdx.x * WARPS + warp;
    const PeerParams& pp = p.peer;
    const bool push = pp.on && pp.rank + 1 < pp.ngpu;      // someone reads this rank's totals
    grid_dep_launch();          // Stage 3 may be scheduled now (it loads its data meanwhile)
    grid_dep_wait();            // Stage 1's chunk reductions are complete and visible
    if (push) {
        // the mailbox half this call writes was last read by call epoch-2 of ranks > rank
        if (threadIdx.x == 0 && pp.epoch > 2)
            for (int q = pp.rank + 1; q < pp.ngpu; ++q) peer_wait_ge(pp.my_acks + q, pp.epoch - 2);
        __syncthreads();
    }
    if (g < p.G) aux_scan_problem<Op>(p, g, lane, push);
    if (push) {
        __syncthreads();
        if (threadIdx.x == 0 && peer_last_cta(pp.counters + 0))
            for (int q = pp.rank + 1; q < pp.ngpu; ++q) st_release_sys_u64(pp.push_flag[q], pp.epoch);
    }
}

// ------------------------------------------------------------------ Stage 3 / CTA cascade
template <class Op, int WARPS, int V>
__global__ void __launch_bounds__(WARPS * 32) chunk_scan_kernel(ChunkParams p) {
    using T = typename Op::T;
    using C = typename Op::Carry;
    constexpr int TILE = WARPS * 32 * V * 4, WCH = V * 128;
    static_assert(WARPS % 4 == 0, "warp slots are read as 16-byte vectors");
    __shared__ __align__(16) T s_wval[2][WARPS];
    const int warp = threadIdx.x >> 5, lane = lane_id();
    const int64_t g = (int64_t)blockIdx.x / p.Bx, c = (int64_t)blockIdx.x % p.Bx;
    const int64_t row = g * p.N;
    const int64_t start = c * p.chunk;
    const int64_t end = (start + p.chunk < p.N) ? start + p.chunk : p.N;
    const T* in = (const T*)p.in;
    T* out = (T*)p.out;
    // the next kernel on the stream may be scheduled once every CTA of this grid has
    // started (it waits for this grid's completion before touching memory)
    grid_dep_launch();
    // (no L2 prefetch before the wait here: in large grids it cost the configs[1] step ~1 %,
    //  in one-wave grids it was a wash: profiles/r02_pdl_prefetch_ab.txt)
    if (p.pdl_first) grid_dep_wait();      // a previous call may still be writing our input

    // Stage 2 results folded in: carries of earlier ranks (sharded mode),
    // then the exclusive prefix of the chunks before this one.  Read after
    // the first tile's loads are in flight: launched as a dependent of Stage 2 (p.pdl), the
    // CTA starts while Stage 2 still runs and only grid_dep_wait() orders the reads below.
    auto fold_carry = [&]() -> C {
        grid_dep_wait();
        C carry = Op::cidentity();
        const int64_t stride = p.carry_stride ? p.carry_stride : p.G;
        if (p.peer.on && p.peer.rank > 0) {
            // fused exchange: wait for the totals rows of ranks < rank in this rank's mailbox
            // (pushed by their Stage 2), fold them, and acknowledge once every CTA has read
            __shared__ C s_carry;
            if (threadIdx.x == 0) {
                for (int r = 0; r < p.peer.rank; ++r) peer_wait_ge(p.peer.my_flags + r, p.peer.epoch);
                C cr = Op::cidentity();
                for (int r = 0; r < p.carry_rows; ++r)
                    cr = Op::capply(cr, slot_get<C>(ld_relaxed_sys_u64(p.carry_src + (int64_t)r * stride + g)));
                s_carry = cr;
                if (peer_last_cta(p.peer.counters + 1))
                    for (int r = 0; r < p.peer.rank; ++r) st_release_sys_u64(p.peer.push_ack[r], p.peer.epoch);
            }
            __syncthreads();
            carry = s_carry;
        } else {
            for (int r = 0; r < p.carry_rows; ++r) carry = Op::capply(carry, slot_get<C>(p.carry_src[(int64_t)r * stride + g]));
        }
        if (p.aux && p.aux_raw) {
            // Stage 2 folded into Stage 3 (few chunks per problem): each warp reduces the
            // raw reductions of the chunks before this one itself -- one L2 round trip
            // instead of a third launch
            C pre = Op::cidentity();
            for (int64_t k = lane; k < c; k += 32) pre = Op::capply(pre, slot_get<C>(p.aux[g * p.Bx + k]));
            carry = Op::capply(carry, warp_reduce_carry<Op>(pre));
        } else if (p.aux) {
            carry = Op::capply(carry, slot_get<C>(p.aux[g * p.Bx + c]));
        }
        return carry;
    };
    C carry = Op::cidentity();

    // one tile: scan, block combine, store with the running carry (the cascade, Fig. 5)
    auto process = [&](WarpTile<Op, false, V>& wt, int64_t off, int it) {
        const int64_t wb = row + off + warp * WCH;
        if (it == 0) carry = fold_carry();
        wt.scan();
        if (lane == 0) s_wval[it & 1][warp] = wt.wtot;
        __syncthreads();
        // the WARPS slots of this tile's buffer, read as exactly WARPS/4 16-byte vectors
        // (double-buffered by tile parity: one barrier per tile; slot it&1 is rewritten in
        // tile it+2, after barrier it+1, which every warp reaches after these reads)
        T wv[WARPS];
#pragma unroll
        for (int q = 0; q < WARPS / 4; ++q) {
            uint4 u;
            asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];"
                         : "=r"(u.x), "=r"(u.y), "=r"(u.z), "=r"(u.w)
                         : "r"(smem_u32(&s_wval[it & 1][4 * q])) : "memory");
            wv[4 * q] = from_bits<T>(u.x); wv[4 * q + 1] = from_bits<T>(u.y);
            wv[4 * q + 2] = from_bits<T>(u.z); wv[4 * q + 3] = from_bits<T>(u.w);
        }
        T wp = Op::identity(), tot = Op::identity();
#pragma unroll
        for (int w = 0; w < WARPS; ++w) {
            if (w < warp) wp = Op::apply(wp, wv[w]);
            tot = Op::apply(tot, wv[w]);
        }
        wt.store(out, wb, row + end, p.vec, wp, false, Op::from_carry(carry), p.exclusive);
        carry = Op::capply(carry, Op::to_carry(tot));
    };
    // software pipeline over the chunk's tiles: the loads of tile i+1 are issued before
    // tile i is scanned, so every thread keeps two tiles' rows in flight (ping-pong
    // registers A/B, compile-time indexed)
    WarpTile<Op, false, V> A, B;
    int it = 0;
    int64_t off = start;
    if (off < end) A.load(in, row + off + warp * WCH, row + end, p.vec);
    while (off < end) {
        if (off + TILE < end) B.load(in, row + off + TILE + warp * WCH, row + end, p.vec);
        process(A, off, it++);
        off += TILE;
        if (off >= end) break;
        if (off + TILE < end) A.load(in, row + off + TILE + warp * WCH, row + end, p.vec);
        process(B, off, it++);
        off += TILE;
    }
}

// ------------------------------------------------------------------ warp-per-problem cascade
template <class Op, int WARPS, int V>
__global__ void __launch_bounds__(WARPS * 32) warp_cascade_kernel(ChunkParams p) {
    using T = typename Op::T;
    using C = typename Op::Carry;
    constexpr int WCH = V * 128;
    const int warp = threadIdx.x >> 5;
    const int64_t g = (int64_t)blockIdx.x * WARPS + warp;
    grid_dep_launch();
    if (p.pdl_first) grid_dep_wait();      // cross-call programmatic launch (ChunkParams)
    if (g >= p.G) return;
    const int64_t row = g * p.N;
    const T* in = (const T*)p.in;
    T* out = (T*)p.out;
    C carry = Op::cidentity();
    const int64_t stride = p.carry_stride ? p.carry_stride : p.G;
    for (int r = 0; r < p.carry_rows; ++r) carry = Op::capply(carry, slot_get<C>(p.carry_src[(int64_t)r * stride + g]));
    for (int64_t off = 0; off < p.N; off += WCH) {
        WarpTile<Op, false, V> wt;
        wt.load(in, row + off, row + p.N, p.vec);
        wt.scan();
        wt.store(out, row + off, row + p.N, p.vec, Op::identity(), false, Op::from_carry(carry), p.exclusive);
        carry = Op::capply(carry, Op::to_carry(wt.wtot));
    }
}

// ------------------------------------------------------------------ warp per problem, sharded path
// Short portions (N_local <= 4096, one chunk per problem, many problems): Stage 1 and
// Stage 3 of the sharded pipeline with one WARP per problem
// instead of one 256-thread CTA per (problem, chunk), which left most of each CTA idle
// (N_local = 1024: Stage 1 0.33, Stage 3 0.28 of copy; profiles/r02_mps_phases_W1.jsonl).
// Stages 1+2 in one kernel: with one chunk per problem Stage 2 is the identity on the chunk
// prefixes and only copies each problem's total out (and pushes it to the later ranks'
// mailboxes) -- a separate aux_scan launch of G/8 CTAs cost 60 us at G = 2^18 for 2 MB, so
// the warp stores its total directly with aux_scan_kernel's exchange protocol (wait for the
// acks of call epoch-2 before overwriting a mailbox half; the last CTA raises the flags).
template <class Op, int WARPS, int V>
__global__ void __launch_bounds__(WARPS * 32) warp_reduce_kernel(ChunkParams p) {
    using T = typename Op::T;
    using C = typename Op::Carry;
    constexpr int WCH = V * 128;
    const int warp = threadIdx.x >> 5, lane = lane_id();
    const int64_t g = (int64_t)blockIdx.x * WARPS + warp;
    const bool live = g < p.G;
    const PeerParams& pp = p.peer;
    const bool push = pp.on && pp.rank + 1 < pp.ngpu;      // someone reads this rank's totals
    if (p.pdl_first) grid_dep_wait();      // the library's ordering rule (chunk_reduce_kernel)
    grid_dep_launch();
    C acc = Op::cidentity();
    if (live) {
        const int64_t row = g * p.N;
        const T* in = (const T*)p.in;
        for (int64_t off = 0; off < p.N; off += WCH) {
            Row4<T> x[V];
#pragma unroll
            for (int j = 0; j < V; ++j) x[j] = load_row<Op>(in, row + off + j * 128 + lane * 4, row + p.N, p.vec);
            T t = Op::identity();
#pragma unroll
            for (int j = 0; j < V; ++j)
#pragma unroll
                for (int k = 0; k < 4; ++k) t = Op::apply(t, x[j].v[k]);
            acc = Op::capply(acc, Op::to_carry(t));
        }
        acc = warp_reduce_carry<Op>(acc);
    }
    if (push) {
        // the mailbox half this call writes was last read by call epoch-2 of ranks > rank
        if (threadIdx.x == 0 && pp.epoch > 2)
            for (int q = pp.rank + 1; q < pp.ngpu; ++q) peer_wait_ge(pp.my_acks + q, pp.epoch - 2);
        __syncthreads();
    }
    if (live && lane == 0) {
        p.totals[g] = slot_put(acc);
        if (push)
            for (int q = pp.rank + 1; q < pp.ngpu; ++q) st_relaxed_sys_u64(pp.push_totals[q] + g, slot_put(acc));
    }
    if (push) {
        __syncthreads();
        if (threadIdx.x == 0 && peer_last_cta(pp.counters + 0))
            for (int q = pp.rank + 1; q < pp.ngpu; ++q) st_release_sys_u64(pp.push_flag[q], pp.epoch);
    }
}

// Stage 3: carry = the totals of the ranks before this one (fused exchange: wait for their
// rows in this rank's mailbox, then acknowledge once every CTA has read -- as
// chunk_scan_kernel's fold_carry), then the warp cascade over the problem.  With one chunk
// per problem the chunk prefix of Stage 2 is the identity.  Launched as a dependent of
// Stage 2: waits for it before any access.
template <class Op, int WARPS, int V>
__global__ void __launch_bounds__(WARPS * 32) warp_shard_scan_kernel(ChunkParams p) {
    using T = typename Op::T;
    using C = typename Op::Carry;
    constexpr int WCH = V * 128;
    const int warp = threadIdx.x >> 5, lane = lane_id();
    const int64_t g = (int64_t)blockIdx.x * WARPS + warp;
    const bool live = g < p.G;
    grid_dep_launch();
    grid_dep_wait();
    C carry = Op::cidentity();
    const int64_t stride = p.carry_stride ? p.carry_stride : p.G;
    const bool peer_wait = p.peer.on && p.peer.rank > 0;
    if (peer_wait) {
        if (live && lane == 0) {
            for (int r = 0; r < p.peer.rank; ++r) peer_wait_ge(p.peer.my_flags + r, p.peer.epoch);
            for (int r = 0; r < p.carry_rows; ++r)
                carry = Op::capply(carry, slot_get<C>(ld_relaxed_sys_u64(p.carry_src + (int64_t)r * stride + g)));
        }
        carry = shfl_idx_c<C>(carry, 0);
    } else if (live) {
        for (int r = 0; r < p.carry_rows; ++r) carry = Op::capply(carry, slot_get<C>(p.carry_src[(int64_t)r * stride + g]));
    }
    if (live) {
        const int64_t row = g * p.N;
        const T* in = (const T*)p.in;
        T* out = (T*)p.out;
        for (int64_t off = 0; off < p.N; off += WCH) {
            WarpTile<Op, false, V> wt;
            wt.load(in, row + off, row + p.N, p.vec);
            wt.scan();
            wt.store(out, row + off, row + p.N, p.vec, Op::identity(), false, Op::from_carry(carry), p.exclusive);
            carry = Op::capply(carry, Op::to_carry(wt.wtot));
        }
    }
    if (peer_wait) {
        __syncthreads();                   // every warp of the CTA has read its mailbox row
        if (threadIdx.x == 0 && peer_last_cta(p.peer.counters + 1))
            for (int r = 0; r < p.peer.rank; ++r) st_release_sys_u64(p.peer.push_ack[r], p.peer.epoch);
    }
}

// ------------------------------------------------------------------ packed short problems
// Several whole problems per warp (L_x < 32 threads per problem): warp w owns
// problems [w*k, (w+1)*k) -- one contiguous span of k*N elements that starts and ends on
// problem boundaries, 16-byte aligned (k*N % 4 == 0, chosen on the host) -- and walks it in
// V*128-element windows with a SEGMENTED scan (heads every N elements).  No carry crosses
// a span, so there is no inter-warp dependency at all; inside the span the segmented carry
// runs from window to window (a head resets it).
template <class Op, int WARPS, int V, bool EXCL>
__global__ void __launch_bounds__(WARPS * 32) packed_warp_kernel(ChunkParams p) {
    using T = typename Op::T;
    using C = typename Op::Carry;
    constexpr int WCH = V * 128;
    const int warp = threadIdx.x >> 5, lane = lane_id();
    const int64_t k = p.chunk;                       // problems per span
    const int64_t g0 = ((int64_t)blockIdx.x * WARPS + warp) * k;
    grid_dep_launch();
    if (p.pdl_first) grid_dep_wait();
    if (g0 >= p.G) return;
    const int64_t base = g0 * p.N;
    const int64_t end = min(g0 + k, p.G) * p.N;
    const T* in = (const T*)p.in;
    T* out = (T*)p.out;
    const uint32_t N32 = (uint32_t)p.N;
    // position of this lane's row inside its problem, advanced by 128 mod N per row (one
    // compare-subtract instead of a division per row)
    const uint32_t step = 128u % N32;
    uint32_t r = (uint32_t)(lane * 4) % N32;
    C carry = Op::cidentity();                       // segmented: value since the last head
    for (int64_t off = base; off < end; off += WCH) {
        Row4<T> x[V];                                // the whole window in flight at once
#pragma unroll
        for (int j = 0; j < V; ++j) x[j] = load_row<Op>(in, off + j * 128 + lane * 4, end, p.vec);
        // then row by row: only the running carry lives across rows (few registers)
#pragma unroll
        for (int j = 0; j < V; ++j) {
            const unsigned hd = row_heads_from_r(r, N32);
            r += step;
            if (r >= N32) r -= N32;
            T v = row_reduce<Op, true>(x[j], hd);
            const unsigned hm = __ballot_sync(FULL, hd != 0u);
            T lin; bool lfl;
            T incl = warp_seg_scan<Op, true>(v, hm, lin, lfl);
            T rt = shfl_idx<T>(incl, 31);
            store_row<Op>(out, off + j * 128 + lane * 4, end, p.vec,
                          row_output<Op, true, EXCL>(x[j], hd, lin, lfl, Op::from_carry(carry)));
            carry = hm ? Op::to_carry(rt) : Op::capply(carry, Op::to_carry(rt));
        }
    }
}

// Power-of-two N <= 512 (the paper's problem sizes): every V*128-element
// window of the flat array holds whole problems, so warp w simply owns window w and the
// segment structure is regular -- no head flags, no ballots:
//   N <= 4        a problem lies inside one lane's 4-element row: serial, resets in-lane;
//   8 <= N <= 128 a problem spans L = N/4 lanes: sub-warp scan (shfl.up, segments of L);
//   N >= 256      a problem spans R = N/128 rows: full-warp scan per row, the row carry
//                 resets every R rows.
template <class Op>
__device__ __forceinline__ typename Op::T shfl_up_w(typename Op::T v, int d, int width) {
    return from_bits<typename Op::T>(__shfl_up_sync(FULL, to_bits<typename Op::T>(v), d, width));
}
template <class Op, int WARPS, int V, bool EXCL>
__global__ void __launch_bounds__(WARPS * 32) packed_pow2_kernel(ChunkParams p) {
    using T = typename Op::T;
    constexpr int WCH = V * 128;
    const int warp = threadIdx.x >> 5, lane = lane_id();
    const int64_t base = ((int64_t)blockIdx.x * WARPS + warp) * WCH;
    const int64_t total = p.N * p.G;
    grid_dep_launch();
    if (p.pdl_first) grid_dep_wait();
    if (base >= total) return;
    const T* in = (const T*)p.in;
    T* out = (T*)p.out;
    const int n = (int)p.N;
    Row4<T> x[V];
#pragma unroll
    for (int j = 0; j < V; ++j) x[j] = load_row<Op>(in, base + j * 128 + lane * 4, total, p.vec);
    if (n <= 4) {
        const unsigned hd = n == 1 ? 0xFu : n == 2 ? 0x5u : 0x1u;
#pragma unroll
        for (int j = 0; j < V; ++j)
            store_row<Op>(out, base + j * 128 + lane * 4, total, p.vec,
                          row_output<Op, true, EXCL>(x[j], hd, Op::identity(), true, Op::identity()));
    } else if (n <= 128) {
        const int L = n >> 2;                       // lanes per problem
        const int sl = lane & (L - 1);              // lane index inside its problem
#pragma unroll
        for (int j = 0; j < V; ++j) {
            T v = row_reduce<Op, false>(x[j], 0u);
            for (int d = 1; d < L; d <<= 1) {
                T y = shfl_up_w<Op>(v, d, L);
                if (sl >= d) v = Op::apply(y, v);
            }
            T e = shfl_up_w<Op>(v, 1, L);
            if (sl == 0) e = Op::identity();
            store_row<Op>(out, base + j * 128 + lane * 4, total, p.vec,
                          row_output<Op, false, EXCL>(x[j], 0u, e, false, Op::identity()));
        }
    } else {
        const int R = n >> 7;                       // rows per problem (2 or 4)
        T run = Op::identity();
#pragma unroll
        for (int j = 0; j < V; ++j) {
            T v = row_reduce<Op, false>(x[j], 0u);
            T e; bool ef;
            T incl = warp_seg_scan<Op, false>(v, 0u, e, ef);
            T rt = shfl_idx<T>(incl, 31);
            if ((j & (R - 1)) == 0) run = Op::identity();
            store_row<Op>(out, base + j * 128 + lane * 4, total, p.vec,
                          row_output<Op, false, EXCL>(x[j], 0u, Op::apply(run, e), false, Op::identity()));
            run = Op::apply(run, rt);
        }
    }
}

// fused exchange, empty local portion: wait for ranks < rank, acknowledge them
__global__ void peer_ack_kernel(PeerParams pp) {
    if (threadIdx.x != 0) return;
    for (int r = 0; r < pp.rank; ++r) peer_wait_ge(pp.my_flags + r, pp.epoch);
    __threadfence_system();
    for (int r = 0; r < pp.rank; ++r) st_release_sys_u64(pp.push_ack[r], pp.epoch);
}

// launch, as a programmatic dependent of the stream's previous kernel when p.pdl
template <class Kern>
cudaError_t launch_maybe_pdl(Kern kern, unsigned blocks, unsigned threads, const ChunkParams& p, cudaStream_t s) {
    if (!p.pdl) {
        kern<<<blocks, threads, 0, s>>>(p);
        return cudaGetLastError();
    }
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(blocks);
    cfg.blockDim = dim3(threads);
    cfg.dynamicSmemBytes = 0;
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, kern, p);
}
template <class Op>
cudaError_t reduce_op(const ChunkParams& p, cudaStream_t s) {
    int64_t blocks = p.G * p.Bx;
    if (blocks == 0) return cudaSuccess;
    if (blocks > 0x7FFFFFFF) return cudaErrorInvalidConfiguration;
    return launch_maybe_pdl(chunk_reduce_kernel<Op, CH_WARPS, CH_V>, (unsigned)blocks, CH_WARPS * 32, p, s);
}
template <class Op>
cudaError_t auxscan_op(const ChunkParams& p, cudaStream_t s) {
    if (p.Bx > 32 * AUX_ITEMS) {    // many chunks per problem: a CTA per problem
        if (p.G > 0x7FFFFFFF) return cudaErrorInvalidConfiguration;
        return launch_maybe_pdl(aux_scan_cta_kernel<Op, 32>, (unsigned)p.G, 32 * 32, p, s);
    }
    int64_t blocks = (p.G + 7) / 8;
    if (blocks == 0) return cudaSuccess;
    return launch_maybe_pdl(aux_scan_kernel<Op, 8>, (unsigned)blocks, 8 * 32, p, s);
}
template <class Op>
cudaError_t scan_op(const ChunkParams& p, cudaStream_t s) {
    int64_t blocks = p.G * p.Bx;
    if (blocks == 0) return cudaSuccess;
    if (blocks > 0x7FFFFFFF) return cudaErrorInvalidConfiguration;
    return launch_maybe_pdl(chunk_scan_kernel<Op, CH_WARPS, CH_V>, (unsigned)blocks, CH_WARPS * 32, p, s);
}
template <class Op>
cudaError_t warp_op(const ChunkParams& p, cudaStream_t s) {
    int64_t blocks = (p.G + WC_WARPS - 1) / WC_WARPS;
    if (blocks > 0x7FFFFFFF) return cudaErrorInvalidConfiguration;
    if (blocks == 0) return cudaSuccess;
    return launch_maybe_pdl(warp_cascade_kernel<Op, WC_WARPS, WC_V>, (unsigned)blocks, WC_WARPS * 32, p, s);
}
template <class Op>
cudaError_t warp_reduce_op(const ChunkParams& p, cudaStream_t s) {
    int64_t blocks = (p.G + WC_WARPS - 1) / WC_WARPS;
    if (blocks > 0x7FFFFFFF) return cudaErrorInvalidConfiguration;
    if (blocks == 0) return cudaSuccess;
    return launch_maybe_pdl(warp_reduce_kernel<Op, WC_WARPS, WC_V>, (unsigned)blocks, WC_WARPS * 32, p, s);
}
template <class Op>
cudaError_t warp_shard_scan_op(const ChunkParams& p, cudaStream_t s) {
    int64_t blocks = (p.G + WC_WARPS - 1) / WC_WARPS;
    if (blocks > 0x7FFFFFFF) return cudaErrorInvalidConfiguration;
    if (blocks == 0) return cudaSuccess;
    return launch_maybe_pdl(warp_shard_scan_kernel<Op, WC_WARPS, WC_V>, (unsigned)blocks, WC_WARPS * 32, p, s);
}
template <class Op>
cudaError_t packed_op(const ChunkParams& p, cudaStream_t s) {
    const bool pow2 = p.N > 0 && p.N <= 512 && (p.N & (p.N - 1)) == 0;
    if (pow2 && p.vec) {                                   // regular segments, one window per warp
        constexpr int WCH = WC_V * 128;
        const int64_t windows = (p.N * p.G + WCH - 1) / WCH;
        const int64_t blocks = (windows + WC_WARPS - 1) / WC_WARPS;
        if (blocks == 0) return cudaSuccess;
        if (blocks > 0x7FFFFFFF) return cudaErrorInvalidConfiguration;
        return p.exclusive ? launch_maybe_pdl(packed_pow2_kernel<Op, WC_WARPS, WC_V, true>, (unsigned)blocks, WC_WARPS * 32, p, s)
                           : launch_maybe_pdl(packed_pow2_kernel<Op, WC_WARPS, WC_V, false>, (unsigned)blocks, WC_WARPS * 32, p, s);
    }
    const int64_t spans = (p.G + p.chunk - 1) / p.chunk;
    const int64_t blocks = (spans + WC_WARPS - 1) / WC_WARPS;
    if (blocks == 0) return cudaSuccess;
    if (blocks > 0x7FFFFFFF) return cudaErrorInvalidConfiguration;
    return p.exclusive ? launch_maybe_pdl(packed_warp_kernel<Op, WC_WARPS, WC_V, true>, (unsigned)blocks, WC_WARPS * 32, p, s)
                       : launch_maybe_pdl(packed_warp_kernel<Op, WC_WARPS, WC_V, false>, (unsigned)blocks, WC_WARPS * 32, p, s);
}

#define SCANB200_DISPATCH(fn)                                          \
    switch (op) {                                                      \
    case OpCode::AddU32: return fn<OpAddU32>(p, s);                    \
    case OpCode::MaxI32: return fn<OpMaxI32>(p, s);                    \
    case OpCode::MaxU32: return fn<OpMaxU32>(p, s);                    \
    case OpCode::MaxF32: return fn<OpMaxF32>(p, s);                    \
    case OpCode::AddF32: return fn<OpAddF32>(p, s);                    \
    }                                                                  \
    return cudaErrorInvalidValue;

}  // namespace

int64_t chunk_tile_elems() { return CH_WARPS * 32 * CH_V * 4; }
int64_t warp_tile_elems() { return WC_V * 128; }

cudaError_t launch_chunk_reduce(OpCode op, const ChunkParams& p, cudaStream_t s) { SCANB200_DISPATCH(reduce_op) }
cudaError_t launch_aux_scan(OpCode op, const ChunkParams& p, cudaStream_t s) { SCANB200_DISPATCH(auxscan_op) }
cudaError_t launch_chunk_scan(OpCode op, const ChunkParams& p, cudaStream_t s) { SCANB200_DISPATCH(scan_op) }
cudaError_t launch_warp_cascade(OpCode op, const ChunkParams& p, cudaStream_t s) { SCANB200_DISPATCH(warp_op) }
cudaError_t launch_warp_reduce(OpCode op, const ChunkParams& p, cudaStream_t s) { SCANB200_DISPATCH(warp_reduce_op) }
cudaError_t launch_warp_shard_scan(OpCode op, const ChunkParams& p, cudaStream_t s) { SCANB200_DISPATCH(warp_shard_scan_op) }
cudaError_t launch_packed_warp(OpCode op, const ChunkParams& p, cudaStream_t s) { SCANB200_DISPATCH(packed_op) }
cudaError_t launch_peer_ack(const PeerParams& pp, cudaStream_t s) {
    if (!pp.on || pp.rank == 0) return cudaSuccess;
    peer_ack_kernel<<<1, 32, 0, s>>>(pp);
    return cudaGetLastError();
}

}  // namespace scanb200
