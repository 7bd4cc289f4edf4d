// scan_lookback.cu -- single-pass batched scan with decoupled look-back (sm_100a).
//
// The paper solves large problems with three kernels (Chunk Reduce -> Intermediate Scan ->
// Scan+Addition, PAPER.md:110-118 [§3.1, Fig. 3]), i.e. 3N element transfers, and notes
// that its Stage 2 leaves the GPU "underused" at G=1.  On one B200 the
// byte-optimal schedule is single pass (2N transfers): each tile publishes its aggregate
// as soon as it has it and looks back over its predecessors' published values, the
// barrier-free idea of StreamScan [25] that the paper cites.  The
// three-stage form is kept in scan_three_stage.cu (deterministic mode + sharded path).
//
// The G problems of N elements are scanned as ONE flat array of G*N elements
// cut into tiles of WARPS*32*V*4 elements; a tile that contains a problem start publishes
// its (trailing-segment) inclusive value immediately, so every look-back stops at the
// problem it belongs to and no carry crosses problems.  Small N therefore costs no extra
// launches and rows need not be 16-byte aligned (only the base pointers).
//
// Descriptor protocol (per tile t, reset-free thanks to a 30-bit epoch tag):
//   packed (32-bit carries): u64 = value<<32 | tag<<2 | status   (status 0 X, 1 A, 2 P)
//   split  (f32 add, fp64 carries): u64 tag<<2|status + f64 aggregate[t] + f64 inclusive[t];
//          the value is written first, the status with st.release; readers ld.acquire.
// Tiles are numbered by an atomic ticket in CTA start order (forward progress: every tile
// a CTA waits on belongs to a CTA that already started).  The last CTA to finish resets
// the ticket and done counters and advances the epoch, so consecutive launches (also CUDA
// graph replays) need no memset.
#include "scan_common.cuh"
#include "scan_internal.h"

namespace scanb200 {

namespace {

constexpr uint32_t ST_A = 1u, ST_P = 2u;
constexpr uint32_t TAG_MASK = 0x3FFFFFFFu;

template <class Op>
struct Desc {
    using C = typename Op::Carry;
    static __device__ __forceinline__ void publish(const LookbackParams& p, int64_t t, uint32_t tag,
                                                   uint32_t st, C v) {
        if constexpr (Op::kSplitDesc) {
            st_relaxed_f64((st == ST_P ? p.incl : p.agg) + t, v);
            st_release_u64(p.desc + t, (uint64_t)((tag << 2) | st));
        } else {
            uint64_t w = ((uint64_t)to_bits<C>(v) << 32) | (uint64_t)((tag << 2) | st);
            st_release_u64(p.desc + t, w);
        }
    }
    // returns status (0 when stale / not yet written) and the matching value
    static __device__ __forceinline__ uint32_t read(const LookbackParams& p, int64_t t, uint32_t tag, C& v) {
        if constexpr (Op::kSplitDesc) {
            uint64_t w = ld_acquire_u64(p.desc + t);
            uint32_t s = (uint32_t)w;
            if ((s >> 2) != tag || (w >> 32) != 0ull) return 0u;
            uint32_t st = s & 3u;
            v = ld_relaxed_f64((st == ST_P ? p.incl : p.agg) + t);
            return st;
        } else {
            uint64_t w = ld_acquire_u64(p.desc + t);
            if ((((uint32_t)w) >> 2) != tag) return 0u;
            v = from_bits<C>((uint32_t)(w >> 32));
            return (uint32_t)w & 3u;
        }
    }
};

// Warp-cooperative look-back for tile `t` (t > first tile of its problem).  Lane i inspects
// predecessor t-1-i; the window slides back 32 tiles at a time until an inclusive (P)
// descriptor is found.  Only the lanes up to the nearest P are waited for.
template <class Op>
__device__ __forceinline__ typename Op::Carry look_back(const LookbackParams& p, int64_t t, uint32_t tag) {
    using C = typename Op::Carry;
    const int lane = lane_id();
    C run = Op::cidentity();
    int64_t pred = t - 1 - lane;
    while (true) {
        C v = Op::cidentity();
        uint32_t st;
        unsigned pm;
        int fp;
        int spins = 0;
        while (true) {
            st = pred >= 0 ? Desc<Op>::read(p, pred, tag, v) : ST_P;   // (never needed: tile 0 starts a problem)
            pm = __ballot_sync(FULL, st == ST_P);
            unsigned xm = __ballot_sync(FULL, st == 0u);
            fp = pm ? (__ffs(pm) - 1) : 32;
            unsigned need = fp >= 32 ? FULL : ((1u << fp) - 1u);
            if ((xm & need) == 0u) break;
            if (++spins > 4) __nanosleep(64);
        }
        C mine = (lane <= fp && pred >= 0) ? v : Op::cidentity();
        C w = warp_reduce_carry<Op>(mine);
        run = Op::capply(w, run);          // the window is older than what we have so far
        if (pm) break;
        pred -= 32;
    }
    return run;
}

template <class Op, bool SEG, int WARPS, int V>
__device__ __forceinline__ void tile_body(const LookbackParams& p, int64_t tile, uint32_t tag,
                                          int64_t r, typename Op::Carry* s_carry,
                                          typename Op::T* s_wval, uint32_t* s_wflag) {
    using T = typename Op::T;
    using C = typename Op::Carry;
    constexpr int TILE = WARPS * 32 * V * 4;
    constexpr int WCH = V * 128;
    const int warp = threadIdx.x >> 5, lane = lane_id();
    const int64_t base = tile * (int64_t)TILE;
    const int64_t wbase = base + warp * WCH;
    const T* in = (const T*)p.in;
    T* out = (T*)p.out;

    WarpTile<Op, SEG, V> wt;
    wt.load(in, wbase, p.total, p.vec);
    if (SEG) {
        const bool small = p.N < TILE;
        int first = -1;
        if (!small) first = r == 0 ? 0 : (int)(p.N - r);      // < TILE: SEG implies a head in the tile
        wt.heads(warp * WCH, small, (uint32_t)(small ? r : 0), (uint32_t)(small ? p.N : 1), first);
    }
    wt.scan();
    if (lane == 0) { s_wval[warp] = wt.wtot; s_wflag[warp] = wt.wfl; }
    __syncthreads();

    T wp = Op::identity(); bool wpf = false;
#pragma unroll
    for (int w = 0; w < WARPS; ++w) {
        if (w < warp) {
            T v = s_wval[w]; bool f = SEG && s_wflag[w];
            wp = SEG ? seg_fold<Op>(wp, f, v) : Op::apply(wp, v);
            wpf = wpf || f;
        }
    }

    if (warp == WARPS - 1) {
        // tile aggregate = (warps < last) . (last warp)
        T agg = SEG ? seg_fold<Op>(wp, wt.wfl, wt.wtot) : Op::apply(wp, wt.wtot);
        const bool starts = (r == 0);
        const bool has_head = SEG ? (wpf || wt.wfl) : starts;
        const C aggc = Op::to_carry(agg);
        if (lane == 0) Desc<Op>::publish(p, tile, tag, has_head ? ST_P : ST_A, aggc);
        C carry = Op::cidentity();
        if (!starts) carry = look_back<Op>(p, tile, tag);
        if (lane == 0) {
            if (!has_head) Desc<Op>::publish(p, tile, tag, ST_P, Op::capply(carry, aggc));
            *s_carry = carry;
        }
    }
    __syncthreads();
    const T cin = Op::from_carry(*s_carry);
    wt.store(out, wbase, p.total, p.vec, wp, wpf, cin, p.exclusive);
}

template <class Op, int WARPS, int V>
__global__ void __launch_bounds__(WARPS * 32) lookback_kernel(LookbackParams p) {
    using T = typename Op::T;
    using C = typename Op::Carry;
    constexpr int TILE = WARPS * 32 * V * 4;
    __shared__ int64_t s_tile, s_r;
    __shared__ uint32_t s_tag, s_seg;
    __shared__ C s_carry;
    __shared__ T s_wval[WARPS];
    __shared__ uint32_t s_wflag[WARPS];
    __shared__ int s_last;

    if (threadIdx.x == 0) {
        int64_t t = (int64_t)atomicAdd(p.ctl + 0, 1u);
        uint32_t e;
        asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(e) : "l"(p.ctl + 2) : "memory");
        int64_t base = t * (int64_t)TILE;
        int64_t r = base % p.N;
        int64_t count = p.total - base < TILE ? p.total - base : TILE;
        int64_t next_head = r == 0 ? p.N : p.N - r;          // first head after offset 0
        s_tile = t; s_r = r; s_tag = (e + 1u) & TAG_MASK;
        s_seg = next_head < count ? 1u : 0u;
    }
    __syncthreads();
    const int64_t tile = s_tile, r = s_r;
    const uint32_t tag = s_tag;
    if (s_seg) tile_body<Op, true, WARPS, V>(p, tile, tag, r, &s_carry, s_wval, s_wflag);
    else       tile_body<Op, false, WARPS, V>(p, tile, tag, r, &s_carry, s_wval, s_wflag);

    // ---- self-cleaning epilogue: the last CTA resets the counters and advances the epoch
    if (threadIdx.x == 0) {
        __threadfence();
        uint32_t prev = atomicAdd(p.ctl + 1, 1u);
        s_last = (prev == gridDim.x - 1) ? 1 : 0;
        if (s_last) {
            __threadfence();
            uint32_t e = *((volatile uint32_t*)(p.ctl + 2)) + 1u;
            bool wrap = e + 1u >= TAG_MASK;
            if (wrap) {
                // once every 2^30 launches: invalidate every descriptor ever written
                for (int64_t i = 0; i < p.capacity; ++i) p.desc[i] = 0ull;
                e = 0u;
            }
            ((volatile uint32_t*)p.ctl)[0] = 0u;
            ((volatile uint32_t*)p.ctl)[1] = 0u;
            ((volatile uint32_t*)p.ctl)[2] = e;
            __threadfence();
        }
    }
}

template <class Op, int WARPS, int V>
cudaError_t launch_variant(const LookbackParams& p, cudaStream_t s) {
    constexpr int TILE = WARPS * 32 * V * 4;
    int64_t tiles = (p.total + TILE - 1) / TILE;
    if (tiles > 0x7FFFFFFF) return cudaErrorInvalidConfiguration;
    lookback_kernel<Op, WARPS, V><<<(unsigned)tiles, WARPS * 32, 0, s>>>(p);
    return cudaGetLastError();
}

template <class Op>
cudaError_t launch_op(const LookbackParams& p, int variant, cudaStream_t s) {
    switch (variant) {
    case 0: return launch_variant<Op, 8, 4>(p, s);     // 4096-element tiles
    case 1: return launch_variant<Op, 8, 8>(p, s);     // 8192-element tiles
    default: return launch_variant<Op, 16, 4>(p, s);   // 8192-element tiles, 16 warps
    }
}

}  // namespace

int64_t lookback_tile_elems(int variant) {
    switch (variant) {
    case 0: return 8 * 32 * 4 * 4;
    case 1: return 8 * 32 * 8 * 4;
    default: return 16 * 32 * 4 * 4;
    }
}

cudaError_t launch_lookback(OpCode op, const LookbackParams& p, int variant, cudaStream_t s) {
    switch (op) {
    case OpCode::AddU32: return launch_op<OpAddU32>(p, variant, s);
    case OpCode::MaxI32: return launch_op<OpMaxI32>(p, variant, s);
    case OpCode::MaxU32: return launch_op<OpMaxU32>(p, variant, s);
    case OpCode::MaxF32: return launch_op<OpMaxF32>(p, variant, s);
    case OpCode::AddF32: return launch_op<OpAddF32>(p, variant, s);
    }
    return cudaErrorInvalidValue;
}

}  // namespace scanb200
