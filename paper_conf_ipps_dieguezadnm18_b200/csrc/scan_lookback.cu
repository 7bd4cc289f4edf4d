// scan_lookback.cu -- single-pass batched scan with decoupled look-back (sm_100a).
//
// The paper solves large problems with three kernels (Chunk Reduce -> Intermediate Scan ->
// Scan+Addition, PAPER.md:110-118 [§3.1, Fig. 3]), i.e. 3N element transfers, and notes
// that its Stage 2 leaves the GPU "underused" at G=1.  On one B200 the
// byte-optimal schedule is single pass (2N transfers): each tile publishes its aggregate
// as soon as it has it and looks back over its predecessors' published values -- the
// barrier-free idea of StreamScan [25] that the paper cites.  The
// three-stage form is kept in scan_chunked.cu (deterministic mode + sharded path).
//
// The G problems of N elements are scanned as ONE flat array of G*N elements
// cut into tiles; a tile that contains a problem start publishes its (trailing-segment)
// inclusive value immediately, so every look-back stops inside its own problem and no
// carry crosses problems.  Small N costs no extra launches and rows need not be 16-byte
// aligned (only the base pointers).
//
// Variants (scan_batch_ex `param`; AUTO uses 1, 2 and 3, scan_autotune also tries 0, 10):
//   3  lookback_l2_kernel -- the default for few large problems (G*N >= 2^22), configs[2]:
//      persistent, one CTA per SM, tiles of 8192 elements (32 KiB) assigned round robin
//      (tile = cta + k * grid, launched cooperatively so the whole grid is co-resident);
//      every tile is read TWICE but from HBM once: read 1 (TMA bulk copy into a smem ring,
//      SASS UBLKCP) feeds 8 reducer warps that publish the tile aggregate (A) at once and
//      free the slot; 2 look-back warps resolve the carry LAZILY (from the tile's own A
//      on: the window of the grid - 1 predecessors is loaded in one round trip and the CTA's
//      own previous tile supplies the inclusive prefix from shared memory) while the data
//      waits in L2; read 2 (L2 -> smem) feeds 8 scanner warps that add the carry and store
//      (the CTA's last two tiles are scanned from their read-1 slots).  The next round's read 1 is
//      L2-prefetched (UBLKPF).  ~100 % of measured copy from 2^27 on, 0.82 / 0.90 at 2^24 / 2^25.
//   0/1 lookback_pipelined_kernel -- persistent, one read: a producer warp streams 64 / 32
//      KiB tiles into a 3-slot TMA ring, 16 / 8 consumer warps scan each staged tile in two
//      passes, a dedicated look-back warp resolves the carry (window of 160 / 128 tiles);
//      the tile holds its smem slot until its carry arrives (Little's law: ~85-91 % of
//      copy for one huge problem).  1 = the AUTO choice for small totals (< 2^22).
//   2  lookback_tma_kernel -- one 8192-element tile per CTA in blockIdx order (in-order
//      dispatch: every tile a CTA waits on belongs to a running CTA); short / unaligned rows.
//   10 lookback_regtile_kernel -- one 8192-element register tile per CTA (no smem staging).
// Measured limits (tools/trace_lookback.py): a descriptor round trip costs
// ~2 us under full HBM load; the L2-staged form keeps the waiting data in L2, not smem.
//
// Descriptors (one per tile; reset-free thanks to a 30-bit epoch tag in every word):
//   word = payload32 << 32 | tag << 2 | status      status 0 X (not ready), 1 A, 2 P
//   32-bit carries: one word;  fp64 carries (f32 add): two words (hi, lo halves of the
//   double) written by one 128-bit store and read by one 128-bit load; a reader accepts
//   the pair only if both tags are current and both statuses agree.  The payload is
//   self-contained, so relaxed (.STRONG.GPU, L1-bypassing) accesses suffice.
// Consecutive launches (also CUDA-graph replays) need no memset: every CTA reads the launch
// tag once and counts itself at once, and the last CTA to count advances the epoch (the
// next launch reads it only after this grid completed) -- no atomic and no fence on the
// grid's completion path (DESIGN.md §5 item 14).  Only the launch whose next epoch would
// wrap the 30-bit tag ends with a fenced clear of every descriptor slot.
#include "scan_common.cuh"
#include "scan_internal.h"

namespace scanb200 {

namespace {

constexpr uint32_t ST_A = 1u, ST_P = 2u;
constexpr uint32_t TAG_MASK = 0x3FFFFFFFu;
constexpr int LB_M = 4;                      // descriptors per lane per look-back round trip


__device__ __forceinline__ void st_relaxed_u64(uint64_t* p, uint64_t v) {
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" :: "l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ uint64_t ld_relaxed_u64(const uint64_t* p) {
    uint64_t v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_relaxed_v2u64(uint64_t* p, uint64_t a, uint64_t b) {
    asm volatile("st.relaxed.gpu.global.v2.u64 [%0], {%1, %2};" :: "l"(p), "l"(a), "l"(b) : "memory");
}
__device__ __forceinline__ void ld_relaxed_v2u64(const uint64_t* p, uint64_t& a, uint64_t& b) {
    asm volatile("ld.relaxed.gpu.global.v2.u64 {%0, %1}, [%2];" : "=l"(a), "=l"(b) : "l"(p) : "memory");
}

template <class Op>
struct Desc {
    using C = typename Op::Carry;
    static __device__ __forceinline__ void publish(const LookbackParams& p, int64_t t, uint32_t tag,
                                                   uint32_t st, C v) {
        const uint64_t meta = (uint64_t)((tag << 2) | st);
        if constexpr (sizeof(C) == 8) {
            const uint64_t b = (uint64_t)__double_as_longlong(v);
            st_relaxed_v2u64(p.desc + kDescWords * t, (b & 0xFFFFFFFF00000000ull) | meta, (b << 32) | meta);
        } else {
            // one descriptor per 16-byte slot even for 8-byte descriptors: fewer tiles share a
            // 128-byte L2 line, i.e. fewer concurrent writers / pollers per line (measured)
            st_relaxed_u64(p.desc + kDescWords * t, ((uint64_t)to_bits<C>(v) << 32) | meta);
        }
    }
    // raw load of a slot (issued without consuming the result, so a warp can have every
    // load of a window in flight at once) and its decoding
    struct Raw { uint64_t a, b; };
    static __device__ __forceinline__ void load(const LookbackParams& p, int64_t t, Raw& r) {
        if constexpr (sizeof(C) == 8) ld_relaxed_v2u64(p.desc + kDescWords * t, r.a, r.b);
        else r.a = ld_relaxed_u64(p.desc + kDescWords * t);
    }
    static __device__ __forceinline__ uint32_t decode(const Raw& r, uint32_t tag, C& v) {
        if constexpr (sizeof(C) == 8) {
            const uint32_t mh = (uint32_t)r.a, ml = (uint32_t)r.b;
            if ((mh >> 2) != tag || mh != ml) return 0u;
            v = __longlong_as_double((long long)((r.a & 0xFFFFFFFF00000000ull) | (r.b >> 32)));
            return mh & 3u;
        } else {
            if ((((uint32_t)r.a) >> 2) != tag) return 0u;
            v = from_bits<C>((uint32_t)(r.a >> 32));
            return (uint32_t)r.a & 3u;
        }
    }
    // returns status (0 when stale, torn or not yet written) and the matching value
    static __device__ __forceinline__ uint32_t read(const LookbackParams& p, int64_t t, uint32_t tag, C& v) {
        if constexpr (sizeof(C) == 8) {
            uint64_t hi, lo;
            ld_relaxed_v2u64(p.desc + kDescWords * t, hi, lo);
            const uint32_t mh = (uint32_t)hi, ml = (uint32_t)lo;
            if ((mh >> 2) != tag || mh != ml) return 0u;
            v = __longlong_as_double((long long)((hi & 0xFFFFFFFF00000000ull) | (lo >> 32)));
            return mh & 3u;
        } else {
            const uint64_t w = ld_relaxed_u64(p.desc + kDescWords * t);
            if ((((uint32_t)w) >> 2) != tag) return 0u;
            v = from_bits<C>((uint32_t)(w >> 32));
            return (uint32_t)w & 3u;
        }
    }
};

// Warp-cooperative look-back for tile `t` (t is not the first tile of its problem).  Each
// round trip inspects the 32*LB_M nearest unvisited predecessors (lane l, slot m looks at
// distance l + 32 m); it waits only for the predecessors up to the nearest inclusive (P)
// one, folds their values and stops there, or slides the window further back.
template <class Op, int M = LB_M>
__device__ __forceinline__ typename Op::Carry look_back(const LookbackParams& p, int64_t t, uint32_t tag,
                                                        uint32_t* stats = nullptr) {
    using C = typename Op::Carry;
    const int lane = lane_id();
    C run = Op::cidentity();
    int64_t front = t - 1;                  // nearest predecessor not yet folded
    while (true) {
        C v[M];
        uint32_t st[M];
        int dP;
        int spins = 0;
        if (stats) stats[1] += 1;           // windows visited
        while (true) {
            if (stats) stats[0] += 1;       // descriptor read round trips
#pragma unroll
            for (int m = 0; m < M; ++m) {
                const int64_t pred = front - lane - 32 * m;
                v[m] = Op::cidentity();
                st[m] = pred >= 0 ? Desc<Op>::read(p, pred, tag, v[m]) : ST_P;
            }
            dP = 1 << 30;                    // distance of the nearest P in the window
#pragma unroll
            for (int m = M - 1; m >= 0; --m) {
                const unsigned pm = __ballot_sync(FULL, st[m] == ST_P);
                if (pm) dP = 32 * m + __ffs(pm) - 1;
            }
            bool ok = true;
#pragma unroll
            for (int m = 0; m < M; ++m) {
                const unsigned xm = __ballot_sync(FULL, st[m] == 0u && (lane + 32 * m) < dP);
                ok = ok && (xm == 0u);
            }
            if (ok) break;
            if (++spins > 2) __nanosleep(32);
        }
        C mine = Op::cidentity();
#pragma unroll
        for (int m = 0; m < M; ++m)
            if (lane + 32 * m <= dP && front - lane - 32 * m >= 0) mine = Op::capply(v[m], mine);
        run = Op::capply(warp_reduce_carry<Op>(mine), run);   // the window is older than `run`
        if (dP < (1 << 30)) break;
        front -= 32 * M;
    }
    return run;
}

// The same look-back with the window's loads in flight together (one L2 round trip per
// poll instead of M, the serialised form above) and re-polls that re-read only the
// descriptors still missing before the nearest P, with an exponential back-off starting at
// p.poll_ns -- so a waiting warp does not flood the descriptor lines the streaming traffic
// shares L2 with.
template <class Op, int M = LB_M>
__device__ __forceinline__ typename Op::Carry look_back_par(const LookbackParams& p, int64_t t, uint32_t tag,
                                                            uint32_t* stats = nullptr) {
    using C = typename Op::Carry;
    using Raw = typename Desc<Op>::Raw;
    const int lane = lane_id();
    C run = Op::cidentity();
    int64_t front = t - 1;
    while (true) {
        C v[M];
        uint32_t st[M];
        Raw r[M];
        if (stats) { stats[1] += 1; stats[0] += 1; }
#pragma unroll
        for (int m = 0; m < M; ++m) {
            const int64_t pred = front - lane - 32 * m;
            r[m].a = r[m].b = 0ull;
            if (pred >= 0) Desc<Op>::load(p, pred, r[m]);
        }
#pragma unroll
        for (int m = 0; m < M; ++m) {
            const int64_t pred = front - lane - 32 * m;
            v[m] = Op::cidentity();
            st[m] = pred >= 0 ? Desc<Op>::decode(r[m], tag, v[m]) : ST_P;
        }
        int dP;
        uint32_t ns = p.poll_ns;
        while (true) {
            dP = 1 << 30;
#pragma unroll
            for (int m = M - 1; m >= 0; --m) {
                const unsigned pm = __ballot_sync(FULL, st[m] == ST_P);
                if (pm) dP = 32 * m + __ffs(pm) - 1;
            }
            bool pend[M];
            bool any = false;
#pragma unroll
            for (int m = 0; m < M; ++m) {
                pend[m] = st[m] == 0u && (lane + 32 * m) < dP;
                any = any || (__ballot_sync(FULL, pend[m]) != 0u);
            }
            if (!any) break;
            if (ns) { __nanosleep(ns); if (ns < 2048u) ns <<= 1; }
            if (stats) stats[0] += 1;
#pragma unroll
            for (int m = 0; m < M; ++m)
                if (pend[m]) Desc<Op>::load(p, front - lane - 32 * m, r[m]);
#pragma unroll
            for (int m = 0; m < M; ++m)
                if (pend[m]) st[m] = Desc<Op>::decode(r[m], tag, v[m]);
        }
        C mine = Op::cidentity();
#pragma unroll
        for (int m = 0; m < M; ++m)
            if (lane + 32 * m <= dP && front - lane - 32 * m >= 0) mine = Op::capply(v[m], mine);
        run = Op::capply(warp_reduce_carry<Op>(mine), run);   // the window is older than `run`
        if (dP < (1 << 30)) break;
        front -= 32 * M;
    }
    return run;
}

// Look-back of a PERSISTENT round-robin grid (tile t = cta + i * grid): the CTA's own
// previous tile t - grid was resolved by this CTA, so its inclusive prefix is known in
// shared memory (s_incl, tagged with its sequence number in s_iseq).  The carry of t is
//     incl(t - grid)  .  A(t - grid + 1)  .  ...  .  A(t - 1)
// or, if one of those window tiles already published its inclusive value P, the fold from
// the nearest P.  So the window never slides past t - grid: one window of grid - 1 <= 32 M
// descriptors, loaded together; re-polls re-read only the descriptors still missing (X),
// with back-off; once every window tile has at least its aggregate the warp waits on
// shared memory only (no L2 traffic).  If the local slot was already lapped (the ring holds
// 2 x SH sequences), tile t - grid's P descriptor is read instead (it was published before
// the slot was written).
template <class Op, int M>
__device__ __forceinline__ typename Op::Carry look_back_rr(const LookbackParams& p, int64_t t, int64_t i, int64_t grid,
                                                           uint32_t tag, const typename Op::Carry* s_incl,
                                                           const int64_t* s_iseq, int ring, uint32_t* stats) {
    using C = typename Op::Carry;
    using Raw = typename Desc<Op>::Raw;
    const int lane = lane_id();
    const int64_t span = grid - 1;
    C v[M];
    uint32_t st[M];
    Raw r[M];
    if (stats) { stats[1] += 1; stats[0] += 1; }
#pragma unroll
    for (int m = 0; m < M; ++m) {
        const int64_t d = 1 + lane + 32 * m;
        r[m].a = r[m].b = 0ull;
        if (d <= span) Desc<Op>::load(p, t - d, r[m]);
    }
#pragma unroll
    for (int m = 0; m < M; ++m) {
        const int64_t d = 1 + lane + 32 * m;
        v[m] = Op::cidentity();
        st[m] = d <= span ? Desc<Op>::decode(r[m], tag, v[m]) : ST_A;     // outside: identity
    }
    const int slot = (int)((i - 1) % ring);
    bool have_local = false;
    C local = Op::cidentity();
    int dP;
    uint32_t ns = p.poll_ns;
    while (true) {
        dP = 1 << 30;
#pragma unroll
        for (int m = M - 1; m >= 0; --m) {
            const unsigned pm = __ballot_sync(FULL, st[m] == ST_P);
            if (pm) dP = 32 * m + __ffs(pm) - 1;
        }
        bool pend[M];
        bool any = false;
#pragma unroll
        for (int m = 0; m < M; ++m) {
            pend[m] = st[m] == 0u && (lane + 32 * m) < dP;
            any = any || (__ballot_sync(FULL, pend[m]) != 0u);
        }
        if (!any) {
            if (dP < (1 << 30)) break;                   // fold from the nearest P
            const int64_t q = *(const volatile int64_t*)(s_iseq + slot);
            if (q == i - 1) {
                __threadfence_block();
                local = *(const volatile C*)(s_incl + slot);
                have_local = true;
                break;
            }
            if (q > i - 1) {                             // lapped: tile t - grid's P is global
                C pv = Op::cidentity();
                while (Desc<Op>::read(p, t - grid, tag, pv) != ST_P) __nanosleep(64);
                local = pv;
                have_local = true;
                break;
            }
            __nanosleep(20);                             // local prefix not ready: smem only
            continue;
        }
        if (ns) { __nanosleep(ns); if (ns < 2048u) ns <<= 1; }
        if (stats) stats[0] += 1;
#pragma unroll
        for (int m = 0; m < M; ++m)
            if (pend[m]) Desc<Op>::load(p, t - 1 - lane - 32 * m, r[m]);
#pragma unroll
        for (int m = 0; m < M; ++m)
            if (pend[m]) st[m] = Desc<Op>::decode(r[m], tag, v[m]);
    }
    C mine = Op::cidentity();
#pragma unroll
    for (int m = 0; m < M; ++m)
        if (lane + 32 * m <= dP) mine = Op::capply(v[m], mine);
    C run = warp_reduce_carry<Op>(mine);
    if (have_local) run = Op::capply(local, run);
    return run;
}


// debug timeline (scan_debug_trace): stamp e of tile t with %globaltimer (ns)
__device__ __forceinline__ void trace_stamp(const LookbackParams& p, int64_t t, int e) {
    if (p.trace != nullptr && t < p.trace_tiles) {
        uint64_t g;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(g));
        p.trace[8 * t + e] = g;
    }
}
__device__ __forceinline__ void trace_value(const LookbackParams& p, int64_t t, int e, uint64_t v) {
    if (p.trace != nullptr && t < p.trace_tiles) p.trace[8 * t + e] = v;
}

__device__ __forceinline__ void consumer_bar(int nthreads) {
    asm volatile("bar.sync 1, %0;" :: "r"(nthreads) : "memory");
}

// Tile body with the tile already in shared memory: pass 1, look-back by the last warp,
// pass 2.  With NAMED_BAR only the WARPS consumer warps synchronise.
template <class Op, bool SEG, int WARPS, int V, bool NAMED_BAR>
__device__ __forceinline__ void tile_body_smem(const LookbackParams& p, int64_t tile, uint32_t tag, int64_t r,
                                               const typename Op::T* s_tile, bool fast,
                                               typename Op::Carry* s_carry, typename Op::T* s_wval,
                                               uint32_t* s_wflag) {
    using T = typename Op::T;
    using C = typename Op::Carry;
    constexpr int TILE = WARPS * 32 * V * 4;
    constexpr int WCH = V * 128;
    const int warp = threadIdx.x >> 5, lane = lane_id();
    const int64_t base = tile * (int64_t)TILE;
    const T* srow = s_tile + warp * WCH;

    WarpTileS<Op, SEG, V> wt;
    {
        // literal `small` per call (see the L2-staged scanners): no short-problem head test
        // in the long-problem path
        if (SEG && p.N < TILE) wt.pass1(srow, warp * WCH, true, (uint32_t)r, (uint32_t)p.N, -1);
        else wt.pass1(srow, warp * WCH, false, 0u, 1u, SEG ? (r == 0 ? 0 : (int)(p.N - r)) : -1);
    }
    if (lane == 0) { s_wval[warp] = wt.wtot; s_wflag[warp] = wt.wfl; }
    if (NAMED_BAR) consumer_bar(WARPS * 32); else __syncthreads();
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
    if (NAMED_BAR) consumer_bar(WARPS * 32); else __syncthreads();
    const T cin = Op::from_carry(*s_carry);
    wt.pass2(srow, (T*)p.out, base + warp * WCH, p.total, fast, p.vec, p.exclusive, wp, wpf, cin);
}

// Tile classification done once per tile by whoever owns the ticket.
struct TileInfo { int64_t r; uint32_t seg; uint32_t fast; };
__device__ __forceinline__ TileInfo classify(const LookbackParams& p, int64_t t, int tile_elems) {
    TileInfo ti;
    const int64_t base = t * (int64_t)tile_elems;
    ti.r = base % p.N;
    const int64_t count = p.total - base < tile_elems ? p.total - base : tile_elems;
    const int64_t next_head = ti.r == 0 ? p.N : p.N - ti.r;    // first problem start after offset 0
    ti.seg = next_head < count ? 1u : 0u;
    ti.fast = (p.vec && count == tile_elems) ? 1u : 0u;
    return ti;
}

// End-of-grid epilogue of the launch whose next epoch would wrap the 30-bit tag (tag + 1 ==
// TAG_MASK; once per ~2^30 launches): the last CTA to finish clears every descriptor slot and
// restarts the epoch at 0.  It fences first, so that none of this launch's own descriptor
// stores can land after the clear and survive into the next cycle of tags.
__device__ __forceinline__ void epilogue(const LookbackParams& p, uint32_t tag) {
    (void)tag;
    __threadfence();
    const uint32_t prev = atomicAdd(p.ctl + 1, 1u);
    if (prev == gridDim.x - 1) {
        __threadfence();
        for (int64_t i = 0; i < kDescWords * p.capacity; ++i) p.desc[i] = 0ull;
        ((volatile uint32_t*)p.ctl)[0] = 0u;
        ((volatile uint32_t*)p.ctl)[1] = 0u;
        ((volatile uint32_t*)p.ctl)[2] = 0u;
        __threadfence();
    }
}

__device__ __forceinline__ uint32_t read_tag(const LookbackParams& p) {
    uint32_t e;
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(e) : "l"(p.ctl + 2) : "memory");
    return (e + 1u) & TAG_MASK;
}

// Start-of-grid epoch advance (see lookback_l2_kernel): a CTA counts itself right after it
// read the launch tag (once per CTA); the ticket is consumed only at the CTA's end, so the
// atomic's round trip overlaps the CTA's work, and the CTA that counted last advances the
// epoch there without a further round trip.  The wrap launch keeps the fenced epilogue.
__device__ __forceinline__ uint32_t count_tag_read(const LookbackParams& p, uint32_t tag) {
    return tag + 1u < TAG_MASK ? atomicAdd(p.ctl + 1, 1u) : 0xFFFFFFFFu;
}
__device__ __forceinline__ void finish_epoch(const LookbackParams& p, uint32_t tag, uint32_t ticket) {
    if (tag + 1u >= TAG_MASK) {
        epilogue(p, tag);
    } else if (ticket == gridDim.x - 1) {
        ((volatile uint32_t*)p.ctl)[0] = 0u;
        ((volatile uint32_t*)p.ctl)[1] = 0u;
        ((volatile uint32_t*)p.ctl)[2] = tag;
    }
}


// ---------------------------------------------------------------- pipelined, dedicated look-back warp
// Warp roles: WARPS consumer warps, one producer warp (TMA ring), one look-back warp.
// Per ring slot: full (producer -> consumers), p1 (consumers' pass 1 done -> look-back
// warp), cr (carry ready -> consumers), empty (consumers' pass 2 done -> producer).
// Consumers run pass 1 of tile i+1 before pass 2 of tile i, so the look-back of tile i
// (>= 1 L2 round trip) overlaps with useful work instead of idling 8 warps at a barrier.
template <class Op, int WARPS>
struct SlotHdr {
    using T = typename Op::T;
    using C = typename Op::Carry;
    int64_t tid;
    int64_t r;
    uint32_t seg, fast;
    uint32_t keep;          // L2-staged kernel: scan this tile from its read-1 slot
    T wtot[WARPS];
    uint32_t wfl[WARPS];
    T wp[WARPS];
    uint32_t wpf[WARPS];
    C agg;
    uint32_t has_head;
    C carry;
};

template <class Op, int WARPS, int V, int S>
struct PipeCtx {
    using T = typename Op::T;
    static constexpr int TILE = WARPS * 32 * V * 4;
    static constexpr int WCH = V * 128;
    T* data;
    SlotHdr<Op, WARPS>* hdr;
    uint64_t* full;
    uint64_t* p1;
    uint64_t* cr;
    uint64_t* empty;
    int64_t* end;           // sequence index of the end sentinel (INT64_MAX until met)
};

// consumer: pass 1 of the tile in sequence slot i; false at the end sentinel
// The aggregate (A) -- or, for a tile holding a problem start, the inclusive value (P) --
// is published right here by the last consumer warp, not by the look-back warp: a tile's
// A must never wait for the look-back of the CTA's previous tile, or every round of the
// round-robin schedule would serialise behind the previous round's resolution.
template <class Op, int WARPS, int V, int S>
__device__ __forceinline__ bool pipe_pass1(const LookbackParams& p, const PipeCtx<Op, WARPS, V, S>& c,
                                           WarpTileP<Op, V>& st, int64_t i, uint32_t tag) {
    using T = typename Op::T;
    constexpr int TILE = PipeCtx<Op, WARPS, V, S>::TILE, WCH = PipeCtx<Op, WARPS, V, S>::WCH;
    const int slot = (int)(i % S);
    const uint32_t ph = (uint32_t)((i / S) & 1);
    const int warp = threadIdx.x >> 5, lane = lane_id();
    mbar_wait(&c.full[slot], ph);
    SlotHdr<Op, WARPS>& h = c.hdr[slot];
    if (h.tid < 0) {
        if (warp == WARPS - 1 && lane == 0) {
            *(volatile int64_t*)c.end = i;       // look-back warps waiting beyond i leave
            mbar_arrive(&c.p1[slot]);
        }
        return false;
    }
    if (warp == 0 && lane == 0) trace_stamp(p, h.tid, 0);
    const T* srow = c.data + (size_t)slot * TILE + warp * WCH;
    const int64_t r = h.r;
    if (h.seg && p.N < TILE) {
        st.template pass1<true>(srow, warp * WCH, true, (uint32_t)r, (uint32_t)p.N, -1);
    } else if (h.seg) {
        st.template pass1<true>(srow, warp * WCH, false, 0u, 1u, r == 0 ? 0 : (int)(p.N - r));
    } else {
        st.template pass1<false>(srow, warp * WCH, false, 0u, 1u, -1);
    }
    if (lane == 0) {
        h.wtot[warp] = st.wtot;
        h.wfl[warp] = st.wfl ? 1u : 0u;
    }
    consumer_bar(WARPS * 32);
    if (warp == WARPS - 1) {
        const bool seg = h.seg != 0u;
        T run = Op::identity(); bool f = false;
#pragma unroll
        for (int w = 0; w < WARPS; ++w) {                // segmented exclusive prefix of warp totals
            if (lane == w) { h.wp[w] = run; h.wpf[w] = f ? 1u : 0u; }
            const T v = h.wtot[w];
            const bool fw = seg && h.wfl[w] != 0u;
            run = fw ? v : Op::apply(run, v);
            f = f || fw;
        }
        const bool has_head = seg ? f : (r == 0);
        if (lane == 0) {
            h.agg = Op::to_carry(run);
            h.has_head = has_head ? 1u : 0u;
            trace_stamp(p, h.tid, 1);
            Desc<Op>::publish(p, h.tid, tag, has_head ? ST_P : ST_A, h.agg);
        }
        __syncwarp();
        if (lane == 0) mbar_arrive(&c.p1[slot]);
    }
    return true;
}

// consumer: pass 2 of the tile in sequence slot i (carry from the look-back warp)
template <class Op, int WARPS, int V, int S>
__device__ __forceinline__ void pipe_pass2(const LookbackParams& p, const PipeCtx<Op, WARPS, V, S>& c,
                                           const WarpTileP<Op, V>& st, int64_t i) {
    using T = typename Op::T;
    constexpr int TILE = PipeCtx<Op, WARPS, V, S>::TILE, WCH = PipeCtx<Op, WARPS, V, S>::WCH;
    const int slot = (int)(i % S);
    const uint32_t ph = (uint32_t)((i / S) & 1);
    const int warp = threadIdx.x >> 5, lane = lane_id();
    mbar_wait(&c.cr[slot], ph);
    const SlotHdr<Op, WARPS>& h = c.hdr[slot];
    const T* srow = c.data + (size_t)slot * TILE + warp * WCH;
    const int64_t gidx = h.tid * (int64_t)TILE + warp * WCH;
    const bool fast = h.fast != 0u;
    const T cin = Op::from_carry(h.carry);
    const T wp = h.wp[warp];
    const bool wpf = h.wpf[warp] != 0u;
    if (h.seg) st.template pass2<true>(srow, (T*)p.out, gidx, p.total, fast, p.vec, p.exclusive, wp, wpf, cin);
    else       st.template pass2<false>(srow, (T*)p.out, gidx, p.total, fast, p.vec, p.exclusive, wp, wpf, cin);
    // every lane's smem reads of this slot are ordered before lane 0's release-arrive on
    // `empty`; the producer's acquire-wait on it precedes any rewrite of the slot
    __threadfence_block();
    __syncwarp();
    if (warp == 0 && lane == 0) trace_stamp(p, h.tid, 3);
    if (lane == 0) mbar_arrive(&c.empty[slot]);
}

template <class Op, int WARPS, int V, int S, int M, int NLB, int PF = 0>
__global__ void __launch_bounds__((WARPS + 1 + NLB) * 32) lookback_pipelined_kernel(LookbackParams p, int64_t num_tiles) {
    using T = typename Op::T;
    using C = typename Op::Carry;
    using Ctx = PipeCtx<Op, WARPS, V, S>;
    constexpr int TILE = Ctx::TILE;
    extern __shared__ __align__(128) unsigned char dsm[];
    __shared__ SlotHdr<Op, WARPS> s_hdr[S];
    __shared__ uint64_t s_full[S], s_p1[S], s_cr[S], s_empty[S];
    __shared__ uint32_t s_tag;
    __shared__ int64_t s_end;
    const int warp = threadIdx.x >> 5, lane = lane_id();
    Ctx c{(T*)dsm, s_hdr, s_full, s_p1, s_cr, s_empty, &s_end};

    if (threadIdx.x == 0) {
        s_end = INT64_MAX;
#pragma unroll
        for (int s = 0; s < S; ++s) {
            mbar_init(&s_full[s], 1); mbar_init(&s_p1[s], 1);
            mbar_init(&s_cr[s], 1);   mbar_init(&s_empty[s], WARPS);
        }
        fence_mbar_init();
        s_tag = read_tag(p);
    }
    uint32_t ticket = 0u;
    if (threadIdx.x == 0) ticket = count_tag_read(p, s_tag);
    __syncthreads();
    const uint32_t tag = s_tag;

    if (warp < WARPS) {
        // ---------------- consumers: pass1(i+1) then pass2(i), two register states
        WarpTileP<Op, V> A, B;
        int64_t i = 0;
        if (pipe_pass1<Op, WARPS, V, S>(p, c, A, 0, tag)) {
            while (true) {
                ++i;
                bool more = pipe_pass1<Op, WARPS, V, S>(p, c, B, i, tag);
                pipe_pass2<Op, WARPS, V, S>(p, c, A, i - 1);
                if (!more) break;
                ++i;
                more = pipe_pass1<Op, WARPS, V, S>(p, c, A, i, tag);
                pipe_pass2<Op, WARPS, V, S>(p, c, B, i - 1);
                if (!more) break;
            }
        }
    } else if (warp == WARPS) {
        // ---------------- producer: this CTA's tiles (round robin) into the TMA ring
        const T* in = (const T*)p.in;
        const uint64_t pol = l2_evict_first_policy();
        int64_t i = 0;
        for (int64_t t = blockIdx.x;; t += gridDim.x, ++i) {
            const int slot = (int)(i % S);
            const uint32_t ph = (uint32_t)((i / S) & 1);
            mbar_wait(&s_empty[slot], ph ^ 1u);
            SlotHdr<Op, WARPS>& h = s_hdr[slot];
            if (t >= num_tiles) {
                if (lane == 0) { h.tid = -1; mbar_arrive(&s_full[slot]); }
                break;
            }
            const TileInfo ti = classify(p, t, TILE);
            T* dst = c.data + (size_t)slot * TILE;
            const int64_t base = t * (int64_t)TILE;
            if (lane == 0) { h.tid = t; h.r = ti.r; h.seg = ti.seg; h.fast = ti.fast; }
            if (ti.fast) {
                if (lane == 0) {
                    mbar_expect_tx(&s_full[slot], TILE * 4);
                    tma_load_1d(dst, in + base, TILE * 4, &s_full[slot], pol);
                }
            } else {
                for (int k = lane; k < TILE; k += 32)
                    dst[k] = base + k < p.total ? from_bits<T>(ld_stream_u32(in + base + k)) : Op::identity();
                __syncwarp();
                if (lane == 0) mbar_arrive(&s_full[slot]);
            }
            if constexpr (PF > 0) {
                // warm L2 with this CTA's tiles PF rounds ahead (first iteration: rounds 1..PF)
                if (lane == 0 && p.vec) {
#pragma unroll
                    for (int r = (PF > 0 ? 1 : 0); r <= PF; ++r) {
                        if (i > 0 && r < PF) continue;
                        const int64_t tp = t + (int64_t)r * gridDim.x;
                        if ((tp + 1) * (int64_t)TILE <= p.total) prefetch_l2_bulk(in + tp * (int64_t)TILE, TILE * 4);
                    }
                }
            }
        }
    } else {
        // ---------------- NLB look-back warps (tile sequence i -> warp i mod NLB); p1 phases
        // complete in sequence order, so NLB <= S keeps every wait on the right phase
        // The tile of sequence i is known statically (round robin), and a look-back reads
        // only the tile's predecessors, so it starts BEFORE the tile's own pass 1 is done;
        // only publishing P waits for this tile's aggregate (p1).
        static_assert(NLB <= S, "look-back warps must not lap the ring");
        for (int64_t i = warp - (WARPS + 1);; i += NLB) {
            const int64_t t = (int64_t)blockIdx.x + i * (int64_t)gridDim.x;
            if (t >= num_tiles) break;
            const int slot = (int)(i % S);
            const uint32_t ph = (uint32_t)((i / S) & 1);
            const bool starts = ((t * (int64_t)TILE) % p.N) == 0;
            C carry = Op::cidentity();
            uint32_t stats[2] = {0u, 0u};
            if (lane == 0) trace_stamp(p, t, 4);
            if (!starts) carry = look_back<Op, M>(p, t, tag, p.trace ? stats : nullptr);
            mbar_wait(&s_p1[slot], ph);                   // this tile's aggregate is in the header
            SlotHdr<Op, WARPS>& h = s_hdr[slot];
            const bool has_head = h.has_head != 0u;
            const C aggc = h.agg;
            if (lane == 0) {
                if (!has_head) Desc<Op>::publish(p, t, tag, ST_P, Op::capply(carry, aggc));
                h.carry = carry;
                trace_stamp(p, t, 2);
                trace_value(p, t, 5, stats[0]);
                trace_value(p, t, 6, stats[1]);
            }
            __syncwarp();
            if (lane == 0) mbar_arrive(&s_cr[slot]);
        }
    }
    __syncthreads();
    if (threadIdx.x == 0) finish_epoch(p, tag, ticket);
}

// ---------------------------------------------------------------- two reads, L2-staged (variant 3)
// Little's law: a tile that waits in shared memory for its carry holds a slot for the
// whole look-back latency (several us under full HBM load), which caps a single huge
// problem at ~5 TB/s.  Here the tile is read TWICE but from HBM only once:
//   read 1 (TMA, HBM -> smem ring R, L2 evict_last)   reducer warps fold it, publish the
//          aggregate (A) or, for a tile holding a problem start, the inclusive value (P);
//          the R slot is released at once;
//   look-back warp resolves the carry (no smem held while it waits);
//   read 2 (TMA, L2 -> smem ring W, evict_first) issued once the carry is known: the
//          tile is still L2-resident (a few MB in flight vs a 126 MB L2), so this read
//          costs L2 bandwidth, not HBM; scanner warps scan it with the carry and store.
// HBM traffic stays 2N; the look-back wait costs only a header slot.
// Roles: NS scanner warps | NR reducer warps | P1 (read 1) | P2 (read 2) | LB.
template <class Op, int V>
__device__ __forceinline__ typename Op::T warp_reduce_rows(const typename Op::T* srow) {
    using T = typename Op::T;
    const int lane = lane_id();
    T acc = Op::identity();
#pragma unroll
    for (int j = 0; j < V; ++j) {
        Row4<T> x = row_from_u4<T>(lds_v4(srow + j * 128 + lane * 4));
        acc = Op::apply(acc, Op::apply(Op::apply(x.v[0], x.v[1]), Op::apply(x.v[2], x.v[3])));
    }
#pragma unroll
    for (int d = 16; d >= 1; d >>= 1) acc = Op::apply(acc, from_bits<T>(__shfl_xor_sync(FULL, to_bits<T>(acc), d)));
    return acc;
}

// The same over the chunk's elements at tile offsets >= first only (o0 = the chunk's tile
// offset); the earlier ones belong to the previous problem.  Commutative ops only (add, max).
template <class Op, int V>
__device__ __forceinline__ typename Op::T warp_reduce_rows_from(const typename Op::T* srow, int o0, int first) {
    using T = typename Op::T;
    const int lane = lane_id();
    T acc = Op::identity();
#pragma unroll
    for (int j = 0; j < V; ++j) {
        Row4<T> x = row_from_u4<T>(lds_v4(srow + j * 128 + lane * 4));
        const int o = o0 + j * 128 + lane * 4;
#pragma unroll
        for (int q = 0; q < 4; ++q)
            if (o + q >= first) acc = Op::apply(acc, x.v[q]);
    }
#pragma unroll
    for (int d = 16; d >= 1; d >>= 1) acc = Op::apply(acc, from_bits<T>(__shfl_xor_sync(FULL, to_bits<T>(acc), d)));
    return acc;
}

template <class Op, int NS, int NR, int SR, int SW, int SH, int M, int NLB>
__global__ void __launch_bounds__((NS + NR + 2 + NLB) * 32, 1) lookback_l2_kernel(LookbackParams p, int64_t num_tiles) {
    using T = typename Op::T;
    using C = typename Op::Carry;
    constexpr int V = 8, WCH = V * 128, TILE = NS * WCH;
    static_assert(SR >= 2, "kept tail tiles must leave a read-1 slot for the end sentinel");
    extern __shared__ __align__(128) unsigned char dsm[];
    T* bufR = (T*)dsm;                       // SR x TILE
    T* bufW = bufR + (size_t)SR * TILE;      // SW x TILE
    __shared__ SlotHdr<Op, NS> s_hdr[SH];
    __shared__ uint64_t fullR[SR], emptyR[SR], fullW[SW], emptyW[SW], aggd[SH], crd[SH], emptyH[SH];
    __shared__ int64_t s_end;
    constexpr int RING = 2 * SH;             // local inclusive prefixes of this CTA's tiles
    __shared__ C s_incl[RING];
    __shared__ int64_t s_iseq[RING];
    __shared__ uint32_t s_tag;               // the launch's descriptor tag (read once per CTA)
    __shared__ uint64_t tagbar;              // s_tag is valid
    const int warp = threadIdx.x >> 5, lane = lane_id();
    if (threadIdx.x == 0) trace_stamp(p, blockIdx.x, 7);     // CTA entry (debug timeline)
    // every CTA is resident before a dependent grid can launch (launch_dependents counts
    // all of them), so the static round robin's inter-CTA waits cannot be starved of SMs;
    // the wait orders the previous kernel's writes (our input, the epoch) before any access
    grid_dep_launch();
    // the shared-memory set-up touches no global memory, so it runs before the wait for the
    // stream's previous kernel, one ring slot per lane of warp 0 (CTA entry -> first bulk
    // copy is ~0.8 us either way: the wait for the previous grid's completion dominates)
    static_assert(SR <= 32 && SW <= 32 && RING <= 32, "one barrier slot per lane");
    if (warp == 0) {
        if (lane < SR) { mbar_init(&fullR[lane], 1); mbar_init(&emptyR[lane], NR); }
        if (lane < SW) { mbar_init(&fullW[lane], 1); mbar_init(&emptyW[lane], NS); }
        if (lane < SH) { mbar_init(&aggd[lane], 1); mbar_init(&crd[lane], 1); mbar_init(&emptyH[lane], NS); }
        if (lane < RING) s_iseq[lane] = -1;
        if (lane == 0) { s_end = INT64_MAX; mbar_init(&tagbar, 1); }
        fence_mbar_init();
    }
    // the HBM -> L2 part of this CTA's first SR tiles starts before that wait: a bulk L2
    // prefetch moves no data to the SM and L2 is the point of coherence, so it cannot
    // expose stale data -- the reads proper (TMA, after the wait) see every write of the
    // previous kernel -- but the ~0.8 us between the CTAs' entry and the previous grid's
    // completion is no longer lost to HBM
    if (warp == NS + NR && lane == 0 && p.vec && p.pdl_first) {
#pragma unroll 1
        for (int k = 0; k < SR; ++k) {
            const int64_t tk = (int64_t)blockIdx.x + (int64_t)k * gridDim.x;
            if ((tk + 1) * (int64_t)TILE <= p.total) prefetch_l2_bulk((const T*)p.in + tk * (int64_t)TILE, TILE * 4);
        }
    }
    if (p.pdl_first) grid_dep_wait();
    __syncthreads();
    // The launch tag (an L2 round trip) is read once, by the first look-back warp -- not by
    // the read-1 producer, so the first bulk copies are not queued behind it -- and handed
    // to the reducers and look-back warps through shared memory.  Right after reading it
    // the CTA counts itself; the LAST CTA to have read the tag advances the epoch at once.
    // Every CTA of this launch has then read its tag, and the next launch reads the new
    // epoch only after this grid completed, so the advance needs no end-of-grid epilogue
    // (an atomic round trip plus the reset on the grid's completion path).  Only a launch
    // whose next epoch would wrap keeps the end-of-grid form (fenced, clears every slot).
    if (warp == NS + NR + 2 && lane == 0) {
        const uint32_t t = read_tag(p);
        s_tag = t;
        mbar_arrive(&tagbar);
        if (t + 1u < TAG_MASK && atomicAdd(p.ctl + 1, 1u) == gridDim.x - 1) {
            ((volatile uint32_t*)p.ctl)[1] = 0u;
            ((volatile uint32_t*)p.ctl)[2] = t;        // the epoch this launch used
        }
    }
    uint32_t tag = 0u;
    if (warp >= NS && warp != NS + NR && warp != NS + NR + 1) {   // reducers, look-back warps
        mbar_wait(&tagbar, 0u);
        tag = s_tag;
    }
    const T* in = (const T*)p.in;

    if (warp < NS) {
        // ---------------- scanners: read 2 landed -> full scan with the carry -> store
        for (int64_t i = 0;; ++i) {
            const int sW = (int)(i % SW), sH = (int)(i % SH);
            mbar_wait(&fullW[sW], (uint32_t)((i / SW) & 1));
            const SlotHdr<Op, NS>& h = s_hdr[sH];
            const int64_t t = h.tid;
            if (t < 0) break;
            if (p.early_read2) mbar_wait(&crd[sH], (uint32_t)((i / SH) & 1));   // the carry
            // a kept tile (the CTA's last) is still in its read-1 slot: no second read
            const T* srow = (h.keep ? bufR + (size_t)(i % SR) * TILE : bufW + (size_t)sW * TILE) + warp * WCH;
            const T cin = Op::from_carry(h.carry);
            const T wp = h.wp[warp];
            const bool wpf = h.wpf[warp] != 0u, fast = h.fast != 0u;
            const int64_t gidx = t * (int64_t)TILE + warp * WCH;
            WarpTileP<Op, V> st;
            // the two head-placement modes are separate calls with a literal `small`, so each
            // inlined copy keeps only its own head test (a runtime `small` left the per-row
            // modulo of the short-problem test in the long-problem path: segmented tiles took
            // 2.5 us instead of ~1 us to scan, DESIGN.md §5 item 11)
            if (h.seg && p.N >= TILE) {
                const int first = (int)(p.N - h.r);          // one problem start in the tile
                st.template pass1<true>(srow, warp * WCH, false, 0u, 1u, first);
                st.template pass2<true>(srow, (T*)p.out, gidx, p.total, fast, p.vec, p.exclusive, wp, wpf, cin);
            } else if (h.seg) {
                st.template pass1<true>(srow, warp * WCH, true, (uint32_t)h.r, (uint32_t)p.N, -1);
                st.template pass2<true>(srow, (T*)p.out, gidx, p.total, fast, p.vec, p.exclusive, wp, wpf, cin);
            } else {
                st.template pass1<false>(srow, warp * WCH, false, 0u, 1u, -1);
                st.template pass2<false>(srow, (T*)p.out, gidx, p.total, fast, p.vec, p.exclusive, wp, wpf, cin);
            }
            __syncwarp();
            if (lane == 0) {
                if (warp == 0) trace_stamp(p, t, 3);
                mbar_arrive(&emptyW[sW]);
                mbar_arrive(&emptyH[sH]);
            }
        }
    } else if (warp < NS + NR) {
        // ---------------- reducers: read 1 landed -> per-1024 totals -> A (or P)
        const int rr = warp - NS;
        for (int64_t i = 0;; ++i) {
            const int sR = (int)(i % SR), sH = (int)(i % SH);
            mbar_wait(&fullR[sR], (uint32_t)((i / SR) & 1));
            SlotHdr<Op, NS>& h = s_hdr[sH];
            const int64_t t = h.tid;
            if (t < 0) {
                if (rr == NR - 1 && lane == 0) {
                    *(volatile int64_t*)&s_end = i;      // look-back warps waiting beyond i leave
                    mbar_arrive(&aggd[sH]);
                }
                break;
            }
            if (rr == NR - 1 && lane == 0) trace_stamp(p, t, 0);
            const bool seg = h.seg != 0u;
            const int64_t r = h.r;
            for (int k = rr; k < NS; k += NR) {
                const T* srow = bufR + (size_t)sR * TILE + k * WCH;
                T tot; bool fl = false;
                if (seg && p.N >= TILE) {
                    // N >= TILE: the tile holds exactly one problem start, at `first`; the
                    // chunk that contains it folds only the elements from there on (the new
                    // problem's head), every other chunk is a plain total -- a masked
                    // reduction instead of a full segmented scan (ready -> A of such tiles
                    // 2.25 -> 0.75 us, DESIGN.md §5 item 11)
                    const int first = (int)(p.N - r);
                    const int lo = k * WCH;
                    fl = first >= lo && first < lo + WCH;
                    tot = fl ? warp_reduce_rows_from<Op, V>(srow, lo, first) : warp_reduce_rows<Op, V>(srow);
                } else if (seg) {
                    WarpTileP<Op, V> st;
                    st.template pass1<true>(srow, k * WCH, true, (uint32_t)r, (uint32_t)p.N, -1);
                    tot = st.wtot; fl = st.wfl;
                } else {
                    tot = warp_reduce_rows<Op, V>(srow);
                }
                if (lane == 0) { h.wtot[k] = tot; h.wfl[k] = fl ? 1u : 0u; }
            }
            __syncwarp();
            // a kept tile keeps its slot: read-1 never reuses it (at most SR - 1 tiles of the
            // CTA are kept, and the end sentinel takes the remaining slot)
            if (lane == 0 && !h.keep) mbar_arrive(&emptyR[sR]);
            asm volatile("bar.sync 2, %0;" :: "r"(NR * 32) : "memory");
            if (rr == NR - 1) {
                T run = Op::identity(); bool f = false;
#pragma unroll
                for (int w = 0; w < NS; ++w) {
                    if (lane == w) { h.wp[w] = run; h.wpf[w] = f ? 1u : 0u; }
                    const T v = h.wtot[w];
                    const bool fw = seg && h.wfl[w] != 0u;
                    run = fw ? v : Op::apply(run, v);
                    f = f || fw;
                }
                const bool has_head = seg ? f : (r == 0);
                if (lane == 0) {
                    h.agg = Op::to_carry(run);
                    h.has_head = has_head ? 1u : 0u;
                    Desc<Op>::publish(p, t, tag, has_head ? ST_P : ST_A, h.agg);
                    trace_stamp(p, t, 1);
                }
                __syncwarp();
                if (lane == 0) mbar_arrive(&aggd[sH]);
            }
        }
    } else if (warp == NS + NR) {
        // ---------------- P1: read 1 of this CTA's tiles (round robin) into ring R
        const uint64_t pol = l2_evict_last_policy();
        int64_t i = 0;
        for (int64_t t = blockIdx.x;; t += gridDim.x, ++i) {
            const int sR = (int)(i % SR), sH = (int)(i % SH);
            mbar_wait(&emptyR[sR], (uint32_t)((i / SR) & 1) ^ 1u);
            mbar_wait(&emptyH[sH], (uint32_t)((i / SH) & 1) ^ 1u);
            SlotHdr<Op, NS>& h = s_hdr[sH];
            if (t >= num_tiles) {
                if (lane == 0) { h.tid = -1; mbar_arrive(&fullR[sR]); }
                break;
            }
            const TileInfo ti = classify(p, t, TILE);
            T* dst = bufR + (size_t)sR * TILE;
            const int64_t base = t * (int64_t)TILE;
            if (lane == 0) {
                h.tid = t; h.r = ti.r; h.seg = ti.seg; h.fast = ti.fast;
                // the CTA's last SR - 1 tiles are scanned from their read-1 slots (no second
                // read on the kernel's tail); the slots they keep are never needed again
                h.keep = (p.keep_last && t + (int64_t)(SR - 1) * gridDim.x >= num_tiles) ? 1u : 0u;
            }
            if (ti.fast) {
                if (lane == 0) {
                    mbar_expect_tx(&fullR[sR], TILE * 4);
                    tma_load_1d(dst, in + base, TILE * 4, &fullR[sR], pol);
                }
            } else {
                for (int k = lane; k < TILE; k += 32)
                    dst[k] = base + k < p.total ? from_bits<T>(ld_stream_u32(in + base + k)) : Op::identity();
                __syncwarp();
                if (lane == 0) mbar_arrive(&fullR[sR]);
            }
            // start the HBM -> L2 part of the next round's read 1 now
            const int64_t tn = t + gridDim.x;
            if (lane == 0 && p.vec && (tn + 1) * (int64_t)TILE <= p.total)
                prefetch_l2_bulk(in + tn * (int64_t)TILE, TILE * 4);
        }
    } else if (warp == NS + NR + 1) {
        // ---------------- P2: read 2 (from L2) once the carry is known, into ring W
        const uint64_t pol = l2_evict_first_policy();
        for (int64_t i = 0;; ++i) {
            const int sW = (int)(i % SW), sH = (int)(i % SH);
            // read 2 goes out once the tile's carry is known -- or, with early_read2, once
            // its aggregate is (the data waits in the W ring instead of in L2 while the
            // look-back resolves; the scanners then wait for the carry themselves)
            if (p.early_read2) mbar_wait(&aggd[sH], (uint32_t)((i / SH) & 1));
            else mbar_wait(&crd[sH], (uint32_t)((i / SH) & 1));
            mbar_wait(&emptyW[sW], (uint32_t)((i / SW) & 1) ^ 1u);
            const SlotHdr<Op, NS>& h = s_hdr[sH];
            const int64_t t = h.tid;
            if (t < 0) {
                if (lane == 0) mbar_arrive(&fullW[sW]);
                break;
            }
            T* dst = bufW + (size_t)sW * TILE;
            const int64_t base = t * (int64_t)TILE;
            if (h.keep) {
                if (lane == 0) mbar_arrive(&fullW[sW]);      // data already in the read-1 slot
            } else if (h.fast) {
                if (lane == 0) {
                    mbar_expect_tx(&fullW[sW], TILE * 4);
                    tma_load_1d(dst, in + base, TILE * 4, &fullW[sW], pol);
                }
            } else {
                for (int k = lane; k < TILE; k += 32)
                    dst[k] = base + k < p.total ? from_bits<T>(ld_stream_u32(in + base + k)) : Op::identity();
                __syncwarp();
                if (lane == 0) mbar_arrive(&fullW[sW]);
            }
        }
    } else {
        // ---------------- NLB look-back warps, tile sequence i handled by warp i mod NLB
        // speculative: tile ids are static (round robin), so each look-back starts before the
        // tile's read 1 / reduction; only publishing P waits for this tile's aggregate
        static_assert(NLB <= SH && SH % NLB == 0, "look-back warps must not lap the header ring");
        const int lb = warp - (NS + NR + 2);
        const int64_t n_mine = (num_tiles - blockIdx.x + gridDim.x - 1) / gridDim.x;   // index of the sentinel
        for (int64_t i = lb; i <= n_mine; i += NLB) {
            const int sH = (int)(i % SH);
            const int64_t t = (int64_t)blockIdx.x + i * (int64_t)gridDim.x;
            C carry = Op::cidentity();
            uint32_t stats[2] = {0u, 0u};
            // lazy (default, lb_mode != 0): the look-back starts once this tile's own aggregate is out --
            // its predecessors' aggregates arrive around the same time, so the window is
            // (nearly) complete at the first poll and no warp spins on descriptors that
            // cannot be ready yet (such polls slow the streaming reads they share L2 with)
            const bool lazy = p.lb_mode != 0;
            if (lazy) mbar_wait(&aggd[sH], (uint32_t)((i / SH) & 1));
            if (i < n_mine) {
                if (lane == 0) trace_stamp(p, t, 4);
                if (((t * (int64_t)TILE) % p.N) != 0 && lazy) {
                    if (i > 0 && (int64_t)gridDim.x - 1 <= 32 * M)
                        carry = look_back_rr<Op, M>(p, t, i, gridDim.x, tag, s_incl, s_iseq, RING,
                                                    p.trace ? stats : nullptr);
                    else
                        carry = look_back_par<Op, M>(p, t, tag, p.trace ? stats : nullptr);
                } else if (((t * (int64_t)TILE) % p.N) != 0) {
                    // mode 0 (round 1, kept for A/B): speculative serialized polls
                    carry = look_back<Op, M>(p, t, tag, p.trace ? stats : nullptr);
                }
            }
            if (!lazy) mbar_wait(&aggd[sH], (uint32_t)((i / SH) & 1));
            SlotHdr<Op, NS>& h = s_hdr[sH];
            if (i == n_mine) {                       // forward the end sentinel to P2
                if (lane == 0) mbar_arrive(&crd[sH]);
                break;
            }
            if (lane == 0) {
                const C incl = h.has_head ? h.agg : Op::capply(carry, h.agg);
                if (!h.has_head) Desc<Op>::publish(p, t, tag, ST_P, incl);
                // the next tile of this CTA (another look-back warp) takes it from here
                s_incl[i % RING] = incl;
                __threadfence_block();
                *(volatile int64_t*)(s_iseq + (i % RING)) = i;
                h.carry = carry;
                trace_stamp(p, t, 2);
                trace_value(p, t, 5, stats[0]);
                trace_value(p, t, 6, stats[1]);
            }
            __syncwarp();
            if (lane == 0) mbar_arrive(&crd[sH]);
        }
    }
    __syncthreads();
    if (threadIdx.x == 0 && s_tag + 1u >= TAG_MASK) epilogue(p, s_tag);   // the wrap launch only
}

template <class Op, int NS, int NR, int SR, int SW, int SH, int M, int NLB>
cudaError_t launch_l2(const LookbackParams& p, cudaStream_t s) {
    constexpr int TILE = NS * 1024;
    constexpr int SMEM = (SR + SW) * TILE * 4;
    constexpr int THREADS = (NS + NR + 2 + NLB) * 32;
    auto kern = lookback_l2_kernel<Op, NS, NR, SR, SW, SH, M, NLB>;
    int64_t tiles = (p.total + TILE - 1) / TILE;
    LookbackParams pc = p;
    void* args[] = {&pc, &tiles};
    return launch_persistent((const void*)kern, args, tiles, THREADS, SMEM, p.pdl_first, s);
}

// ---------------------------------------------------------------- one tile per CTA (comparison)
template <class Op, int WARPS, int V>
__global__ void __launch_bounds__(WARPS * 32) lookback_tma_kernel(LookbackParams p) {
    using T = typename Op::T;
    using C = typename Op::Carry;
    constexpr int TILE = WARPS * 32 * V * 4;
    constexpr int WCH = V * 128;
    extern __shared__ __align__(128) unsigned char dsm[];
    T* s_tile = (T*)dsm;
    __shared__ uint64_t s_bar[WARPS];
    __shared__ int64_t s_tile_id, s_r;
    __shared__ uint32_t s_tag, s_seg, s_fast;
    __shared__ C s_carry;
    __shared__ __align__(16) T s_wval[(WARPS + 3) & ~3];   // 16-byte aligned and padded: vectorised slot reads never cover a neighbour
    __shared__ __align__(16) uint32_t s_wflag[(WARPS + 3) & ~3];
    const int warp = threadIdx.x >> 5, lane = lane_id();

    // tiles follow blockIdx (blocks are dispatched in index order, so every tile a CTA
    // waits on belongs to a CTA that is already running); the bulk copy of each warp's
    // share is issued first, the bookkeeping overlaps with it
    const int64_t tile = blockIdx.x;
    const int64_t base = tile * (int64_t)TILE;
    const bool fast = p.vec && base + TILE <= p.total;
    const T* in = (const T*)p.in;
    if (fast && lane == 0) {
        mbar_init(&s_bar[warp], 1);
        fence_mbar_init();
        mbar_expect_tx(&s_bar[warp], WCH * 4);
        tma_load_1d(s_tile + warp * WCH, in + base + warp * WCH, WCH * 4, &s_bar[warp], l2_evict_first_policy());
    }
    if (threadIdx.x == 0) {
        const TileInfo ti = classify(p, tile, TILE);
        s_tile_id = tile; s_r = ti.r; s_seg = ti.seg; s_fast = ti.fast;
        s_tag = read_tag(p);
    }
    uint32_t ticket = 0u;
    if (threadIdx.x == 0) ticket = count_tag_read(p, s_tag);
    __syncthreads();
    const int64_t r = s_r;
    const uint32_t tag = s_tag;
    if (fast) {
        mbar_wait(&s_bar[warp], 0);
    } else {
        for (int i = threadIdx.x; i < TILE; i += WARPS * 32)
            s_tile[i] = base + i < p.total ? from_bits<T>(ld_stream_u32(in + base + i)) : Op::identity();
        __syncthreads();
    }
    if (s_seg) tile_body_smem<Op, true, WARPS, V, false>(p, tile, tag, r, s_tile, fast, &s_carry, s_wval, s_wflag);
    else       tile_body_smem<Op, false, WARPS, V, false>(p, tile, tag, r, s_tile, fast, &s_carry, s_wval, s_wflag);
    __syncthreads();
    if (threadIdx.x == 0) finish_epoch(p, tag, ticket);
}

// ---------------------------------------------------------------- one register tile per CTA
// Latency-bound totals (configs[0]: 2^20 elements = 128 tiles, L2-resident).  Every thread
// holds its V 128-bit rows in registers (no shared-memory staging, one pass); the CTA's
// aggregate is published as soon as the block combine is done and the last warp looks
// back while the others wait at one barrier; then everyone adds the carry and stores.
// Tiles follow blockIdx (in-order dispatch, as lookback_tma_kernel).
template <class Op, bool SEG, int WARPS, int V>
__device__ __forceinline__ void regtile_body(const LookbackParams& p, int64_t tile, uint32_t* s_tag, uint32_t& ticket,
                                             int64_t r, typename Op::T* s_wval, uint32_t* s_wflag,
                                             typename Op::Carry* s_carry) {
    using T = typename Op::T;
    using C = typename Op::Carry;
    constexpr int TILE = WARPS * 32 * V * 4;
    constexpr int WCH = V * 128;
    const int warp = threadIdx.x >> 5, lane = lane_id();
    const int64_t wb = tile * (int64_t)TILE + warp * WCH;
    const T* in = (const T*)p.in;
    WarpTile<Op, SEG, V> wt;
    if (threadIdx.x == 0) trace_stamp(p, tile, 7);
    wt.load(in, wb, p.total, p.vec);
    // the launch tag is read once (thread 0, its round trip overlapping the tile's loads)
    // and counted at once (start-of-grid epoch advance, count_tag_read)
    if (threadIdx.x == 0) { *s_tag = read_tag(p); ticket = count_tag_read(p, *s_tag); }
    if (SEG) {
        if (p.N < TILE) wt.heads(warp * WCH, true, (uint32_t)r, (uint32_t)p.N, -1);
        else wt.heads(warp * WCH, false, 0u, 1u, r == 0 ? 0 : (int)(p.N - r));
    }
    wt.scan();
    if (lane == 0) { s_wval[warp] = wt.wtot; s_wflag[warp] = wt.wfl; }
    __syncthreads();
    const uint32_t tag = *s_tag;                  // read once per CTA (thread 0), visible now
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
        T agg = SEG ? seg_fold<Op>(wp, wt.wfl, wt.wtot) : Op::apply(wp, wt.wtot);
        const bool starts = (r == 0);
        const bool has_head = SEG ? (wpf || wt.wfl) : starts;
        const C aggc = Op::to_carry(agg);
        if (lane == 0) { trace_stamp(p, tile, 0); Desc<Op>::publish(p, tile, tag, has_head ? ST_P : ST_A, aggc); }
        if (lane == 0) { trace_stamp(p, tile, 1); trace_stamp(p, tile, 4); }
        C carry = Op::cidentity();
        uint32_t stats[2] = {0u, 0u};
        if (!starts) carry = look_back<Op>(p, tile, tag, p.trace ? stats : nullptr);
        if (lane == 0) {
            if (!has_head) Desc<Op>::publish(p, tile, tag, ST_P, Op::capply(carry, aggc));
            trace_stamp(p, tile, 2);
            trace_value(p, tile, 5, stats[0]);
            trace_value(p, tile, 6, stats[1]);
            *s_carry = carry;
        }
    }
    __syncthreads();
    wt.store((T*)p.out, wb, p.total, p.vec, wp, wpf, Op::from_carry(*s_carry), p.exclusive);
    if (threadIdx.x == 0) trace_stamp(p, tile, 3);
}

template <class Op, int WARPS, int V>
__global__ void __launch_bounds__(WARPS * 32) lookback_regtile_kernel(LookbackParams p) {
    using T = typename Op::T;
    using C = typename Op::Carry;
    constexpr int TILE = WARPS * 32 * V * 4;
    __shared__ __align__(16) T s_wval[(WARPS + 3) & ~3];   // 16-byte aligned and padded: vectorised slot reads never cover a neighbour
    __shared__ __align__(16) uint32_t s_wflag[(WARPS + 3) & ~3];
    __shared__ C s_carry;
    __shared__ uint32_t s_tag;
    const int64_t tile = blockIdx.x;
    const TileInfo ti = classify(p, tile, TILE);
    uint32_t ticket = 0u;
    if (ti.seg) regtile_body<Op, true, WARPS, V>(p, tile, &s_tag, ticket, ti.r, s_wval, s_wflag, &s_carry);
    else        regtile_body<Op, false, WARPS, V>(p, tile, &s_tag, ticket, ti.r, s_wval, s_wflag, &s_carry);
    __syncthreads();
    if (threadIdx.x == 0) finish_epoch(p, s_tag, ticket);
}

// ---------------------------------------------------------------- launchers
template <class Op, int WARPS, int V>
cudaError_t launch_tma(const LookbackParams& p, cudaStream_t s) {
    constexpr int TILE = WARPS * 32 * V * 4;
    constexpr int SMEM = TILE * 4;
    const int64_t tiles = (p.total + TILE - 1) / TILE;
    if (tiles > 0x7FFFFFFF) return cudaErrorInvalidConfiguration;
    cudaError_t e = kernel_prepare((const void*)lookback_tma_kernel<Op, WARPS, V>, WARPS * 32, SMEM, false, nullptr);
    if (e != cudaSuccess) return e;
    lookback_tma_kernel<Op, WARPS, V><<<(unsigned)tiles, WARPS * 32, SMEM, s>>>(p);
    return cudaGetLastError();
}

template <class Op, int WARPS, int V>
cudaError_t launch_regtile(const LookbackParams& p, cudaStream_t s) {
    constexpr int TILE = WARPS * 32 * V * 4;
    const int64_t tiles = (p.total + TILE - 1) / TILE;
    if (tiles > 0x7FFFFFFF) return cudaErrorInvalidConfiguration;
    lookback_regtile_kernel<Op, WARPS, V><<<(unsigned)tiles, WARPS * 32, 0, s>>>(p);
    return cudaGetLastError();
}

template <class Op, int WARPS, int V, int S, int M, int NLB, int PF = 0>
cudaError_t launch_pipelined(const LookbackParams& p, cudaStream_t s) {
    constexpr int TILE = WARPS * 32 * V * 4;
    constexpr int SMEM = S * TILE * 4;
    constexpr int THREADS = (WARPS + 1 + NLB) * 32;
    auto kern = lookback_pipelined_kernel<Op, WARPS, V, S, M, NLB, PF>;
    int64_t tiles = (p.total + TILE - 1) / TILE;
    LookbackParams pc = p;
    void* args[] = {&pc, &tiles};
    return launch_persistent((const void*)kern, args, tiles, THREADS, SMEM, false, s);
}

template <class Op>
cudaError_t launch_op(const LookbackParams& p, int variant, cudaStream_t s) {
    switch (variant) {
    case 0: return launch_pipelined<Op, 16, 8, 3, 5, 1, 1>(p, s);  // 64 KiB tiles, window 160, L2 prefetch +1 round
    case 1: return launch_pipelined<Op, 8, 8, 3, 4, 1, 0>(p, s);   // 32 KiB tiles (small, L2-resident totals)
    case 2: return launch_tma<Op, 8, 8>(p, s);                     // one 8192-element tile per CTA
    // two reads (L2-staged), 8-tile header ring; 8 scanner, 8 reducer and 2 look-back warps
    // (18 warps: 96 registers per thread; the lazy look-back needs few warps -- measured
    // against 4 reducers + 8 look-back warps: 2^24 0.79 -> 0.82, 2^25 0.85 -> 0.90 of copy)
    case 3: return launch_l2<Op, 8, 8, 3, 3, 8, 5, 2>(p, s);
    case 10: return launch_regtile<Op, 16, 4>(p, s);               // one 8192-element register tile per CTA
    default: return cudaErrorInvalidValue;
    }
}

}  // namespace

// Variants of the product library.  The research variants measured in round 1 (4-9 and
// 11-14: two look-back warps, register-resident waiting tiles, 16/72 KiB tiles, one 4096 /
// 16384-element tile per CTA, clustered look-back) were removed after they lost on every
// shape (DESIGN.md §5 keeps their numbers); their ids stay unused.
bool lookback_variant_valid(int variant) {
    return variant == 0 || variant == 1 || variant == 2 || variant == 3 || variant == 10;
}
int64_t lookback_tile_elems(int variant) {
    if (!lookback_variant_valid(variant)) return 0;
    return variant == 0 ? 16384 : 8192;
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
