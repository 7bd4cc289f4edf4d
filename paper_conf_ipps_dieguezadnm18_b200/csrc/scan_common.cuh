// scan_common.cuh -- device building blocks shared by every scan kernel of the library.
//
// Structure of one tile (PAPER.md:120-126 [§3.1, Figs. 4-5], re-shaped for sm_100a):
//   * every lane of a warp owns V "rows" of 4 consecutive elements, loaded as one 128-bit
//     vector each (int4 loads, P elements per thread; here P = 4V);
//     row j of warp w covers elements  w*V*128 + j*128 + lane*4 .. +3  of the tile, so a
//     warp-wide load instruction reads 512 contiguous bytes (fully coalesced);
//   * each lane scans its 4 elements serially in registers (the "thread scan");
//   * the 32 lane totals of a row are scanned with 5 warp shuffles (we use
//     the Kogge-Stone shuffle pattern, same depth as the paper's Ladner-Fischer one);
//   * rows are chained inside the warp, warp totals go through shared memory (one slot per
//     warp, S <= 32) and every warp folds the totals of the warps before it;
//   * the carry from earlier tiles comes from the look-back (scan_lookback.cu), from the
//     cascade register (scan_cascade.cu) or from the aux array
//     (scan_three_stage.cu).
//
// Every scan value travels as a SEGMENTED pair (flag, value): flag = "a problem starts at
// or before this position inside the current window".  The batch layout is G problems of
// N elements stored back to back, so a tile of the flat array may cross
// problem boundaries; the segmented combine  (f1,v1) . (f2,v2) = (f1|f2, f2 ? v2 : v1 op v2)
// stops every carry at a problem start.  When a kernel knows a window has no boundary it
// instantiates the SEG=false variant and all flag logic folds away at compile time.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace scanb200 {

constexpr unsigned FULL = 0xFFFFFFFFu;

// ------------------------------------------------------------------ operators and dtypes
// Value type T is what lives in memory; Carry is the type used to chain tiles.  For f32 add
// the inter-tile carry is fp64 (reading R3: an f32 carry chain breaks the
// 1e-5 * sum|x| bound at N = 2^30); every other case carries T itself (exact).
struct OpAddU32 {   // i32 and u32 add: the same bits modulo 2^32 (reading R1)
    using T = uint32_t; using Carry = uint32_t;
    static __device__ __forceinline__ T identity() { return 0u; }
    static __device__ __forceinline__ T apply(T a, T b) { return a + b; }
    static __device__ __forceinline__ Carry cidentity() { return 0u; }
    static __device__ __forceinline__ Carry capply(Carry a, Carry b) { return a + b; }
    static __device__ __forceinline__ Carry to_carry(T v) { return v; }
    static __device__ __forceinline__ T from_carry(Carry c) { return c; }
    static constexpr bool kSplitDesc = false;
};
struct OpMaxI32 {
    using T = int32_t; using Carry = int32_t;
    static __device__ __forceinline__ T identity() { return INT32_MIN; }
    static __device__ __forceinline__ T apply(T a, T b) { return b > a ? b : a; }
    static __device__ __forceinline__ Carry cidentity() { return INT32_MIN; }
    static __device__ __forceinline__ Carry capply(Carry a, Carry b) { return b > a ? b : a; }
    static __device__ __forceinline__ Carry to_carry(T v) { return v; }
    static __device__ __forceinline__ T from_carry(Carry c) { return c; }
    static constexpr bool kSplitDesc = false;
};
struct OpMaxU32 {
    using T = uint32_t; using Carry = uint32_t;
    static __device__ __forceinline__ T identity() { return 0u; }
    static __device__ __forceinline__ T apply(T a, T b) { return b > a ? b : a; }
    static __device__ __forceinline__ Carry cidentity() { return 0u; }
    static __device__ __forceinline__ Carry capply(Carry a, Carry b) { return b > a ? b : a; }
    static __device__ __forceinline__ Carry to_carry(T v) { return v; }
    static __device__ __forceinline__ T from_carry(Carry c) { return c; }
    static constexpr bool kSplitDesc = false;
};
struct OpMaxF32 {
    using T = float; using Carry = float;
    static __device__ __forceinline__ T identity() { return __int_as_float(0xff800000); }  // -inf
    static __device__ __forceinline__ T apply(T a, T b) { return b > a ? b : a; }
    static __device__ __forceinline__ Carry cidentity() { return __int_as_float(0xff800000); }
    static __device__ __forceinline__ Carry capply(Carry a, Carry b) { return b > a ? b : a; }
    static __device__ __forceinline__ Carry to_carry(T v) { return v; }
    static __device__ __forceinline__ T from_carry(Carry c) { return c; }
    static constexpr bool kSplitDesc = false;
};
struct OpAddF32 {
    using T = float; using Carry = double;
    static __device__ __forceinline__ T identity() { return 0.0f; }
    static __device__ __forceinline__ T apply(T a, T b) { return __fadd_rn(a, b); }   // no FMA contraction
    static __device__ __forceinline__ Carry cidentity() { return 0.0; }
    static __device__ __forceinline__ Carry capply(Carry a, Carry b) { return __dadd_rn(a, b); }
    static __device__ __forceinline__ Carry to_carry(T v) { return (double)v; }
    static __device__ __forceinline__ T from_carry(Carry c) { return __double2float_rn(c); }
    static constexpr bool kSplitDesc = true;
};

// 32-bit raw views (for shuffles and packed descriptors)
template <class T> __device__ __forceinline__ uint32_t to_bits(T v);
template <> __device__ __forceinline__ uint32_t to_bits<uint32_t>(uint32_t v) { return v; }
template <> __device__ __forceinline__ uint32_t to_bits<int32_t>(int32_t v) { return (uint32_t)v; }
template <> __device__ __forceinline__ uint32_t to_bits<float>(float v) { return __float_as_uint(v); }
template <class T> __device__ __forceinline__ T from_bits(uint32_t b);
template <> __device__ __forceinline__ uint32_t from_bits<uint32_t>(uint32_t b) { return b; }
template <> __device__ __forceinline__ int32_t from_bits<int32_t>(uint32_t b) { return (int32_t)b; }
template <> __device__ __forceinline__ float from_bits<float>(uint32_t b) { return __uint_as_float(b); }

template <class T> __device__ __forceinline__ T shfl_up(T v, int d) {
    return from_bits<T>(__shfl_up_sync(FULL, to_bits<T>(v), d));
}
template <class T> __device__ __forceinline__ T shfl_idx(T v, int src) {
    return from_bits<T>(__shfl_sync(FULL, to_bits<T>(v), src));
}
__device__ __forceinline__ double shfl_idx(double v, int src) { return __shfl_sync(FULL, v, src); }
__device__ __forceinline__ double shfl_down_d(double v, int d) { return __shfl_down_sync(FULL, v, d); }

__device__ __forceinline__ int lane_id() { return threadIdx.x & 31; }

// ------------------------------------------------------------------ global memory access
// 128-bit streaming load through the non-coherent path without L1 allocation (each input
// byte is read exactly once) and a streaming 128-bit store (evict-first in L2).
__device__ __forceinline__ uint4 ld_stream_v4(const void* p) {
    uint4 r;
    asm("ld.global.nc.L1::no_allocate.L2::256B.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
    return r;
}
__device__ __forceinline__ void st_stream_v4(void* p, uint4 v) {
    asm volatile("st.global.cs.v4.u32 [%0], {%1,%2,%3,%4};"
                 :: "l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
}
__device__ __forceinline__ uint32_t ld_stream_u32(const void* p) {
    uint32_t r;
    asm("ld.global.nc.u32 %0, [%1];" : "=r"(r) : "l"(p));
    return r;
}
__device__ __forceinline__ void st_stream_u32(void* p, uint32_t v) {
    asm volatile("st.global.cs.u32 [%0], %1;" :: "l"(p), "r"(v) : "memory");
}

// release/acquire at GPU scope for the inter-CTA protocol
__device__ __forceinline__ void st_release_u64(uint64_t* p, uint64_t v) {
    asm volatile("st.release.gpu.global.u64 [%0], %1;" :: "l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ uint64_t ld_acquire_u64(const uint64_t* p) {
    uint64_t v;
    asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release_u32(uint32_t* p, uint32_t v) {
    asm volatile("st.release.gpu.global.u32 [%0], %1;" :: "l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ uint32_t ld_acquire_u32(const uint32_t* p) {
    uint32_t v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ double ld_relaxed_f64(const double* p) {
    double v;
    asm volatile("ld.relaxed.gpu.global.f64 %0, [%1];" : "=d"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_relaxed_f64(double* p, double v) {
    asm volatile("st.relaxed.gpu.global.f64 [%0], %1;" :: "l"(p), "d"(v) : "memory");
}

// Programmatic dependent launch (sm_90+): a kernel launched with the
// programmatic-stream-serialization attribute may start while the previous kernel of the
// stream still runs; `grid_dep_wait` blocks until that kernel completed and its memory is
// visible (a no-op for a normal launch); `grid_dep_launch` lets the next kernel start.
__device__ __forceinline__ void grid_dep_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void grid_dep_launch() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }

// system scope: the fused peer-memory exchange of the sharded path (other GPUs' memory
// mapped into this address space over NVLink, or another process's memory on this GPU)
__device__ __forceinline__ void st_release_sys_u64(uint64_t* p, uint64_t v) {
    asm volatile("st.release.sys.global.u64 [%0], %1;" :: "l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ uint64_t ld_acquire_sys_u64(const uint64_t* p) {
    uint64_t v;
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_relaxed_sys_u64(uint64_t* p, uint64_t v) {
    asm volatile("st.relaxed.sys.global.u64 [%0], %1;" :: "l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ uint64_t ld_relaxed_sys_u64(const uint64_t* p) {
    uint64_t v;
    asm volatile("ld.relaxed.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

// ------------------------------------------------------------------ a row of 4 elements
template <class T>
struct Row4 { T v[4]; };

template <class T> __device__ __forceinline__ Row4<T> row_from_u4(uint4 u) {
    Row4<T> r; r.v[0] = from_bits<T>(u.x); r.v[1] = from_bits<T>(u.y);
    r.v[2] = from_bits<T>(u.z); r.v[3] = from_bits<T>(u.w); return r;
}
template <class T> __device__ __forceinline__ uint4 row_to_u4(const Row4<T>& r) {
    return make_uint4(to_bits<T>(r.v[0]), to_bits<T>(r.v[1]), to_bits<T>(r.v[2]), to_bits<T>(r.v[3]));
}

// Load a row: vector path when the 4 elements are in range and 16-byte aligned, else
// guarded scalar loads with the identity for out-of-range positions.
template <class Op>
__device__ __forceinline__ Row4<typename Op::T> load_row(const typename Op::T* base, int64_t idx,
                                                         int64_t limit, bool vec) {
    using T = typename Op::T;
    Row4<T> r;
    if (vec && idx + 4 <= limit) {
        r = row_from_u4<T>(ld_stream_v4(base + idx));
    } else {
#pragma unroll
        for (int k = 0; k < 4; ++k)
            r.v[k] = (idx + k < limit) ? from_bits<T>(ld_stream_u32(base + idx + k)) : Op::identity();
    }
    return r;
}
template <class Op>
__device__ __forceinline__ void store_row(typename Op::T* base, int64_t idx, int64_t limit, bool vec,
                                          const Row4<typename Op::T>& r) {
    using T = typename Op::T;
    if (vec && idx + 4 <= limit) {
        st_stream_v4(base + idx, row_to_u4<T>(r));
    } else {
#pragma unroll
        for (int k = 0; k < 4; ++k)
            if (idx + k < limit) st_stream_u32(base + idx + k, to_bits<T>(r.v[k]));
    }
}

// ------------------------------------------------------------------ segmented pair helpers
// fold(acc, (f, v)):  f ? v : acc op v      (acc is the OLDER value)
template <class Op>
__device__ __forceinline__ typename Op::T seg_fold(typename Op::T acc, bool f, typename Op::T v) {
    return f ? v : Op::apply(acc, v);
}

// Head flags (bit k <=> element k of the row starts a problem) of the row at tile offset
// `o`.  Small-N form (N < tile): `r_tile` = (tile origin) mod N, so the row's first element
// sits at position (r_tile + o) mod N of its problem.  Large-N form (N >= tile): at most
// one head in the tile, at offset `first` (or none when first < 0).
__device__ __forceinline__ unsigned row_heads_small(uint32_t o, uint32_t r_tile, uint32_t N) {
    uint32_t r = (r_tile + o) % N;
    uint32_t k = r ? N - r : 0u;
    unsigned m = 0;
#pragma unroll
    for (int i = 0; i < 4; ++i) {      // at most 4 heads per row (N == 1)
        if (k < 4u) { m |= 1u << k; k += N; }
    }
    return m;
}
// The same from r = (row offset) mod N, maintained incrementally by the caller (no
// division per row).
__device__ __forceinline__ unsigned row_heads_from_r(uint32_t r, uint32_t N) {
    uint32_t k = r ? N - r : 0u;
    unsigned m = 0;
#pragma unroll
    for (int i = 0; i < 4; ++i) {
        if (k < 4u) { m |= 1u << k; k += N; }
    }
    return m;
}
__device__ __forceinline__ unsigned row_heads_big(int o, int first) {
    int d = first - o;
    return (d >= 0 && d < 4) ? (1u << d) : 0u;
}

// Serial reduction of a row under head flags -> (any_head, trailing-segment value).
template <class Op, bool SEG>
__device__ __forceinline__ typename Op::T row_reduce(const Row4<typename Op::T>& r, unsigned heads) {
    using T = typename Op::T;
    T acc = r.v[0];
#pragma unroll
    for (int k = 1; k < 4; ++k) {
        if (SEG) acc = seg_fold<Op>(acc, (heads >> k) & 1u, r.v[k]);
        else     acc = Op::apply(acc, r.v[k]);
    }
    return acc;
}

// Final serial pass of a row.  `in`/`in_f` is the segmented prefix of everything before
// the row's first element inside the current tile, `cin` the carry from before the tile.
// At a head the running value restarts from the identity (each problem's
// scan starts at its element 0).  For f32 add the carry is added last, onto the complete
// tile-local prefix (better rounding: the local partial sums are small); for the exact
// operators it is folded in first (one op per element).
template <class Op, bool SEG, bool EXCL>
__device__ __forceinline__ Row4<typename Op::T> row_output(const Row4<typename Op::T>& r, unsigned heads,
                                                           typename Op::T in, bool in_f,
                                                           typename Op::T cin) {
    using T = typename Op::T;
    Row4<T> o;
    if constexpr (Op::kSplitDesc) {
        T run = in; bool f = SEG && in_f;
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            if (SEG && ((heads >> k) & 1u)) { run = Op::identity(); f = true; }
            if (EXCL) { o.v[k] = f ? run : Op::apply(cin, run); run = Op::apply(run, r.v[k]); }
            else      { run = Op::apply(run, r.v[k]); o.v[k] = f ? run : Op::apply(cin, run); }
        }
    } else {
        T run = (SEG && in_f) ? in : Op::apply(cin, in);
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            if (SEG && ((heads >> k) & 1u)) run = Op::identity();
            if (EXCL) { o.v[k] = run; run = Op::apply(run, r.v[k]); }
            else      { run = Op::apply(run, r.v[k]); o.v[k] = run; }
        }
    }
    return o;
}

// Warp-wide segmented inclusive scan (Kogge-Stone over lanes, "shuffle
// instructions" -- LF and KS both take log2(32) = 5 steps).  `hm` = ballot of lanes whose
// row holds a head.  Returns the inclusive value; `excl` receives the exclusive value
// (identity on lane 0) and `excl_flag` whether a head lies in lanes < lane.
template <class Op, bool SEG>
__device__ __forceinline__ typename Op::T warp_seg_scan(typename Op::T v, unsigned hm,
                                                        typename Op::T& excl, bool& excl_flag) {
    using T = typename Op::T;
    const int lane = lane_id();
    int lo = 0;
    if (SEG) {
        unsigned le = hm & (FULL >> (31 - lane));
        lo = le ? (31 - __clz(le)) : 0;
    }
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        T y = shfl_up<T>(v, d);
        if (lane - d >= lo) v = Op::apply(y, v);
    }
    T e = shfl_up<T>(v, 1);
    excl = lane ? e : Op::identity();
    excl_flag = SEG ? ((hm & ((1u << lane) - 1u)) != 0u) : false;
    return v;
}

// Warp reduction of Carry values (full warp, result on all lanes).
template <class Op>
__device__ __forceinline__ typename Op::Carry warp_reduce_carry(typename Op::Carry v) {
#pragma unroll
    for (int d = 16; d >= 1; d >>= 1) {
        typename Op::Carry o;
        if constexpr (sizeof(typename Op::Carry) == 8) o = __shfl_xor_sync(FULL, v, d);
        else o = from_bits<typename Op::Carry>(__shfl_xor_sync(FULL, to_bits<typename Op::Carry>(v), d));
        v = Op::capply(v, o);
    }
    return v;
}

// ------------------------------------------------------------------ the warp tile engine
// One warp's share of a tile: V rows x 32 lanes x 4 elements = 128 V contiguous elements
// starting at global index `wbase`.  Used by every scan kernel (look-back, cascade,
// three-stage Stage 3).
template <class Op, bool SEG, int V>
struct WarpTile {
    using T = typename Op::T;
    Row4<T> x[V];
    unsigned hd[V];          // head bits per row
    T lin[V];  bool lfl[V];  // lane-exclusive prefix inside the row
    T rp[V];   bool rpf[V];  // prefix of the rows before row j (inside this warp)
    T wtot;    bool wfl;     // warp total (segmented)

    __device__ __forceinline__ void load(const T* in, int64_t wbase, int64_t limit, bool vec) {
        const int lane = lane_id();
#pragma unroll
        for (int j = 0; j < V; ++j) x[j] = load_row<Op>(in, wbase + j * 128 + lane * 4, limit, vec);
    }
    // heads for a window whose element offset `o0` (relative to the tile origin) starts the
    // warp; small-N (N < tile) or big-N (single head at `first`, -1 if none) form
    __device__ __forceinline__ void heads(int o0, bool small, uint32_t r_tile, uint32_t N32, int first) {
        const int lane = lane_id();
#pragma unroll
        for (int j = 0; j < V; ++j) {
            int o = o0 + j * 128 + lane * 4;
            hd[j] = !SEG ? 0u : (small ? row_heads_small((uint32_t)o, r_tile, N32) : row_heads_big(o, first));
        }
    }
    __device__ __forceinline__ void scan() {
        T run = Op::identity(); bool f = false;
#pragma unroll
        for (int j = 0; j < V; ++j) {
            T v = row_reduce<Op, SEG>(x[j], hd[j]);
            unsigned hm = SEG ? __ballot_sync(FULL, hd[j] != 0u) : 0u;
            T incl = warp_seg_scan<Op, SEG>(v, hm, lin[j], lfl[j]);
            T rt = shfl_idx<T>(incl, 31);
            rp[j] = run; rpf[j] = f;
            run = SEG ? seg_fold<Op>(run, hm != 0u, rt) : Op::apply(run, rt);
            f = f || (hm != 0u);
        }
        wtot = run; wfl = f;
    }
    // wp/wpf: segmented prefix of the warps before this one inside the tile;
    // cin: carry of everything before the tile (already rounded to T)
    __device__ __forceinline__ void store(T* out, int64_t wbase, int64_t limit, bool vec,
                                          T wp, bool wpf, T cin, bool excl_kind) {
        const int lane = lane_id();
#pragma unroll
        for (int j = 0; j < V; ++j) {
            T in; bool inf;
            if (SEG) {
                in = seg_fold<Op>(wp, rpf[j], rp[j]); inf = wpf || rpf[j];
                in = seg_fold<Op>(in, lfl[j], lin[j]); inf = inf || lfl[j];
            } else {
                in = Op::apply(Op::apply(wp, rp[j]), lin[j]); inf = false;
            }
            Row4<T> o = excl_kind ? row_output<Op, SEG, true>(x[j], hd[j], in, inf, cin)
                                  : row_output<Op, SEG, false>(x[j], hd[j], in, inf, cin);
            store_row<Op>(out, wbase + j * 128 + lane * 4, limit, vec, o);
        }
    }
};

}  // namespace scanb200

namespace scanb200 {

// ------------------------------------------------------------------ TMA bulk copies (sm_90+/sm_100a)
// 1-D bulk copies global -> shared (SASS UBLKCP) completing on an mbarrier (SYNCS.*).  They
// keep the bytes in flight without holding registers, so the number of outstanding loads
// per SM is bounded by shared memory instead of the register file.
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ uint64_t l2_evict_first_policy() {
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    return pol;
}
__device__ __forceinline__ void tma_load_1d(void* dst_smem, const void* src, uint32_t bytes, uint64_t* bar,
                                            uint64_t policy) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;"
        :: "r"(smem_u32(dst_smem)), "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(policy) : "memory");
}
__device__ __forceinline__ uint64_t l2_evict_last_policy() {
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
    return pol;
}
// bulk L2 prefetch (no shared memory, no completion): starts the HBM -> L2 part of a later
// TMA load early, so the shared-memory slot of that load is held for an L2 hit only
__device__ __forceinline__ void prefetch_l2_bulk(const void* src, uint32_t bytes) {
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" :: "l"(src), "r"(bytes) : "memory");
}
// Bulk L2 prefetch of the elements [p, p + n), clipped to whole 16-byte units.  Issued by
// the cross-call programmatic kernels BEFORE their griddepcontrol.wait: a prefetch moves no
// data to the SM and L2 is the point of coherence, so the loads after the wait still see
// every write of the previous kernel, while the HBM -> L2 part of the first tiles overlaps
// the previous grid's completion (~0.8 us between a CTA's entry and the end of its wait).
template <class T>
__device__ __forceinline__ void prefetch_l2_span(const T* p, int64_t n) {
    if (n <= 0) return;
    const uintptr_t a = ((uintptr_t)p + 15u) & ~(uintptr_t)15u, b = (uintptr_t)(p + n) & ~(uintptr_t)15u;
    if (b > a) prefetch_l2_bulk((const void*)a, (uint32_t)(b - a));
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" :: "r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t phase) {
    asm volatile(
        "{\n .reg .pred p;\n WAIT_%=:\n"
        " mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
        " @!p bra WAIT_%=;\n}\n" :: "r"(smem_u32(bar)), "r"(phase) : "memory");
}
// wait for an mbarrier phase, or give up once the stream's end index (published in shared
// memory by the role that met the end sentinel) is < i; returns false in that case.  The
// warp that owns the sentinel index itself (end == i) must wait: it forwards the sentinel.
__device__ __forceinline__ bool mbar_wait_or_end(uint64_t* bar, uint32_t phase, const int64_t* end, int64_t i) {
    while (true) {
        uint32_t ok;
        asm volatile(
            "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
            : "=r"(ok) : "r"(smem_u32(bar)), "r"(phase) : "memory");
        if (ok) return true;
        if (*(const volatile int64_t*)end < i) return false;
    }
}
__device__ __forceinline__ uint4 lds_v4(const void* p) {
    uint4 r;
    asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
                 : "r"(smem_u32(p)));
    return r;
}

// ------------------------------------------------------------------ the warp tile engine, smem-staged
// Same row structure as WarpTile, but the rows live in shared memory (landed there by a
// bulk copy) and are read twice: pass 1 computes the lane / row / warp prefixes (only
// 2V values + 3 bitmasks stay in registers), pass 2 re-reads each row once the carry is
// known and writes the outputs with 128-bit streaming stores.  Row reads are 512
// contiguous bytes per warp instruction: bank-conflict free.
template <class Op, bool SEG, int V>
struct WarpTileS {
    using T = typename Op::T;
    static_assert(V <= 8, "head masks pack 4 bits per row into 32 bits");
    T lin[V];
    T rp[V];
    uint32_t hdm = 0;     // 4 head bits per row
    uint32_t lflm = 0;    // bit j: a head lies in lanes < lane of row j
    uint32_t rpfm = 0;    // bit j: a head lies in rows < j of this warp
    T wtot; bool wfl;

    __device__ __forceinline__ void pass1(const T* srow, int o0, bool small, uint32_t r_tile, uint32_t N32,
                                          int first) {
        const int lane = lane_id();
        T run = Op::identity(); bool f = false;
#pragma unroll
        for (int j = 0; j < V; ++j) {
            Row4<T> x = row_from_u4<T>(lds_v4(srow + j * 128 + lane * 4));
            unsigned hd = 0u;
            if (SEG) {
                int o = o0 + j * 128 + lane * 4;
                hd = small ? row_heads_small((uint32_t)o, r_tile, N32) : row_heads_big(o, first);
                hdm |= hd << (4 * j);
            }
            T v = row_reduce<Op, SEG>(x, hd);
            unsigned hm = SEG ? __ballot_sync(FULL, hd != 0u) : 0u;
            bool lf;
            T incl = warp_seg_scan<Op, SEG>(v, hm, lin[j], lf);
            if (SEG && lf) lflm |= 1u << j;
            T rt = shfl_idx<T>(incl, 31);
            rp[j] = run;
            if (SEG && f) rpfm |= 1u << j;
            run = SEG ? seg_fold<Op>(run, hm != 0u, rt) : Op::apply(run, rt);
            f = f || (hm != 0u);
        }
        wtot = run; wfl = f;
    }
    // gout = output address of the warp's first element (global index gidx); `fast` = whole
    // window in range and 16-byte aligned, else guarded stores against `limit`
    __device__ __forceinline__ void pass2(const T* srow, T* out, int64_t gidx, int64_t limit, bool fast,
                                          bool vec, bool excl_kind, T wp, bool wpf, T cin) {
        const int lane = lane_id();
#pragma unroll
        for (int j = 0; j < V; ++j) {
            Row4<T> x = row_from_u4<T>(lds_v4(srow + j * 128 + lane * 4));
            T in; bool inf;
            if (SEG) {
                bool rf = (rpfm >> j) & 1u, lf = (lflm >> j) & 1u;
                in = seg_fold<Op>(wp, rf, rp[j]); inf = wpf || rf;
                in = seg_fold<Op>(in, lf, lin[j]); inf = inf || lf;
            } else {
                in = Op::apply(Op::apply(wp, rp[j]), lin[j]); inf = false;
            }
            unsigned hd = SEG ? (hdm >> (4 * j)) & 0xFu : 0u;
            Row4<T> o = excl_kind ? row_output<Op, SEG, true>(x, hd, in, inf, cin)
                                  : row_output<Op, SEG, false>(x, hd, in, inf, cin);
            const int64_t idx = gidx + j * 128 + lane * 4;
            if (fast) st_stream_v4(out + idx, row_to_u4<T>(o));
            else store_row<Op>(out, idx, limit, vec, o);
        }
    }
};

// The same engine with the segmentation chosen per call (SEG is a per-tile runtime property
// in the pipelined kernel, which keeps the state of two tiles in flight per warp).
template <class Op, int V>
struct WarpTileP {
    using T = typename Op::T;
    static_assert(V <= 8, "head masks pack 4 bits per row into 32 bits");
    T lin[V];
    T rp[V];
    uint32_t hdm, lflm, rpfm;
    T wtot; bool wfl;

    template <bool SEG>
    __device__ __forceinline__ void pass1(const T* srow, int o0, bool small, uint32_t r_tile, uint32_t N32,
                                          int first) {
        const int lane = lane_id();
        hdm = 0u; lflm = 0u; rpfm = 0u;
        T run = Op::identity(); bool f = false;
#pragma unroll
        for (int j = 0; j < V; ++j) {
            Row4<T> x = row_from_u4<T>(lds_v4(srow + j * 128 + lane * 4));
            unsigned hd = 0u;
            if (SEG) {
                int o = o0 + j * 128 + lane * 4;
                hd = small ? row_heads_small((uint32_t)o, r_tile, N32) : row_heads_big(o, first);
                hdm |= hd << (4 * j);
            }
            T v = row_reduce<Op, SEG>(x, hd);
            unsigned hm = SEG ? __ballot_sync(FULL, hd != 0u) : 0u;
            bool lf;
            T incl = warp_seg_scan<Op, SEG>(v, hm, lin[j], lf);
            if (SEG && lf) lflm |= 1u << j;
            T rt = shfl_idx<T>(incl, 31);
            rp[j] = run;
            if (SEG && f) rpfm |= 1u << j;
            run = SEG ? seg_fold<Op>(run, hm != 0u, rt) : Op::apply(run, rt);
            f = f || (hm != 0u);
        }
        wtot = run; wfl = f;
    }
    template <bool SEG>
    __device__ __forceinline__ void pass2(const T* srow, T* out, int64_t gidx, int64_t limit, bool fast,
                                          bool vec, bool excl_kind, T wp, bool wpf, T cin) const {
        const int lane = lane_id();
#pragma unroll
        for (int j = 0; j < V; ++j) {
            Row4<T> x = row_from_u4<T>(lds_v4(srow + j * 128 + lane * 4));
            T in; bool inf;
            if (SEG) {
                bool rf = (rpfm >> j) & 1u, lf = (lflm >> j) & 1u;
                in = seg_fold<Op>(wp, rf, rp[j]); inf = wpf || rf;
                in = seg_fold<Op>(in, lf, lin[j]); inf = inf || lf;
            } else {
                in = Op::apply(Op::apply(wp, rp[j]), lin[j]); inf = false;
            }
            unsigned hd = SEG ? (hdm >> (4 * j)) & 0xFu : 0u;
            Row4<T> o = excl_kind ? row_output<Op, SEG, true>(x, hd, in, inf, cin)
                                  : row_output<Op, SEG, false>(x, hd, in, inf, cin);
            const int64_t idx = gidx + j * 128 + lane * 4;
            if (fast) st_stream_v4(out + idx, row_to_u4<T>(o));
            else store_row<Op>(out, idx, limit, vec, o);
        }
    }
};

}  // namespace scanb200
