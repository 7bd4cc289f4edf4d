// scan_fused.cu -- the paper's three stages (PAPER.md:110-118 [§3.1, Fig. 3]) fused into ONE
// cooperative launch for latency-bound totals, with the data held on chip between them.
//
//   Stage 1  every CTA loads its 8192-element tile into REGISTERS (8 warps x 8 rows x 128-bit
//            per lane), scans it locally (thread-serial rows, warp shuffles, block combine)
//            and publishes the tile aggregate to the aux array (one 8-byte slot per CTA);
//   Stage 2  one grid-wide barrier (cooperative launch: the whole grid is co-resident);
//            every CTA folds the aggregates of the CTAs before it in its problem -- one
//            warp-parallel read of <= 32 x 19 slots from L2 -- instead of a separate
//            intermediate-scan kernel;
//   Stage 3  the tile, still in registers, is offset by that carry and stored.
// The input is read ONCE (8 B/element instead of the three-kernel form's 12) and there is no
// second launch; the cost is one grid barrier.  Capacity: one tile per CTA and every CTA
// resident at once (~148 x 4 tiles of 8192 elements = 4.8 M elements on B200); eligible
// shapes: one problem (any N), or N a multiple of the tile (each CTA inside one problem).
// f32 add: aggregates and the carry are fp64 (reading R3).
#include <cooperative_groups.h>

#include <algorithm>

#include "scan_common.cuh"
#include "scan_internal.h"

namespace cg = cooperative_groups;

namespace scanb200 {

namespace {

constexpr int FU_WARPS = 8, FU_V = 8;                  // 8192-element tiles, 32 elements / thread
constexpr int FU_TILE = FU_WARPS * FU_V * 128;
constexpr int FU_AUX_ITEMS = 19;                        // aggregates per lane of the fold (<= 608 CTAs)

__device__ __forceinline__ uint64_t ld_relaxed_u64_global(const uint64_t* p) {
    uint64_t v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

template <class C> __device__ __forceinline__ uint64_t fu_put(C v);
template <> __device__ __forceinline__ uint64_t fu_put<uint32_t>(uint32_t v) { return v; }
template <> __device__ __forceinline__ uint64_t fu_put<int32_t>(int32_t v) { return (uint32_t)v; }
template <> __device__ __forceinline__ uint64_t fu_put<float>(float v) { return __float_as_uint(v); }
template <> __device__ __forceinline__ uint64_t fu_put<double>(double v) { return (uint64_t)__double_as_longlong(v); }
template <class C> __device__ __forceinline__ C fu_get(uint64_t s);
template <> __device__ __forceinline__ uint32_t fu_get<uint32_t>(uint64_t s) { return (uint32_t)s; }
template <> __device__ __forceinline__ int32_t fu_get<int32_t>(uint64_t s) { return (int32_t)(uint32_t)s; }
template <> __device__ __forceinline__ float fu_get<float>(uint64_t s) { return __uint_as_float((uint32_t)s); }
template <> __device__ __forceinline__ double fu_get<double>(uint64_t s) { return __longlong_as_double((long long)s); }

template <class Op>
__global__ void __launch_bounds__(FU_WARPS * 32, 4) fused_grid_kernel(FusedParams p) {
    using T = typename Op::T;
    using C = typename Op::Carry;
    constexpr int WCH = FU_V * 128;
    __shared__ __align__(16) T s_wval[FU_WARPS];
    __shared__ C s_carry;
    const int warp = threadIdx.x >> 5, lane = lane_id();
    const int64_t cta = blockIdx.x;
    const int64_t wb = cta * (int64_t)FU_TILE + warp * WCH;
    const T* in = (const T*)p.in;
    grid_dep_launch();
    if (p.pdl_first && threadIdx.x == 0) prefetch_l2_span(in + cta * (int64_t)FU_TILE, min(p.total - cta * (int64_t)FU_TILE, (int64_t)FU_TILE));
    if (p.pdl_first) grid_dep_wait();            // the stream's previous kernel wrote our input

    // Stage 1: the tile into registers, local scan, tile aggregate
    WarpTile<Op, false, FU_V> wt;
    wt.load(in, wb, p.total, p.vec);
    wt.scan();
    if (lane == 0) s_wval[warp] = wt.wtot;
    __syncthreads();
    T wp = Op::identity(), tot = Op::identity();
#pragma unroll
    for (int w = 0; w < FU_WARPS; ++w) {
        const T v = s_wval[w];
        if (w < warp) wp = Op::apply(wp, v);
        tot = Op::apply(tot, v);
    }
    if (threadIdx.x == 0) p.aux[cta] = fu_put<C>(Op::to_carry(tot));

    // Stage 2: grid barrier, then the fold of the aggregates before this CTA in its problem
    cg::this_grid().sync();
    if (warp == 0) {
        const int64_t first = (cta / p.tiles_per_problem) * p.tiles_per_problem;
        C acc = Op::cidentity();
#pragma unroll
        for (int k = 0; k < FU_AUX_ITEMS; ++k) {
            const int64_t j = first + lane + 32 * k;
            if (j < cta) acc = Op::capply(acc, fu_get<C>(ld_relaxed_u64_global(p.aux + j)));
        }
        acc = warp_reduce_carry<Op>(acc);
        if (lane == 0) s_carry = acc;
    }
    __syncthreads();

    // Stage 3: offset by the carry and store
    wt.store((T*)p.out, wb, p.total, p.vec, wp, false, Op::from_carry(s_carry), p.exclusive);
}

template <class Op>
cudaError_t fused_op(const FusedParams& p, cudaStream_t s) {
    auto kern = fused_grid_kernel<Op>;
    const int64_t tiles = (p.total + FU_TILE - 1) / FU_TILE;
    int occ = 0, sms = 0;
    cudaError_t e = kernel_prepare((const void*)kern, FU_WARPS * 32, 0, false, &occ);
    if (e != cudaSuccess) return e;
    e = current_device_sms(&sms);
    if (e != cudaSuccess) return e;
    if (tiles > (int64_t)occ * sms || tiles > 32 * FU_AUX_ITEMS) return cudaErrorInvalidConfiguration;
    FusedParams pc = p;
    void* args[] = {&pc};
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)tiles, 1, 1);
    cfg.blockDim = dim3(FU_WARPS * 32, 1, 1);
    cfg.stream = s;
    cudaLaunchAttribute attr[2];
    attr[0].id = cudaLaunchAttributeCooperative;
    attr[0].val.cooperative = 1;
    attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[1].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = p.pdl_first ? 2 : 1;
    return cudaLaunchKernelExC(&cfg, (const void*)kern, args);
}

}  // namespace

int64_t fused_tile_elems() { return FU_TILE; }

template <class Op>
int64_t fused_max_tiles_op() {
    int occ = 0, sms = 0;
    if (kernel_prepare((const void*)fused_grid_kernel<Op>, FU_WARPS * 32, 0, false, &occ) != cudaSuccess) {
        cudaGetLastError();
        return 0;
    }
    if (current_device_sms(&sms) != cudaSuccess) { cudaGetLastError(); return 0; }
    return std::min<int64_t>((int64_t)occ * sms, 32 * FU_AUX_ITEMS);
}

int64_t fused_max_tiles(OpCode op) {
    switch (op) {
    case OpCode::AddU32: return fused_max_tiles_op<OpAddU32>();
    case OpCode::MaxI32: return fused_max_tiles_op<OpMaxI32>();
    case OpCode::MaxU32: return fused_max_tiles_op<OpMaxU32>();
    case OpCode::MaxF32: return fused_max_tiles_op<OpMaxF32>();
    case OpCode::AddF32: return fused_max_tiles_op<OpAddF32>();
    }
    return 0;
}

cudaError_t launch_fused(OpCode op, const FusedParams& p, cudaStream_t s) {
    switch (op) {
    case OpCode::AddU32: return fused_op<OpAddU32>(p, s);
    case OpCode::MaxI32: return fused_op<OpMaxI32>(p, s);
    case OpCode::MaxU32: return fused_op<OpMaxU32>(p, s);
    case OpCode::MaxF32: return fused_op<OpMaxF32>(p, s);
    case OpCode::AddF32: return fused_op<OpAddF32>(p, s);
    }
    return cudaErrorInvalidValue;
}

}  // namespace scanb200
