// scan_cluster.cu -- cluster-per-problem scan for few medium problems (G small, N up to
// ~2^17), sm_100a thread-block clusters + distributed shared memory.
//
// The paper's answer to "one problem, more than one block" is the three-stage chain with
// its aux array in global memory (PAPER.md:110-118 [§3.1, Fig. 3]); for a single problem
// of 2^13..2^17 elements that costs three launches (or one look-back launch with
// descriptor round trips through L2), ~5 us of latency for < 1 MiB of data.  On sm_100a
// the C CTAs of one problem can instead form ONE thread-block cluster (C <= 16) and trade
// their aggregates through distributed shared memory: a round of the kernel is
//
//   every CTA: load its TILE of the round (registers, 128-bit rows), scan it (thread ->
//              warp shuffle -> block combine), put the CTA aggregate in
//              its own shared memory
//   barrier.cluster (release / acquire)
//   every warp: read the C aggregates of the round over DSMEM (lane q reads CTA q), fold
//              those of CTAs < rank into the carry, store the tile with it
//
// so the "aux array" of the paper lives in the cluster's shared memory and Stage 2 is a
// warp reduction.  Problems longer than one round (C * TILE elements) loop over rounds
// with the running carry in registers (the cascade).  Aggregate slots are
// double-buffered by round parity, so one cluster barrier per round suffices: CTA c
// rewrites slot k&1 in round k+2 only after barrier k+1, which every CTA reaches after
// its reads of round k.  f32 add carries are fp64 (reading R3).
#include <cooperative_groups.h>

#include "scan_common.cuh"
#include "scan_internal.h"

namespace cg = cooperative_groups;

namespace scanb200 {

namespace {

template <class Op, int WARPS, int V>
__global__ void __launch_bounds__(WARPS * 32) cluster_scan_kernel(ChunkParams p) {
    using T = typename Op::T;
    using C = typename Op::Carry;
    constexpr int TILE = WARPS * 32 * V * 4, WCH = V * 128;
    __shared__ __align__(16) T s_wval[(WARPS + 3) & ~3];   // 16-byte aligned and padded: vectorised slot reads never cover a neighbour
    __shared__ C s_agg[2];
    cg::cluster_group cl = cg::this_cluster();
    const unsigned csize = cl.num_blocks(), crank = cl.block_rank();
    const int warp = threadIdx.x >> 5, lane = lane_id();
    const int64_t g = (int64_t)blockIdx.x / csize;
    const T* in = (const T*)p.in + g * p.N;
    T* out = (T*)p.out + g * p.N;
    const int64_t R = (int64_t)csize * TILE;
    grid_dep_launch();                     // cross-call programmatic launch (ChunkParams)
    // a small grid is one wave: every CTA L2-prefetches its first tile while it waits
    // (scan_common.cuh: prefetch_l2_span)
    if (p.pdl_first && threadIdx.x == 0 && (int64_t)gridDim.x <= p.pf_ctas)
        prefetch_l2_span(in + (int64_t)crank * TILE, min(p.N - (int64_t)crank * TILE, (int64_t)TILE));
    if (p.pdl_first) grid_dep_wait();

    C run = Op::cidentity();
    int k = 0;
    for (int64_t base = 0; base < p.N; base += R, ++k) {
        const int64_t wb = base + (int64_t)crank * TILE + warp * WCH;
        WarpTile<Op, false, V> wt;
        wt.load(in, wb, p.N, p.vec);
        wt.scan();
        if (lane == 0) s_wval[warp] = wt.wtot;
        __syncthreads();
        T wp = Op::identity();
#pragma unroll
        for (int w = 0; w < WARPS; ++w)
            if (w < warp) wp = Op::apply(wp, s_wval[w]);
        if (warp == WARPS - 1 && lane == 0) s_agg[k & 1] = Op::to_carry(Op::apply(wp, wt.wtot));
        cl.sync();
        C a = Op::cidentity();
        if ((unsigned)lane < csize) a = *cl.map_shared_rank(&s_agg[k & 1], (unsigned)lane);
        const C pre = warp_reduce_carry<Op>((unsigned)lane < crank ? a : Op::cidentity());
        const C tot = warp_reduce_carry<Op>(a);
        wt.store(out, wb, p.N, p.vec, wp, false, Op::from_carry(Op::capply(run, pre)), p.exclusive);
        run = Op::capply(run, tot);
    }
    // no CTA may leave while a peer can still read its aggregate slots
    cl.sync();
}

template <class Op, int WARPS, int V>
cudaError_t launch_t(const ChunkParams& p, int csize, cudaStream_t s) {
    auto kern = cluster_scan_kernel<Op, WARPS, V>;
    // non-portable cluster sizes (16 CTAs) opted in once per device (scan_launch.cu)
    cudaError_t e = kernel_prepare((const void*)kern, WARPS * 32, 0, true, nullptr);
    if (e != cudaSuccess) return e;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)(p.G * csize), 1, 1);
    cfg.blockDim = dim3(WARPS * 32, 1, 1);
    cfg.dynamicSmemBytes = 0;
    cfg.stream = s;
    cudaLaunchAttribute attr[2];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = (unsigned)csize;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[1].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = p.pdl_first ? 2 : 1;
    return cudaLaunchKernelEx(&cfg, kern, p);
}

template <class Op>
cudaError_t launch_op(const ChunkParams& p, int variant, int csize, cudaStream_t s) {
    switch (variant) {
    case 1: return launch_t<Op, 16, 2>(p, csize, s);     // 4096-element tiles, 512 threads
    case 2: return launch_t<Op, 32, 4>(p, csize, s);     // 16384-element tiles, 1024 threads
    default: return launch_t<Op, 32, 2>(p, csize, s);    // 8192-element tiles, 1024 threads
    }
}

}  // namespace

int64_t cluster_tile_elems(int variant) { return variant == 1 ? 4096 : variant == 2 ? 16384 : 8192; }

cudaError_t launch_cluster_scan(OpCode op, const ChunkParams& p, int variant, int csize, cudaStream_t s) {
    if (csize < 1 || csize > kMaxClusterCtas || (csize & (csize - 1))) return cudaErrorInvalidValue;
    if (p.G * csize > 0x7FFFFFFFll) return cudaErrorInvalidConfiguration;
    switch (op) {
    case OpCode::AddU32: return launch_op<OpAddU32>(p, variant, csize, s);
    case OpCode::MaxI32: return launch_op<OpMaxI32>(p, variant, csize, s);
    case OpCode::MaxU32: return launch_op<OpMaxU32>(p, variant, csize, s);
    case OpCode::MaxF32: return launch_op<OpMaxF32>(p, variant, csize, s);
    case OpCode::AddF32: return launch_op<OpAddF32>(p, variant, csize, s);
    }
    return cudaErrorInvalidValue;
}

}  // namespace scanb200
