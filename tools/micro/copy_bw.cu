// copy_bw.cu -- what a pure streaming copy (read 1 GiB, write 1 GiB) reaches on this B200,
// i.e. the practical roofline of the scan kernels (8 B/element moved, half read, half write).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/micro/copy_bw tools/micro/copy_bw.cu
// Kernels: (a) 128-bit register copy, U loads in flight per thread, grid-stride, several
// CTAs per SM; (b) TMA bulk copy: persistent CTA per SM, S-slot smem ring, one thread loads
// (cp.async.bulk global->shared, mbarrier) and stores (cp.async.bulk shared->global,
// bulk_group).  Prints GB/s (read + write bytes / time), best of 20.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

template <int U>
__global__ void __launch_bounds__(256) copy_ldst(const uint4* __restrict__ in, uint4* __restrict__ out, int64_t n) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x * U;
    for (int64_t i = ((int64_t)blockIdx.x * blockDim.x) * U + threadIdx.x; i < n; i += stride) {
        uint4 v[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int64_t k = i + (int64_t)u * blockDim.x;
            if (k < n) asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                                    : "=r"(v[u].x), "=r"(v[u].y), "=r"(v[u].z), "=r"(v[u].w) : "l"(in + k));
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int64_t k = i + (int64_t)u * blockDim.x;
            if (k < n) asm volatile("st.global.cs.v4.u32 [%0], {%1,%2,%3,%4};"
                                    :: "l"(out + k), "r"(v[u].x), "r"(v[u].y), "r"(v[u].z), "r"(v[u].w) : "memory");
        }
    }
}

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <int S, int CHUNK>
__global__ void __launch_bounds__(32) copy_tma(const char* in, char* out, int64_t bytes) {
    extern __shared__ __align__(128) unsigned char buf[];
    __shared__ __align__(8) uint64_t bar[S];
    if (threadIdx.x != 0) return;
    for (int s = 0; s < S; ++s)
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(smem_u32(&bar[s])));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    const int64_t nchunks = bytes / CHUNK;
    int64_t mine = 0;
    for (int64_t c = blockIdx.x; c < nchunks; c += gridDim.x) ++mine;
    // prologue: fill the ring
    auto issue = [&](int64_t j) {
        const int s = (int)(j % S);
        const int64_t c = blockIdx.x + j * (int64_t)gridDim.x;
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(smem_u32(&bar[s])), "r"(CHUNK) : "memory");
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                     :: "r"(smem_u32(buf + (size_t)s * CHUNK)), "l"(in + c * CHUNK), "r"(CHUNK), "r"(smem_u32(&bar[s])) : "memory");
    };
    for (int64_t j = 0; j < S && j < mine; ++j) issue(j);
    for (int64_t j = 0; j < mine; ++j) {
        const int s = (int)(j % S);
        const uint32_t ph = (uint32_t)((j / S) & 1);
        asm volatile("{ .reg .pred p; W: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1; @!p bra W; }"
                     :: "r"(smem_u32(&bar[s])), "r"(ph) : "memory");
        const int64_t c = blockIdx.x + j * (int64_t)gridDim.x;
        asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;"
                     :: "l"(out + c * CHUNK), "r"(smem_u32(buf + (size_t)s * CHUNK)), "r"(CHUNK) : "memory");
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
        if (j + S < mine) {
            // the slot may be reloaded once its store has READ it
            asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
            issue(j + S);
        }
    }
    asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

template <class F>
float best_ms(F f) {
    cudaEvent_t a, b;
    cudaEventCreate(&a); cudaEventCreate(&b);
    for (int i = 0; i < 3; ++i) f();
    float best = 1e30f;
    for (int r = 0; r < 20; ++r) {
        cudaEventRecord(a); f(); cudaEventRecord(b); cudaEventSynchronize(b);
        float ms; cudaEventElapsedTime(&ms, a, b);
        if (ms < best) best = ms;
    }
    return best;
}

int main() {
    const int64_t bytes = int64_t(1) << 30;
    char *in, *out;
    cudaMalloc(&in, bytes); cudaMalloc(&out, bytes);
    cudaMemset(in, 1, bytes); cudaMemset(out, 0, bytes);
    int sms = 0; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const int64_t n16 = bytes / 16;
    auto rep = [&](const char* name, float ms) { printf("%-34s %8.3f ms  %7.1f GB/s\n", name, ms, 2.0 * bytes / (ms * 1e-3) / 1e9); };
    rep("cudaMemcpyDeviceToDevice", best_ms([&] { cudaMemcpyAsync(out, in, bytes, cudaMemcpyDeviceToDevice); }));
    for (int bps : {2, 4, 8}) {
        char nm[64];
        snprintf(nm, 64, "ldst U=4 %d CTA/SM", bps);
        rep(nm, best_ms([&] { copy_ldst<4><<<sms * bps, 256>>>((const uint4*)in, (uint4*)out, n16); }));
        snprintf(nm, 64, "ldst U=8 %d CTA/SM", bps);
        rep(nm, best_ms([&] { copy_ldst<8><<<sms * bps, 256>>>((const uint4*)in, (uint4*)out, n16); }));
    }
    {
        auto k = copy_tma<6, 32768>;
        cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 6 * 32768);
        rep("tma 6 x 32 KiB, 1 CTA/SM", best_ms([&] { k<<<sms, 32, 6 * 32768>>>(in, out, bytes); }));
        auto k2 = copy_tma<3, 32768>;
        cudaFuncSetAttribute(k2, cudaFuncAttributeMaxDynamicSharedMemorySize, 3 * 32768);
        rep("tma 3 x 32 KiB, 2 CTA/SM", best_ms([&] { k2<<<sms * 2, 32, 3 * 32768>>>(in, out, bytes); }));
        auto k3 = copy_tma<12, 16384>;
        cudaFuncSetAttribute(k3, cudaFuncAttributeMaxDynamicSharedMemorySize, 12 * 16384);
        rep("tma 12 x 16 KiB, 1 CTA/SM", best_ms([&] { k3<<<sms, 32, 12 * 16384>>>(in, out, bytes); }));
    }
    cudaError_t e = cudaDeviceSynchronize();
    printf("status %s\n", cudaGetErrorString(e));
    return 0;
}
