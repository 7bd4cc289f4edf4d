// l2_size_probe.cu -- two questions about the mid-size (2^22..2^26 element) regime:
//  (1) what a plain 50/50 copy reaches AT THAT SIZE (same back-to-back timing as the scan
//      sweeps: a CUDA graph of R consecutive calls, per-call time = graph time / R), i.e.
//      the size-matched ceiling next to the big-copy denominator of MEASURED_PEAKS;
//  (2) whether an input read once with an L2 evict_last policy is still in L2 when it is
//      read again (a) by the next kernel, (b) by the next kernel while it also writes an
//      output of the same size with streaming stores -- the premise of any two-read form.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/micro/l2_size_probe tools/micro/l2_size_probe.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint64_t pol_last() {
    uint64_t p; asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p)); return p;
}
__device__ __forceinline__ uint64_t pol_first() {
    uint64_t p; asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p)); return p;
}

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

// read-only sweep (sum into one word per CTA so nothing is optimised away); mode 0 normal,
// 1 evict_last, 2 evict_first
template <int U>
__global__ void __launch_bounds__(256) read_only(const uint4* __restrict__ in, int64_t n, int mode, uint32_t* sink) {
    const uint64_t pl = pol_last(), pf = pol_first();
    const int64_t stride = (int64_t)gridDim.x * blockDim.x * U;
    uint32_t acc = 0;
    for (int64_t i = ((int64_t)blockIdx.x * blockDim.x) * U + threadIdx.x; i < n; i += stride) {
        uint4 v[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int64_t k = i + (int64_t)u * blockDim.x;
            v[u] = make_uint4(0, 0, 0, 0);
            if (k < n) {
                if (mode == 1)
                    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], %5;"
                                 : "=r"(v[u].x), "=r"(v[u].y), "=r"(v[u].z), "=r"(v[u].w) : "l"(in + k), "l"(pl));
                else if (mode == 2)
                    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], %5;"
                                 : "=r"(v[u].x), "=r"(v[u].y), "=r"(v[u].z), "=r"(v[u].w) : "l"(in + k), "l"(pf));
                else
                    asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                                 : "=r"(v[u].x), "=r"(v[u].y), "=r"(v[u].z), "=r"(v[u].w) : "l"(in + k));
            }
        }
#pragma unroll
        for (int u = 0; u < U; ++u) acc ^= v[u].x ^ v[u].y ^ v[u].z ^ v[u].w;
    }
    if (acc == 0x12345678u) sink[blockIdx.x] = acc;
}

// re-read with evict_first while writing another buffer (streaming stores)
template <int U>
__global__ void __launch_bounds__(256) reread_write(const uint4* __restrict__ in, uint4* __restrict__ out, int64_t n) {
    const uint64_t pf = pol_first();
    const int64_t stride = (int64_t)gridDim.x * blockDim.x * U;
    for (int64_t i = ((int64_t)blockIdx.x * blockDim.x) * U + threadIdx.x; i < n; i += stride) {
        uint4 v[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int64_t k = i + (int64_t)u * blockDim.x;
            if (k < n) asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], %5;"
                                    : "=r"(v[u].x), "=r"(v[u].y), "=r"(v[u].z), "=r"(v[u].w) : "l"(in + k), "l"(pf));
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int64_t k = i + (int64_t)u * blockDim.x;
            if (k < n) asm volatile("st.global.cs.v4.u32 [%0], {%1,%2,%3,%4};"
                                    :: "l"(out + k), "r"(v[u].x), "r"(v[u].y), "r"(v[u].z), "r"(v[u].w) : "memory");
        }
    }
}

__global__ void flush_kernel(uint4* buf, int64_t n, uint32_t v) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        buf[i] = make_uint4(v, v, v, v);
}

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e_)); return 1; } } while (0)

int main() {
    int sms = 0; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const int64_t maxe = (int64_t)1 << 27;                  // elements (4 B)
    uint4 *a, *b, *fl; uint32_t* sink;
    CK(cudaMalloc(&a, maxe * 4)); CK(cudaMalloc(&b, maxe * 4));
    const int64_t fln = (int64_t)512 << 20;                 // 512 MiB flush buffer
    CK(cudaMalloc(&fl, fln)); CK(cudaMalloc(&sink, 4096 * 4));
    CK(cudaMemset(a, 1, maxe * 4)); CK(cudaMemset(b, 0, maxe * 4));
    cudaStream_t s; CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);

    printf("(1) size-matched copy, back-to-back calls in one CUDA graph (R calls), per-call us\n");
    printf("%4s %10s %10s %10s %10s %10s\n", "n", "MiB_in", "ldst_us", "ldst_GBs", "d2d_us", "d2d_GBs");
    for (int n = 20; n <= 27; ++n) {
        const int64_t ne = (int64_t)1 << n, n4 = ne / 4;
        const int R = n <= 24 ? 50 : 10;
        float best[2] = {1e30f, 1e30f};
        for (int form = 0; form < 2; ++form) {
            cudaGraph_t g; cudaGraphExec_t ge;
            CK(cudaStreamBeginCapture(s, cudaStreamCaptureModeGlobal));
            for (int r = 0; r < R; ++r) {
                if (form == 0) copy_ldst<4><<<sms * 4, 256, 0, s>>>(a, b, n4);
                else cudaMemcpyAsync(b, a, ne * 4, cudaMemcpyDeviceToDevice, s);
            }
            CK(cudaStreamEndCapture(s, &g));
            CK(cudaGraphInstantiate(&ge, g, 0));
            for (int w = 0; w < 3; ++w) CK(cudaGraphLaunch(ge, s));
            for (int rep = 0; rep < 10; ++rep) {
                cudaEventRecord(e0, s); cudaGraphLaunch(ge, s); cudaEventRecord(e1, s);
                cudaEventSynchronize(e1);
                float ms; cudaEventElapsedTime(&ms, e0, e1);
                if (ms / R < best[form]) best[form] = ms / R;
            }
            cudaGraphExecDestroy(ge); cudaGraphDestroy(g);
        }
        const double bytes = 8.0 * ne;
        printf("%4d %10.1f %10.2f %10.1f %10.2f %10.1f\n", n, ne * 4.0 / (1 << 20), best[0] * 1e3,
               bytes / (best[0] * 1e-3) / 1e9, best[1] * 1e3, bytes / (best[1] * 1e-3) / 1e9);
    }

    printf("\n(2) L2 retention: flush, kernel A reads X (mode), kernel B re-reads X; us of B\n");
    printf("    cold = B after a flush; B_ro = read-only re-read; B_rw = re-read (evict_first) + write X\n");
    printf("%8s %6s %9s %9s %9s %9s %9s\n", "MiB", "modeA", "A_us", "cold_ro", "B_ro", "cold_rw", "B_rw");
    const char* mname[3] = {"normal", "last", "first"};
    for (int mib : {16, 24, 32, 48, 64, 80, 96}) {
        const int64_t n4 = ((int64_t)mib << 20) / 16;
        for (int mode = 0; mode < 3; ++mode) {
            float tA = 1e30f, tcro = 1e30f, tbro = 1e30f, tcrw = 1e30f, tbrw = 1e30f;
            for (int rep = 0; rep < 5; ++rep) {
                float ms;
                // cold read-only
                flush_kernel<<<sms * 8, 256, 0, s>>>(fl, fln / 16, rep);
                cudaEventRecord(e0, s); read_only<4><<<sms * 4, 256, 0, s>>>(a, n4, 0, sink); cudaEventRecord(e1, s);
                cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1); if (ms < tcro) tcro = ms;
                // A then B read-only
                flush_kernel<<<sms * 8, 256, 0, s>>>(fl, fln / 16, rep);
                cudaEventRecord(e0, s); read_only<4><<<sms * 4, 256, 0, s>>>(a, n4, mode, sink); cudaEventRecord(e1, s);
                cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1); if (ms < tA) tA = ms;
                cudaEventRecord(e0, s); read_only<4><<<sms * 4, 256, 0, s>>>(a, n4, 0, sink); cudaEventRecord(e1, s);
                cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1); if (ms < tbro) tbro = ms;
                // cold re-read + write
                flush_kernel<<<sms * 8, 256, 0, s>>>(fl, fln / 16, rep);
                cudaEventRecord(e0, s); reread_write<4><<<sms * 4, 256, 0, s>>>(a, b, n4); cudaEventRecord(e1, s);
                cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1); if (ms < tcrw) tcrw = ms;
                // A then B re-read + write
                flush_kernel<<<sms * 8, 256, 0, s>>>(fl, fln / 16, rep);
                read_only<4><<<sms * 4, 256, 0, s>>>(a, n4, mode, sink);
                cudaEventRecord(e0, s); reread_write<4><<<sms * 4, 256, 0, s>>>(a, b, n4); cudaEventRecord(e1, s);
                cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1); if (ms < tbrw) tbrw = ms;
            }
            printf("%8d %6s %9.2f %9.2f %9.2f %9.2f %9.2f\n", mib, mname[mode], tA * 1e3, tcro * 1e3, tbro * 1e3,
                   tcrw * 1e3, tbrw * 1e3);
        }
    }
    printf("\n(3) two-phase emulation, back-to-back in one CUDA graph: per call = A (read X, evict_last)\n"
           "    then B (re-read X evict_first + write X); 'rot' cycles over 4 buffer pairs (cold), 'same' reuses one\n");
    printf("%4s %10s %10s %10s %10s\n", "n", "2ph_same", "copy_same", "2ph_rot", "copy_rot");
    {
        const int64_t maxr = (int64_t)1 << 25;
        uint4 *ra[4], *rb[4];
        for (int k = 0; k < 4; ++k) { CK(cudaMalloc(&ra[k], maxr * 4)); CK(cudaMalloc(&rb[k], maxr * 4));
                                      CK(cudaMemset(ra[k], 1, maxr * 4)); }
        for (int n = 22; n <= 25; ++n) {
            const int64_t ne = (int64_t)1 << n, n4 = ne / 4;
            float res[4];
            for (int form = 0; form < 4; ++form) {
                const bool rot = form >= 2, two = (form % 2) == 0;
                const int R = 32;
                cudaGraph_t g; cudaGraphExec_t ge;
                CK(cudaStreamBeginCapture(s, cudaStreamCaptureModeGlobal));
                for (int r = 0; r < R; ++r) {
                    const int k = rot ? r % 4 : 0;
                    if (two) {
                        read_only<4><<<sms * 4, 256, 0, s>>>(ra[k], n4, 1, sink);
                        reread_write<4><<<sms * 4, 256, 0, s>>>(ra[k], rb[k], n4);
                    } else {
                        copy_ldst<4><<<sms * 4, 256, 0, s>>>(ra[k], rb[k], n4);
                    }
                }
                CK(cudaStreamEndCapture(s, &g));
                CK(cudaGraphInstantiate(&ge, g, 0));
                CK(cudaGraphLaunch(ge, s));
                float best = 1e30f;
                for (int rep = 0; rep < 10; ++rep) {
                    cudaEventRecord(e0, s); cudaGraphLaunch(ge, s); cudaEventRecord(e1, s);
                    cudaEventSynchronize(e1);
                    float ms; cudaEventElapsedTime(&ms, e0, e1);
                    if (ms / R < best) best = ms / R;
                }
                res[form] = best * 1e3f;
                cudaGraphExecDestroy(ge); cudaGraphDestroy(g);
            }
            printf("%4d %10.2f %10.2f %10.2f %10.2f\n", n, res[0], res[1], res[2], res[3]);
        }
    }
    CK(cudaGetLastError());
    CK(cudaDeviceSynchronize());
    return 0;
}
