// Micro-benchmark: latency of a look-back style descriptor round trip on B200.
// 128 CTAs; each publishes (tag, value) into slot[cta] (stride S bytes), then one warp
// reads slots [0, cta) (4 per lane) until every tag is current.  Reports per-CTA
// %globaltimer durations of the first read round and of the whole wait.
// Modes: 0 = publish then read (concurrent writers); 1 = read slots already published by a
// previous launch (pure read latency); 2 = one single relaxed load of own slot; 4 = as 0
// after every CTA first loads a 32 KiB tile of a 4 MiB buffer (a register-tile scan CTA).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o desc_latency desc_latency.cu
#include <cstdio>
#include <cstdint>
#include <vector>
#include <algorithm>
#include <cuda_runtime.h>

__device__ __forceinline__ uint64_t gtime() { uint64_t g; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(g)); return g; }
__device__ __forceinline__ uint64_t ldr(const uint64_t* p) { uint64_t v; asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory"); return v; }
__device__ __forceinline__ void str(uint64_t* p, uint64_t v) { asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" :: "l"(p), "l"(v) : "memory"); }
__device__ __forceinline__ uint64_t ldv(const uint64_t* p) { uint64_t v; asm volatile("ld.volatile.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory"); return v; }

__global__ void k(uint64_t* slots, int stride_words, uint64_t tag, int mode, uint64_t* out, const uint4* data) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int b = blockIdx.x;
    __shared__ unsigned s_red;
    if (mode == 4) {
        // like a register-tile scan CTA: load a 32 KiB tile of a 4 MiB buffer first
        unsigned acc = 0;
        for (int i = threadIdx.x; i < 2048; i += blockDim.x) {
            uint4 v = data[(size_t)b * 2048 + i];
            acc += v.x + v.y + v.z + v.w;
        }
        if (threadIdx.x == 0) s_red = 0;
        __syncthreads();
        atomicAdd(&s_red, acc);
    }
    __syncthreads();
    if (warp != 0) return;
    uint64_t t0 = gtime();
    if ((mode == 0 || mode == 4) && lane == 0) str(slots + (size_t)b * stride_words, (tag << 32) | (uint64_t)(b + (mode == 4 ? s_red : 0u)));
    uint64_t t1 = gtime();
    int rounds = 0;
    uint64_t tfirst = 0;
    while (true) {
        bool ok = true;
        uint64_t acc = 0;
        #pragma unroll
        for (int m = 0; m < 4; ++m) {
            int pred = b - 1 - lane - 32 * m;
            if (pred >= 0) {
                uint64_t w = (mode == 3) ? ldv(slots + (size_t)pred * stride_words) : ldr(slots + (size_t)pred * stride_words);
                ok = ok && ((w >> 32) == tag || mode == 2 || mode == 1);
                acc += w;
            }
        }
        ++rounds;
        if (rounds == 1) tfirst = gtime();
        if (__all_sync(0xffffffffu, ok)) { if (acc == 12345) out[0] = 1; break; }
    }
    uint64_t t2 = gtime();
    if (lane == 0) { out[4 * b + 0] = t1 - t0; out[4 * b + 1] = tfirst - t1; out[4 * b + 2] = t2 - t1; out[4 * b + 3] = rounds; }
}

int main() {
    uint64_t *slots, *out;
    uint4* data;
    cudaMalloc(&data, 128 * 2048 * 16);
    cudaMemset(data, 1, 128 * 2048 * 16);
    cudaMalloc(&slots, 128 * 256 * 8);
    cudaMalloc(&out, 128 * 4 * 8);
    cudaMemset(slots, 0, 128 * 256 * 8);
    for (int stride : {1, 2, 8, 16, 32}) {
        for (int mode : {0, 1, 3, 4}) {
            for (int nthreads : {32, 512}) {
                std::vector<double> first, total, rnd;
                for (int rep = 0; rep < 20; ++rep) {
                    uint64_t tag = 1000 + rep + stride * 100 + mode * 10000 + nthreads;
                    if (mode != 0 && mode != 4) {
                        // pre-publish with this tag
                        std::vector<uint64_t> h(128 * stride, 0);
                        for (int i = 0; i < 128; ++i) h[(size_t)i * stride] = (tag << 32) | i;
                        cudaMemcpy(slots, h.data(), h.size() * 8, cudaMemcpyHostToDevice);
                    }
                    k<<<128, nthreads>>>(slots, stride, tag, mode, out, data);
                    std::vector<uint64_t> o(128 * 4);
                    cudaMemcpy(o.data(), out, o.size() * 8, cudaMemcpyDeviceToHost);
                    if (rep < 5) continue;
                    for (int b = 1; b < 128; ++b) { first.push_back(o[4 * b + 1]); total.push_back(o[4 * b + 2]); rnd.push_back(o[4 * b + 3]); }
                }
                auto med = [](std::vector<double> v) { std::sort(v.begin(), v.end()); return v[v.size() / 2]; };
                auto p90 = [](std::vector<double> v) { std::sort(v.begin(), v.end()); return v[v.size() * 9 / 10]; };
                printf("stride %3d B  mode %d  threads %4d : first round med %6.0f ns p90 %6.0f  total med %6.0f p90 %6.0f  rounds med %.0f\n",
                       stride * 8, mode, nthreads, med(first), p90(first), med(total), p90(total), med(rnd));
            }
        }
    }
    cudaError_t e = cudaDeviceSynchronize();
    printf("%s\n", cudaGetErrorString(e));
}
