// spin.cu -- TEST helper (tests/test_gpu_safety.py), not part of the product library.
// A kernel that occupies `ctas` SMs (one CTA per SM through its dynamic shared memory) and
// spins until the host writes a nonzero value into `flag` (pinned, device-visible host
// memory), or a time limit passes.  Used to take SMs away from the library's persistent
// cooperative look-back grid while it is launched on another stream.
#include <cuda_runtime.h>
#include <cstdint>

__global__ void spin_kernel(const volatile int* flag, unsigned long long limit_ns) {
    extern __shared__ unsigned char pad[];
    if (threadIdx.x == 0) {
        unsigned long long t0, t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
        while (*flag == 0) {
            __nanosleep(2000);
            asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
            if (t - t0 > limit_ns) break;
        }
        pad[0] = 1;
    }
    __syncthreads();
}

extern "C" int spin_launch(const int* flag, int ctas, int smem_bytes, unsigned long long limit_ns, void* stream) {
    cudaError_t e = cudaFuncSetAttribute(spin_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem_bytes);
    if (e != cudaSuccess) return (int)e;
    spin_kernel<<<ctas, 128, smem_bytes, (cudaStream_t)stream>>>((const volatile int*)flag, limit_ns);
    return (int)cudaGetLastError();
}
