// racecheck probe: the double-buffered warp-slot pattern of chunk_scan_kernel (one
// __syncthreads per tile, slots[it & 1]) in isolation.  Race-free by construction: the
// write of tile it+2 follows the barrier of tile it+1, which every warp reaches only after
// its reads of tile it.  `compute-sanitizer --tool racecheck ./race_dbuf` tells whether the
// checker flags the idiom itself on sm_100a.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -lineinfo -O3 -o race_dbuf race_dbuf.cu
#include <cstdio>
#include <cuda_runtime.h>

__global__ void dbuf(unsigned* out, int tiles) {
    __shared__ unsigned s[2][8];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    unsigned acc = 0;
    for (int it = 0; it < tiles; ++it) {
        if (lane == 0) s[it & 1][warp] = it * 8 + warp;
        __syncthreads();
        for (int w = 0; w < 8; ++w) acc += s[it & 1][w];
    }
    out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}

int main() {
    unsigned* d;
    cudaMalloc(&d, 256 * 4 * 4);
    dbuf<<<4, 256>>>(d, 18);
    unsigned h[4];
    cudaMemcpy(h, d, 16, cudaMemcpyDeviceToHost);
    // sum over it of sum_w (8 it + w) = 64 * sum(it) + 18 * 28
    printf("acc %u expected %u\n", h[0], 64u * (17u * 18u / 2u) + 18u * 28u);
    cudaFree(d);
    return 0;
}
