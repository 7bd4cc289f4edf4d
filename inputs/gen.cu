// Device twin of inputs/__init__.py: counter-based splitmix64 input generator.
// Holds no scan arithmetic; shared by the oracle-side tests and the benchmarks only so
// that both sides see bit-identical inputs.  See inputs/__init__.py for the formulas.
#include <cstdint>
#include <cuda_runtime.h>

namespace {

__device__ __forceinline__ uint64_t mix(uint64_t seed, uint64_t idx)
{
    uint64_t z = seed + (idx + 1ull) * 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

__device__ __forceinline__ uint32_t element(int dist, uint64_t seed, uint64_t idx, int64_t row_len)
{
    if (dist == 5 || dist == 6) {
        uint64_t v = idx % (uint64_t)row_len + 1ull;
        if (dist == 5) return (uint32_t)(int32_t)(int64_t)v;
        return __float_as_uint((float)(int64_t)v);       // exact while v <= 2^24
    }
    uint64_t h = mix(seed, idx);
    switch (dist) {
    case 0: case 1: return (uint32_t)h;
    case 2: return __float_as_uint(__uint2float_rn((uint32_t)(h >> 40)) * 0x1p-24f);
    case 3: return __float_as_uint((float)((int64_t)(h >> 39) - (1ll << 24)) * 0x1p-24f);
    default: return (uint32_t)((int32_t)(h % 2001ull) - 1000);
    }
}

__global__ void fill_kernel(uint32_t* out, int64_t count, uint64_t seed, int64_t offset,
                            int dist, int64_t row_len)
{
    int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < count; i += stride)
        out[i] = element(dist, seed, (uint64_t)(offset + i), row_len);
}

}  // namespace

extern "C" int inputs_fill(void* out, int64_t count, uint64_t seed, int64_t offset, int dist,
                           int64_t row_len, void* stream)
{
    if (count <= 0) return 0;
    if ((dist == 5 || dist == 6) && row_len <= 0) return (int)cudaErrorInvalidValue;
    int64_t blocks = (count + 255) / 256;
    if (blocks > 148 * 64) blocks = 148 * 64;
    fill_kernel<<<(unsigned)blocks, 256, 0, (cudaStream_t)stream>>>((uint32_t*)out, count, seed, offset,
                                                                  dist, row_len);
    return (int)cudaGetLastError();
}
