/* abi_demo.c -- the C-ABI used from plain C (no Python, no torch): allocate with the CUDA
 * runtime, fill a batch, call scan_batch / scan_batch_ex (every kernel family) /
 * scan_plan_ex / scan_batch_host /
 * scan_shard_totals + scan_shard_scan, and check the results against a sequential loop
 * written here (integer add: exact).  Built and run by tests/test_gpu_c_abi.py. */
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <cuda_runtime.h>
#include "scan_b200.h"

#define CHECK(x) do { scan_status s_ = (x); if (s_ != SCAN_OK) { \
    fprintf(stderr, "%s -> %s\n", #x, scan_status_string(s_)); return 1; } } while (0)

static int verify(const int32_t* x, const int32_t* y, int64_t N, int64_t G, int excl, const char* what) {
    for (int64_t g = 0; g < G; ++g) {
        uint32_t acc = 0;
        for (int64_t i = 0; i < N; ++i) {
            uint32_t want;
            if (excl) { want = acc; acc += (uint32_t)x[g * N + i]; }
            else      { acc += (uint32_t)x[g * N + i]; want = acc; }
            if ((uint32_t)y[g * N + i] != want) {
                fprintf(stderr, "%s mismatch at g=%lld i=%lld\n", what, (long long)g, (long long)i);
                return 1;
            }
        }
    }
    return 0;
}

int main(void) {
    const int64_t N = 100003, G = 5, n = N * G;
    int32_t* hx = (int32_t*)malloc(n * 4);
    int32_t* hy = (int32_t*)malloc(n * 4);
    uint64_t s = 88172645463325252ull;
    for (int64_t i = 0; i < n; ++i) { s ^= s << 13; s ^= s >> 7; s ^= s << 17; hx[i] = (int32_t)s; }
    void *dx, *dy, *dt, *dall;
    if (cudaMalloc(&dx, n * 4) || cudaMalloc(&dy, n * 4) || cudaMalloc(&dt, G * 8) || cudaMalloc(&dall, 2 * G * 8))
        return 2;
    cudaMemcpy(dx, hx, n * 4, cudaMemcpyHostToDevice);

    CHECK(scan_batch(dx, dy, N, G, SCAN_OP_ADD, SCAN_I32, SCAN_INCLUSIVE, NULL));
    cudaMemcpy(hy, dy, n * 4, cudaMemcpyDeviceToHost);
    if (verify(hx, hy, N, G, 0, "scan_batch")) return 1;

    for (int algo = SCAN_ALGO_LOOKBACK; algo <= SCAN_ALGO_THREE_STAGE; ++algo) {
        CHECK(scan_batch_ex(dx, dy, N, G, SCAN_OP_ADD, SCAN_I32, SCAN_EXCLUSIVE, (scan_algo)algo, -1, NULL, 0, NULL));
        cudaMemcpy(hy, dy, n * 4, cudaMemcpyDeviceToHost);
        if (verify(hx, hy, N, G, 1, "scan_batch_ex")) return 1;
    }

    /* the remaining families through scan_batch_ex, and what scan_plan_ex reports for AUTO */
    for (int algo = SCAN_ALGO_PACKED_WARP; algo <= SCAN_ALGO_CLUSTER; ++algo) {
        CHECK(scan_batch_ex(dx, dy, N, G, SCAN_OP_ADD, SCAN_I32, SCAN_INCLUSIVE, (scan_algo)algo, -1, NULL, 0, NULL));
        cudaMemcpy(hy, dy, n * 4, cudaMemcpyDeviceToHost);
        if (verify(hx, hy, N, G, 0, "scan_batch_ex")) return 1;
    }
    CHECK(scan_batch_ex(dx, dy, N, 1, SCAN_OP_ADD, SCAN_I32, SCAN_EXCLUSIVE, SCAN_ALGO_FUSED, -1, NULL, 0, NULL));
    cudaMemcpy(hy, dy, N * 4, cudaMemcpyDeviceToHost);
    if (verify(hx, hy, N, 1, 1, "fused")) return 1;
    if (scan_batch_ex(dx, dy, N, G, SCAN_OP_ADD, SCAN_I32, SCAN_INCLUSIVE, SCAN_ALGO_FUSED, -1, NULL, 0, NULL)
        != SCAN_ERR_UNSUPPORTED) return 3;                  /* ragged N with G > 1 */
    int algo_auto = -1;
    int64_t param_auto = 0;
    CHECK(scan_plan_ex(N, G, SCAN_OP_ADD, SCAN_I32, SCAN_INCLUSIVE, dx, dy, &algo_auto, &param_auto));
    if (algo_auto <= SCAN_ALGO_AUTO || algo_auto > SCAN_ALGO_FUSED) return 3;

    CHECK(scan_batch_host(hx, hy, N, G, SCAN_OP_ADD, SCAN_I32, SCAN_INCLUSIVE));
    if (verify(hx, hy, N, G, 0, "scan_batch_host")) return 1;

    /* elements mode with two virtual ranks on one GPU: portions [0, h) and [h, N) of each
       problem need their own workspaces between the two steps */
    const int64_t h = 40000;
    int32_t* hx0 = (int32_t*)malloc(h * G * 4);
    int32_t* hx1 = (int32_t*)malloc((N - h) * G * 4);
    for (int64_t g = 0; g < G; ++g) {
        for (int64_t i = 0; i < h; ++i) hx0[g * h + i] = hx[g * N + i];
        for (int64_t i = h; i < N; ++i) hx1[g * (N - h) + i - h] = hx[g * N + i];
    }
    void *d0, *d1, *o0, *o1, *w0, *w1;
    size_t b0 = scan_shard_workspace_bytes(h, G), b1 = scan_shard_workspace_bytes(N - h, G);
    if (cudaMalloc(&d0, h * G * 4) || cudaMalloc(&d1, (N - h) * G * 4) || cudaMalloc(&o0, h * G * 4) ||
        cudaMalloc(&o1, (N - h) * G * 4) || cudaMalloc(&w0, b0) || cudaMalloc(&w1, b1))
        return 2;
    cudaMemset(w0, 0, b0);
    cudaMemset(w1, 0, b1);
    cudaMemcpy(d0, hx0, h * G * 4, cudaMemcpyHostToDevice);
    cudaMemcpy(d1, hx1, (N - h) * G * 4, cudaMemcpyHostToDevice);
    CHECK(scan_shard_totals(d0, h, G, SCAN_OP_ADD, SCAN_I32, (char*)dall, w0, b0, NULL));
    CHECK(scan_shard_totals(d1, N - h, G, SCAN_OP_ADD, SCAN_I32, (char*)dall + G * 8, w1, b1, NULL));
    CHECK(scan_shard_scan(d0, o0, h, G, SCAN_OP_ADD, SCAN_I32, SCAN_INCLUSIVE, dall, 0, 2, w0, b0, NULL));
    CHECK(scan_shard_scan(d1, o1, N - h, G, SCAN_OP_ADD, SCAN_I32, SCAN_INCLUSIVE, dall, 1, 2, w1, b1, NULL));
    cudaMemcpy(hx0, o0, h * G * 4, cudaMemcpyDeviceToHost);
    cudaMemcpy(hx1, o1, (N - h) * G * 4, cudaMemcpyDeviceToHost);
    for (int64_t g = 0; g < G; ++g) {
        for (int64_t i = 0; i < h; ++i) hy[g * N + i] = hx0[g * h + i];
        for (int64_t i = h; i < N; ++i) hy[g * N + i] = hx1[g * (N - h) + i - h];
    }
    if (verify(hx, hy, N, G, 0, "sharded")) return 1;

    /* error paths */
    if (scan_batch(dx, (char*)dx + 4, N, G, SCAN_OP_ADD, SCAN_I32, SCAN_INCLUSIVE, NULL) != SCAN_ERR_INVALID_ARG) return 3;
    if (scan_batch(hx, hy, N, G, SCAN_OP_ADD, SCAN_I32, SCAN_INCLUSIVE, NULL) != SCAN_ERR_INVALID_ARG) return 3;
    if (cudaDeviceSynchronize() != cudaSuccess) return 4;
    printf("abi_demo ok\n");
    return 0;
}
