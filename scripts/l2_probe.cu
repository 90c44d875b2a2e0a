// L2 gather-bandwidth probe: the ceiling of a kernel
// whose gathered rows are L2-resident.  Every warp gathers random rows of a
// table that fits in L2 (half-warp 256 B segments, like the PAIR panel path, or
// full-warp 512 B rows), LDG.128, U rows in flight, and sums them; the grid is
// persistent (SMs x blocks).  Prints bytes/time for several table sizes.
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/l2_probe scripts/l2_probe.cu
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <cuda_runtime.h>

template <int ROWB, int U>
__global__ void __launch_bounds__(256) gather(const float4 *__restrict__ tab, int64_t nrows,
                                              int64_t iters, uint32_t seed, float *out) {
    constexpr int LPR = ROWB / 16;          // lanes per row
    constexpr int RPW = 32 / LPR;           // rows per warp instruction
    const int lane = threadIdx.x & 31;
    const int sub = lane / LPR, col = lane % LPR;
    uint32_t x = seed ^ (blockIdx.x * 7919u + threadIdx.x / 32 * 104729u + sub * 31u);
    float4 acc = make_float4(0, 0, 0, 0);
    for (int64_t it = 0; it < iters; ++it) {
        float4 v[U];
#pragma unroll
        for (int k = 0; k < U; ++k) {
            x ^= x << 13; x ^= x >> 17; x ^= x << 5;
            const int64_t r = x % (uint32_t)nrows;
            v[k] = __ldg(tab + r * (ROWB / 16) + col);
        }
#pragma unroll
        for (int k = 0; k < U; ++k) { acc.x += v[k].x; acc.y += v[k].y; acc.z += v[k].z; acc.w += v[k].w; }
    }
    (void)RPW;
    if (acc.x == 12345.f) out[0] = acc.y + acc.z + acc.w;
}

template <int ROWB, int U>
static void run(const float4 *tab, int64_t table_bytes, int sms, float *out) {
    const int64_t nrows = table_bytes / ROWB;
    const int blocks = sms * 4;  // 32 warps/SM
    const int64_t iters = 4000;
    cudaEvent_t a, b;
    cudaEventCreate(&a); cudaEventCreate(&b);
    gather<ROWB, U><<<blocks, 256>>>(tab, nrows, 50, 1, out);
    cudaEventRecord(a);
    gather<ROWB, U><<<blocks, 256>>>(tab, nrows, iters, 7, out);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms = 0; cudaEventElapsedTime(&ms, a, b);
    const double bytes = (double)blocks * 256 * 16 * U * iters;  // every lane moves 16 B per row
    printf("{\"row_bytes\": %d, \"U\": %d, \"table_MB\": %.1f, \"ms\": %.3f, \"GBs\": %.1f}\n", ROWB, U,
           table_bytes / 1e6, ms, bytes / ms / 1e6);
}

int main() {
    int sms = 0; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const int64_t maxb = int64_t(1) << 31;
    float4 *tab; float *out;
    cudaMalloc(&tab, maxb); cudaMalloc(&out, 64);
    cudaMemset(tab, 0, maxb);
    for (int64_t tb : {int64_t(16) << 20, int64_t(60) << 20, int64_t(100) << 20, int64_t(2) << 30}) {
        run<256, 4>(tab, tb, sms, out);
        run<256, 8>(tab, tb, sms, out);
        run<512, 4>(tab, tb, sms, out);
    }
    // large tables (HBM random-row gathers vs table size: address-translation
    // reach; R-MAT-24's X is 8.6 GB)
    if (getenv("PROBE_BIG")) {
        float4 *big = nullptr;
        const int64_t bb = int64_t(9) << 30;
        if (cudaMalloc(&big, bb) == cudaSuccess) {
            cudaMemset(big, 0, bb);
            for (int64_t tb : {int64_t(1) << 30, int64_t(2) << 30, int64_t(4) << 30, int64_t(8) << 30})
                run<512, 4>(big, tb, sms, out);
            cudaFree(big);
        }
    }
    // narrow rows (narrow feature panels for X >> L2, e.g. products F = 100):
    // 16..128-byte random rows from an L2-resident table
    if (getenv("PROBE_NARROW"))
        for (int64_t tb : {int64_t(60) << 20, int64_t(78) << 20}) {
            run<16, 8>(tab, tb, sms, out);
            run<32, 8>(tab, tb, sms, out);
            run<64, 8>(tab, tb, sms, out);
            run<128, 8>(tab, tb, sms, out);
        }
    return 0;
}
