// l2_ceiling.cu -- measurement tool of bench.py (not part of the product path):
// the L2 random-row gather ceiling that bounds the panel-mode aggregation
// kernels.  A persistent grid (SMs x 4 CTAs x 8 warps,
// the aggregation kernels' occupancy) gathers random rows of a table sized like
// one panel-major strip block (n_src x 256 B) that stays L2-resident: each warp
// instruction moves two 256-byte rows (half-warps, LDG.128, as the PAIR
// gathers), U independent rows in flight per half-warp, row indices from a
// register hash (no index traffic), and sums them.  The table holds random
// (incompressible) fp32 values.  bench.py times it with CUDA events in the same
// run as the aggregation, with the clocks sampled.
//
// C ABI: l2c_run(table_bytes, iters, &ms, &bytes) -> 0 on success.
#include <cstdint>
#include <cuda_runtime.h>

namespace {

__global__ void fill(float4 *t, int64_t n4, uint32_t seed) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n4; i += (int64_t)gridDim.x * blockDim.x) {
        uint32_t x = (uint32_t)i * 2654435761u ^ seed;
        x ^= x >> 15; x *= 2246822519u; x ^= x >> 13;
        t[i] = make_float4((x & 0xffff) * 1e-5f, (x >> 16) * 1e-5f, (x % 977) * 1e-3f, (x % 613) * 1e-3f);
    }
}

constexpr int U = 8;

__global__ void __launch_bounds__(256, 4) gather(const float4 *__restrict__ tab, uint32_t nrows,
                                                 int iters, uint32_t seed, float *out) {
    const int lane = threadIdx.x & 31;
    const int half = lane >> 4, col = lane & 15;  // 16 lanes x 16 B = one 256-byte row
    uint32_t x = seed ^ ((blockIdx.x * 8u + (threadIdx.x >> 5)) * 2u + half) * 0x9E3779B9u;
    float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
    for (int it = 0; it < iters; ++it) {
        float4 v[U];
#pragma unroll
        for (int k = 0; k < U; ++k) {
            x ^= x << 13; x ^= x >> 17; x ^= x << 5;
            v[k] = __ldg(tab + (int64_t)__umulhi(x, nrows) * 16 + col);  // fast range reduction
        }
#pragma unroll
        for (int k = 0; k < U; ++k) { acc.x += v[k].x; acc.y += v[k].y; acc.z += v[k].z; acc.w += v[k].w; }
    }
    if (acc.x + acc.y + acc.z + acc.w == -1.f) out[0] = acc.x;  // keeps the loads live
}

}  // namespace

extern "C" int l2c_run(int64_t table_bytes, int iters, float *ms_out, double *bytes_out) {
    int dev = 0, sms = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    float4 *tab = nullptr;
    float *out = nullptr;
    if (cudaMalloc(&tab, table_bytes) != cudaSuccess) return 1;
    if (cudaMalloc(&out, 64) != cudaSuccess) { cudaFree(tab); return 1; }
    const uint32_t nrows = (uint32_t)(table_bytes / 256);
    fill<<<sms * 8, 256>>>(tab, table_bytes / 16, 12345u);
    const int blocks = sms * 4;
    gather<<<blocks, 256>>>(tab, nrows, 64, 1u, out);  // warm: table into L2
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    cudaEventRecord(a);
    for (int r = 0; r < 5; ++r) gather<<<blocks, 256>>>(tab, nrows, iters, 7u + r, out);
    cudaEventRecord(b);
    cudaError_t e = cudaEventSynchronize(b);
    float ms = 0.f;
    cudaEventElapsedTime(&ms, a, b);
    *ms_out = ms / 5.f;
    *bytes_out = (double)blocks * 256.0 * 16.0 * U * iters;  // every lane moves 16 B per row
    cudaEventDestroy(a);
    cudaEventDestroy(b);
    cudaFree(tab);
    cudaFree(out);
    return e == cudaSuccess ? 0 : 2;
}
