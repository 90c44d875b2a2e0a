// tma_gather_probe.cu -- measurement for DESIGN.md "Blackwell data-movement
// options": random 256-byte row gathers from an L2-resident table (one
// panel-major strip block, n_src x 64 floats) by
//   (a) LDG.128 half-warps, U rows in flight per half-warp (the PAIR kernels'
//       instruction pattern; the bench's l2_ceiling probe), and
//   (b) TMA tile::gather4 (cp.async.bulk.tensor.2d ... gather4): one elected
//       thread per CTA issues 4-row gathers into a shared-memory ring of S
//       stages (mbarrier complete_tx), the CTA's warps sum the landed rows
//       from shared memory and release the stage.
// Prints GB/s of gathered row bytes for each.  Not part of the product path.
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/tma_probe bench_probe/tma_gather_probe.cu -lcuda
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { printf("CUDA %s at %d\n", cudaGetErrorString(e_), __LINE__); return 1; } } while (0)

__global__ void fill(float4 *t, int64_t n4) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n4; i += (int64_t)gridDim.x * blockDim.x) {
        uint32_t x = (uint32_t)i * 2654435761u;
        x ^= x >> 15; x *= 2246822519u; x ^= x >> 13;
        t[i] = make_float4((x & 0xffff) * 1e-5f, (x >> 16) * 1e-5f, (x % 977) * 1e-3f, (x % 613) * 1e-3f);
    }
}

template <int U>
__global__ void __launch_bounds__(256, 4) ldg_gather(const float4 *__restrict__ tab, uint32_t nrows, int iters, float *out) {
    const int lane = threadIdx.x & 31, half = lane >> 4, col = lane & 15;
    uint32_t x = 0x9E3779B9u * ((blockIdx.x * 8u + (threadIdx.x >> 5)) * 2u + half + 1);
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
    if (acc.x + acc.y + acc.z + acc.w == -1.f) out[0] = acc.x;
}

// ---- TMA gather4 -----------------------------------------------------------
constexpr int S = 16;         // stages
constexpr int G4 = 4;         // gather4 ops per stage (16 rows = 4 KB)
constexpr int STAGE_BYTES = G4 * 4 * 256;

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

__global__ void __launch_bounds__(256, 1) tma_gather(const __grid_constant__ CUtensorMap tmap, uint32_t nrows,
                                                     int iters, float *out) {
    extern __shared__ __align__(1024) unsigned char smem[];
    __shared__ __align__(8) uint64_t full[S], empty[S];
    const int tid = threadIdx.x;
    if (tid == 0) {
        for (int s = 0; s < S; ++s) {
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&full[s])));
            asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(&empty[s])), "r"(blockDim.x / 32));
        }
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    __syncthreads();
    uint32_t x = 0x9E3779B9u * (blockIdx.x + 1);
    float acc = 0.f;
    // producer (thread 0) keeps S - 1 stages in flight ahead of the consumers
    auto produce = [&](int j) {
        const int s = j % S;
        if (j >= S) {  // wait until the consumers released this stage's previous use
            const uint32_t ph = ((j / S) - 1) & 1;
            asm volatile("{\n .reg .pred p;\n W: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n @!p bra W;\n}"
                         ::"r"(smem_u32(&empty[s])), "r"(ph));
        }
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(&full[s])), "r"(STAGE_BYTES));
        for (int q = 0; q < G4; ++q) {
            int r[4];
            for (int k = 0; k < 4; ++k) { x ^= x << 13; x ^= x >> 17; x ^= x << 5; r[k] = (int)__umulhi(x, nrows); }
            asm volatile(
                "cp.async.bulk.tensor.2d.shared::cluster.global.tile::gather4.mbarrier::complete_tx::bytes"
                " [%0], [%1, {%2, %3, %4, %5, %6}], [%7];"
                ::"r"(smem_u32(smem + s * STAGE_BYTES + q * 1024)), "l"(&tmap), "r"(0),
                  "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(smem_u32(&full[s]))
                : "memory");
        }
    };
    if (tid == 0)
        for (int j = 0; j < S - 1 && j < iters; ++j) produce(j);
    for (int it = 0; it < iters; ++it) {
        if (tid == 0 && it + S - 1 < iters) produce(it + S - 1);
        const int s = it % S;
        const uint32_t ph = (it / S) & 1;
        asm volatile("{\n .reg .pred p;\n W2: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n @!p bra W2;\n}"
                     ::"r"(smem_u32(&full[s])), "r"(ph));
        const float4 *st = reinterpret_cast<const float4 *>(smem + s * STAGE_BYTES);
        const float4 v = st[tid];  // 256 threads x 16 B = the stage's 4 KB
        acc += v.x + v.y + v.z + v.w;
        __syncwarp();
        if ((tid & 31) == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&empty[s])));
    }
    if (acc == -1.f) out[0] = acc;
}

typedef CUresult (*EncodeFn)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *,
                             const cuuint64_t *, const cuuint32_t *, const cuuint32_t *, CUtensorMapInterleave,
                             CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

int main() {
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    int clk = 0;
    cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
    const int64_t table = (int64_t)232965 * 256;  // one Reddit strip block (59.6 MB)
    const uint32_t nrows = (uint32_t)(table / 256);
    float4 *tab; float *out;
    CK(cudaMalloc(&tab, table)); CK(cudaMalloc(&out, 64));
    fill<<<sms * 8, 256>>>(tab, table / 16);
    CK(cudaDeviceSynchronize());
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    float ms;
    // (a) LDG
    {
        const int iters = 600, blocks = sms * 4;
        ldg_gather<8><<<blocks, 256>>>(tab, nrows, 50, out);
        cudaEventRecord(a);
        for (int r = 0; r < 5; ++r) ldg_gather<8><<<blocks, 256>>>(tab, nrows, iters, out);
        cudaEventRecord(b); CK(cudaEventSynchronize(b)); cudaEventElapsedTime(&ms, a, b); ms /= 5;
        const double bytes = (double)blocks * 256 * 16 * 8 * iters;
        printf("{\"probe\": \"ldg_halfwarp_U8\", \"table_MB\": %.1f, \"ms\": %.3f, \"GBs\": %.1f}\n", table / 1e6, ms, bytes / ms / 1e6);
    }
    // (b) TMA gather4
    void *fn = nullptr;
    cudaDriverEntryPointQueryResult q;
    CK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q));
    CUtensorMap tm;
    cuuint64_t dims[2] = {64, nrows};
    cuuint64_t strides[1] = {256};
    cuuint32_t box[2] = {64, 1};
    cuuint32_t estr[2] = {1, 1};
    CUresult cr = ((EncodeFn)fn)(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, tab, dims, strides, box, estr,
                                 CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                                 CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (cr != CUDA_SUCCESS) { printf("{\"probe\": \"tma_gather4\", \"error\": \"encode %d\"}\n", (int)cr); return 0; }
    const int smem = S * STAGE_BYTES;
    CK(cudaFuncSetAttribute(tma_gather, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
    for (int ctas_per_sm : {1, 2, 3}) {
        const int iters = 3000, blocks = sms * ctas_per_sm;
        tma_gather<<<blocks, 256, smem>>>(tm, nrows, 64, out);
        CK(cudaGetLastError());
        cudaEventRecord(a);
        for (int r = 0; r < 3; ++r) tma_gather<<<blocks, 256, smem>>>(tm, nrows, iters, out);
        cudaEventRecord(b); CK(cudaEventSynchronize(b)); cudaEventElapsedTime(&ms, a, b); ms /= 3;
        const double bytes = (double)blocks * STAGE_BYTES * iters;
        printf("{\"probe\": \"tma_gather4_S%d_G%d\", \"ctas_per_sm\": %d, \"table_MB\": %.1f, \"ms\": %.3f, \"GBs\": %.1f}\n",
               S, G4, ctas_per_sm, table / 1e6, ms, bytes / ms / 1e6);
    }
    return 0;
}
