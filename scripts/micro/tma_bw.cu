// Microbenchmark: streaming read bandwidth of 1-D bulk copies (cp.async.bulk,
// the sweep kernel's record staging) vs plain 16-byte loads, with CTAs that
// do nothing else: how fast can the staging path move a CTA tile?
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/tma_bw scripts/micro/tma_bw.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t su32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

// each CTA: loop over its tiles, copy TILE bytes per array (4 arrays) into
// shared memory with NCOPY bulk copies per array, wait, touch one word
template <int TILE_BYTES, int NCOPY>
__global__ void __launch_bounds__(256) bulk_kernel(const uint32_t *src, size_t n_tiles, uint32_t *sink)
{
    extern __shared__ __align__(128) unsigned char sm[];
    __shared__ unsigned long long bar;
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar)));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    uint32_t phase = 0, acc = 0;
    for (size_t t = blockIdx.x; t < n_tiles; t += gridDim.x) {
        if (threadIdx.x == 0) {
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&bar)),
                         "r"(4 * TILE_BYTES) : "memory");
            for (int a = 0; a < 4; a++)
                for (int q = 0; q < NCOPY; q++) {
                    const uint32_t piece = TILE_BYTES / NCOPY;
                    const unsigned char *g = reinterpret_cast<const unsigned char *>(src) +
                                             ((size_t)a * n_tiles + t) * TILE_BYTES + q * piece;
                    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                                 ::"r"(su32(sm + a * TILE_BYTES + q * piece)), "l"(g), "r"(piece), "r"(su32(&bar))
                                 : "memory");
                }
        }
        asm volatile("{\n .reg .pred p;\nW%=:\n mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n @!p bra W%=;\n}"
                     ::"r"(su32(&bar)), "r"(phase) : "memory");
        phase ^= 1u;
        acc += reinterpret_cast<const uint32_t *>(sm)[threadIdx.x];
        __syncthreads();
    }
    if (acc == 0x12345678u) sink[0] = acc;
}

// plain 16-byte loads of the same tiles (every thread, coalesced)
template <int TILE_BYTES>
__global__ void __launch_bounds__(256) ldg_kernel(const uint4 *src, size_t n_tiles, uint32_t *sink)
{
    uint32_t acc = 0;
    constexpr int V = TILE_BYTES / 16;
    for (size_t t = blockIdx.x; t < n_tiles; t += gridDim.x)
#pragma unroll
        for (int a = 0; a < 4; a++) {
            uint4 v[V / 256];
#pragma unroll
            for (int i = 0; i < V / 256; i++) v[i] = __ldg(src + ((size_t)a * n_tiles + t) * V + i * 256 + threadIdx.x);
#pragma unroll
            for (int i = 0; i < V / 256; i++) acc += v[i].x ^ v[i].w;
        }
    if (acc == 0x12345678u) sink[0] = acc;
}

template <class F>
float time_it(F f)
{
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    f();
    cudaDeviceSynchronize();
    float best = 1e30f;
    for (int r = 0; r < 5; r++) {
        cudaEventRecord(e0);
        f();
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        if (ms < best) best = ms;
    }
    return best;
}

int main()
{
    const size_t bytes = 8ull << 30;   // 8 GiB (>> L2)
    unsigned char *d;
    uint32_t *sink;
    cudaMalloc(&d, bytes);
    cudaMalloc(&sink, 4);
    cudaMemset(d, 1, bytes);
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    constexpr int TB = 16384;
    const size_t n_tiles = bytes / (4 * TB);
    auto k1 = bulk_kernel<TB, 1>;
    auto k4 = bulk_kernel<TB, 4>;
    cudaFuncSetAttribute(k1, cudaFuncAttributeMaxDynamicSharedMemorySize, 4 * TB);
    cudaFuncSetAttribute(k4, cudaFuncAttributeMaxDynamicSharedMemorySize, 4 * TB);
    for (int per_sm = 1; per_sm <= 3; per_sm++) {
        const int grid = sms * per_sm;
        float ms = time_it([&] { k1<<<grid, 256, 4 * TB>>>((const uint32_t *)d, n_tiles, sink); });
        printf("bulk 4x16KB per tile, %d CTA/SM (one tile in flight per CTA): %.0f GB/s\n", per_sm, bytes / ms / 1e6);
        ms = time_it([&] { k4<<<grid, 256, 4 * TB>>>((const uint32_t *)d, n_tiles, sink); });
        printf("bulk 16x4KB per tile, %d CTA/SM: %.0f GB/s\n", per_sm, bytes / ms / 1e6);
    }
    for (int per_sm = 2; per_sm <= 8; per_sm *= 2) {
        const int grid = sms * per_sm;
        float ms = time_it([&] { ldg_kernel<TB><<<grid, 256>>>((const uint4 *)d, n_tiles, sink); });
        printf("ldg.128 tiles, %d CTA/SM: %.0f GB/s\n", per_sm, bytes / ms / 1e6);
    }
    cudaError_t e = cudaGetLastError();
    printf("%s\n", cudaGetErrorString(e));
    return 0;
}
