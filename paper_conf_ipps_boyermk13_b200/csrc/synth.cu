// Synthetic candidate records generated directly in HBM (bench / tests only;
// not part of the method).  Independent CUDA implementation of the closed
// form documented in synth/records.py: SplitMix64 counter outputs per group.
#include <cuda_runtime.h>
#include <stdint.h>

#include "grophecy.h"
#include "internal.h"

namespace grophecy {

__device__ __forceinline__ unsigned long long sm64(unsigned long long seed, unsigned long long k)
{
    unsigned long long z = seed + (k + 1ull) * 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

__global__ void synth_kernel(const grophecy_synth_rule *rules, uint32_t n_rules,
                             unsigned long long n_total, uint32_t X, unsigned long long seed,
                             unsigned long long start, unsigned long long count, uint32_t *skx,
                             uint32_t *nx, uint32_t *ny, uint32_t *iters)
{
    const unsigned long long G = (n_total + X - 1) / X;
    for (unsigned long long j = blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x; j < count;
         j += (unsigned long long)gridDim.x * blockDim.x) {
        const unsigned long long i = start + j;
        const unsigned long long g = i / X;
        const uint32_t x = (uint32_t)(i % X);
        const uint32_t s = (uint32_t)((g * n_rules) / G);
        const grophecy_synth_rule r = rules[s];
        const unsigned long long z0 = sm64(seed, 4 * g), z1 = sm64(seed, 4 * g + 1),
                                 z2 = sm64(seed, 4 * g + 2);
        unsigned long long span = (unsigned long long)r.hi - r.lo + 1;
        uint32_t a = 0, b = 0;
        if (r.kind != GROPHECY_SYNTH_FIXED) {
            a = r.lo + (uint32_t)(z0 % span);
            b = r.lo + (uint32_t)(z1 % span);
        }
        uint32_t vx, vy;
        switch (r.kind) {
        case GROPHECY_SYNTH_SQUARE: vx = a; vy = a; break;
        case GROPHECY_SYNTH_INDEP: vx = a; vy = b; break;
        case GROPHECY_SYNTH_ONED: vx = a; vy = 1; break;
        default: vx = r.lo; vy = r.hi; break;
        }
        const unsigned long long ispan = (unsigned long long)r.it_hi - r.it_lo + 1;
        skx[j] = (s << 16) | x;
        nx[j] = vx;
        ny[j] = vy;
        iters[j] = r.it_lo + (uint32_t)(z2 % ispan);
    }
}

}  // namespace grophecy

using namespace grophecy;

extern "C" int grophecy_synth_records(const grophecy_synth_rule *rules, uint32_t n_rules,
                                      uint64_t n_total, uint32_t n_xforms, uint64_t seed,
                                      uint64_t start, uint64_t count, uint32_t *skx, uint32_t *nx,
                                      uint32_t *ny, uint32_t *iters, void *stream)
{
    if (!rules || n_rules == 0 || n_xforms == 0 || (count && (!skx || !nx || !ny || !iters)) ||
        start + count > n_total) {
        set_error("grophecy_synth_records: bad arguments");
        return GROPHECY_EINVAL;
    }
    if (count == 0) return GROPHECY_OK;
    cudaStream_t st = (cudaStream_t)stream;
    grophecy_synth_rule *drules = nullptr;
    cudaError_t e = cudaMallocAsync((void **)&drules, sizeof(grophecy_synth_rule) * n_rules, st);
    if (e != cudaSuccess) return cuda_fail(e, "cudaMallocAsync(rules)");
    e = cudaMemcpyAsync(drules, rules, sizeof(grophecy_synth_rule) * n_rules,
                        cudaMemcpyHostToDevice, st);
    if (e != cudaSuccess) return cuda_fail(e, "rules H2D");
    int dev = 0, nsm = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    unsigned long long blocks = (count + 255) / 256;
    if (blocks > (unsigned long long)nsm * 16) blocks = (unsigned long long)nsm * 16;
    synth_kernel<<<(unsigned)blocks, 256, 0, st>>>(drules, n_rules, n_total, n_xforms, seed, start,
                                                   count, skx, nx, ny, iters);
    count_launch();
    e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e, "synth_kernel launch");
    // the copy above is from pageable memory, so it has completed on return
    e = cudaFreeAsync(drules, st);
    if (e != cudaSuccess) return cuda_fail(e, "cudaFreeAsync(rules)");
    return GROPHECY_OK;
}
