// Best transformation per group ("the
// predicted kernel execution time is the predicted time of the best-
// performing version of the kernel").  A group is a maximal run of
// consecutive records with equal (skeleton, nx, ny, iters) — one projection
// point whose records differ only by transformation.
//
//   1. grophecy_eval projects every candidate into temporary device buffers;
//   2. group_count: run heads per 1024-record block;
//   3. group_scan:  exclusive scan of the block counts (one CTA) -> group ids;
//   4. group_reduce: each head walks its run and writes the argmin
//      (t, index) over valid finite records (ties: lowest index).
// Also the other NEXT elementwise entry points: the predicted speedup per
// group and the break-even iteration count (NEXT-2).
#include <cuda_runtime.h>
#include <stdint.h>

#include "grophecy.h"
#include "internal.h"

namespace grophecy {

constexpr int G_THREADS = 256;
constexpr int G_RPT = 4;
constexpr int G_BLOCK = G_THREADS * G_RPT;

__device__ __forceinline__ bool same_group(const uint32_t *skx, const uint32_t *nx,
                                           const uint32_t *ny, const uint32_t *it,
                                           unsigned long long a, unsigned long long b)
{
    return (skx[a] >> 16) == (skx[b] >> 16) && nx[a] == nx[b] && ny[a] == ny[b] && it[a] == it[b];
}

__device__ __forceinline__ unsigned block_heads(const grophecy_batch &B, unsigned long long r0,
                                                unsigned &mask)
{
    mask = 0;
    for (int j = 0; j < G_RPT; j++) {
        const unsigned long long i = r0 + j;
        if (i >= B.n) break;
        if (i == 0 || !same_group(B.skx, B.nx, B.ny, B.iters, i, i - 1)) mask |= 1u << j;
    }
    return __popc(mask);
}

__global__ void group_count(grophecy_batch B, unsigned long long *counts)
{
    __shared__ unsigned s;
    if (threadIdx.x == 0) s = 0;
    __syncthreads();
    unsigned m;
    const unsigned c = block_heads(B, (unsigned long long)blockIdx.x * G_BLOCK + threadIdx.x * G_RPT, m);
    const unsigned w = __reduce_add_sync(0xffffffffu, c);
    if ((threadIdx.x & 31) == 0 && w) atomicAdd(&s, w);
    __syncthreads();
    if (threadIdx.x == 0) counts[blockIdx.x] = s;
}

// exclusive scan of nb counts in place; total -> *total
__global__ void group_scan(unsigned long long *counts, unsigned long long nb,
                          unsigned long long *total)
{
    __shared__ unsigned long long wsum[32];
    __shared__ unsigned long long carry;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    if (threadIdx.x == 0) carry = 0;
    __syncthreads();
    for (unsigned long long base = 0; base < nb; base += blockDim.x) {
        const unsigned long long i = base + threadIdx.x;
        const unsigned long long v = i < nb ? counts[i] : 0ull;
        unsigned long long inc = v;
        for (int o = 1; o < 32; o <<= 1) {
            const unsigned long long u = __shfl_up_sync(0xffffffffu, inc, o);
            if (lane >= o) inc += u;
        }
        if (lane == 31) wsum[warp] = inc;
        __syncthreads();
        if (warp == 0) {
            unsigned long long x = lane < (int)(blockDim.x / 32) ? wsum[lane] : 0ull;
            for (int o = 1; o < 32; o <<= 1) {
                const unsigned long long u = __shfl_up_sync(0xffffffffu, x, o);
                if (lane >= o) x += u;
            }
            wsum[lane] = x;   // inclusive over warps
        }
        __syncthreads();
        const unsigned long long before = (warp ? wsum[warp - 1] : 0ull) + carry;
        if (i < nb) counts[i] = before + inc - v;
        __syncthreads();
        if (threadIdx.x == blockDim.x - 1) carry = before + inc;
        __syncthreads();
    }
    if (threadIdx.x == 0) *total = carry;
}

__global__ void group_reduce(grophecy_batch B, const unsigned long long *offsets,
                             const double *t, const unsigned long long *h2d,
                             const unsigned long long *d2h, grophecy_group_result *out,
                             unsigned long long capacity)
{
    __shared__ unsigned wtot[G_THREADS / 32];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const unsigned long long r0 = (unsigned long long)blockIdx.x * G_BLOCK + threadIdx.x * G_RPT;
    unsigned m;
    const unsigned c = block_heads(B, r0, m);
    unsigned inc = c;
    for (int o = 1; o < 32; o <<= 1) {
        const unsigned u = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane >= o) inc += u;
    }
    if (lane == 31) wtot[warp] = inc;
    __syncthreads();
    unsigned before = 0;
    for (int w = 0; w < warp; w++) before += wtot[w];
    unsigned long long gid = offsets[blockIdx.x] + before + inc - c;
    for (int j = 0; j < G_RPT; j++) {
        if (!((m >> j) & 1u)) continue;
        const unsigned long long i0 = r0 + j;
        double bt = __longlong_as_double(0x7ff0000000000000LL);
        unsigned long long bi = ~0ull, r = i0;
        for (; r < B.n && (r == i0 || same_group(B.skx, B.nx, B.ny, B.iters, r, i0)); r++) {
            const double v = t[r];
            // valid records have non-NaN times; infeasible ones are +inf
            if (v < __longlong_as_double(0x7ff0000000000000LL) && (bi == ~0ull || v < bt)) {
                bt = v;
                bi = r;
            }
        }
        if (gid < capacity) {
            grophecy_group_result g;
            g.best_t_s = bt;
            g.first = B.index_base + i0;
            g.count = r - i0;
            g.best_index = bi == ~0ull ? ~0ull : B.index_base + bi;
            g.h2d_bytes = bi == ~0ull ? 0ull : h2d[bi];
            g.d2h_bytes = bi == ~0ull ? 0ull : d2h[bi];
            out[gid] = g;
        }
        gid++;
    }
}

// S_g = t_cpu[g] / t_gpu[g]
__global__ void speedup_kernel(const grophecy_group_result *g, const double *t_cpu,
                               unsigned long long n, double *out)
{
    for (unsigned long long i = blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x; i < n;
         i += (unsigned long long)gridDim.x * blockDim.x)
        out[i] = __ddiv_rn(t_cpu[i], g[i].best_t_s);
}

// Break-even iteration count (include/grophecy.h grophecy_crossover)
__global__ void crossover_kernel(const double *ti, const double *to, const double *th,
                                 const double *td, const double *cv, double cs,
                                 unsigned long long n, double *nbe, unsigned long long *imin)
{
    for (unsigned long long i = blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x; i < n;
         i += (unsigned long long)gridDim.x * blockDim.x) {
        const double c = cv ? __ldcs(cv + i) : cs;
        const double t_iter = __ldcs(ti + i);
        const double F = __dadd_rn(__dadd_rn(__ldcs(to + i), __ldcs(th + i)), __ldcs(td + i));
        const double den = __dsub_rn(c, t_iter);
        double v;
        if (isnan(F) || isnan(den)) v = __longlong_as_double(0x7ff8000000000000LL);
        else v = den > 0.0 ? __ddiv_rn(F, den) : __longlong_as_double(0x7ff0000000000000LL);
        unsigned long long m;
        if (!(v < 18446744073709551616.0)) m = ~0ull;   // NaN, +inf, >= 2^64
        else if (v < 1.0) m = 1ull;
        else {
            const unsigned long long f = (unsigned long long)floor(v);   // exact: v < 2^64
            m = f == ~0ull ? ~0ull : f + 1ull;
        }
        if (nbe) __stcs(nbe + i, v);
        if (imin) __stcs(imin + i, m);
    }
}

unsigned elementwise_grid(unsigned long long n)
{
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const unsigned long long want = (n + 255) / 256;
    const unsigned long long cap = (unsigned long long)sms * 8;
    return (unsigned)(want < cap ? (want ? want : 1) : cap);
}

}  // namespace grophecy

using namespace grophecy;

extern "C" int grophecy_group_speedup(const grophecy_group_result *groups, const double *t_cpu,
                                      uint64_t n, double *out, void *stream)
{
    if (n && (!groups || !t_cpu || !out)) {
        set_error("grophecy_group_speedup: null argument");
        return GROPHECY_EINVAL;
    }
    if (!n) return GROPHECY_OK;
    speedup_kernel<<<elementwise_grid(n), 256, 0, (cudaStream_t)stream>>>(groups, t_cpu, n, out);
    count_launch();
    const cudaError_t e = cudaGetLastError();
    return e == cudaSuccess ? GROPHECY_OK : cuda_fail(e, "grophecy_group_speedup");
}

extern "C" int grophecy_crossover(const double *t_iter, const double *t_once, const double *t_h2d,
                                  const double *t_d2h, const double *t_cpu_iter,
                                  double t_cpu_iter_scalar, uint64_t n, double *n_be,
                                  uint64_t *iters_min, void *stream)
{
    if (n && (!t_iter || !t_once || !t_h2d || !t_d2h)) {
        set_error("grophecy_crossover: null argument");
        return GROPHECY_EINVAL;
    }
    if (!n || (!n_be && !iters_min)) return GROPHECY_OK;
    crossover_kernel<<<elementwise_grid(n), 256, 0, (cudaStream_t)stream>>>(
        t_iter, t_once, t_h2d, t_d2h, t_cpu_iter, t_cpu_iter_scalar, n, n_be,
        (unsigned long long *)iters_min);
    count_launch();
    const cudaError_t e = cudaGetLastError();
    return e == cudaSuccess ? GROPHECY_OK : cuda_fail(e, "grophecy_crossover");
}

extern "C" int grophecy_group_best(grophecy_space *s, const grophecy_pcie *pc,
                                   const grophecy_batch *b, grophecy_group_result *device_out,
                                   uint64_t capacity, uint64_t *n_groups, void *stream)
{
    if (!s || !pc || !b || !n_groups || (capacity && !device_out)) {
        set_error("grophecy_group_best: null argument");
        return GROPHECY_EINVAL;
    }
    *n_groups = 0;
    if (b->stripe_len) {
        set_error("grophecy_group_best: striped batches are not supported (groups need contiguous indices)");
        return GROPHECY_EINVAL;
    }
    if (b->n == 0) return GROPHECY_OK;
    DeviceGuard guard(s->device);
    cudaStream_t st = (cudaStream_t)stream;
    const unsigned long long n = b->n;
    const unsigned long long nb = (n + G_BLOCK - 1) / G_BLOCK;
    const size_t bytes = n * 24 + (nb + 1) * 8;
    cudaError_t e;
    if (s->gscratch_bytes < bytes) {   // space-owned scratch, grown on demand
        if (s->gscratch) cudaFree(s->gscratch);
        s->gscratch = nullptr;
        s->gscratch_bytes = 0;
        if ((e = cudaMalloc(&s->gscratch, bytes)) != cudaSuccess)
            return cuda_fail(e, "cudaMalloc(group scratch)");
        s->gscratch_bytes = bytes;
    }
    char *tmp = (char *)s->gscratch;
    double *t = (double *)tmp;
    unsigned long long *h2d = (unsigned long long *)(tmp + n * 8);
    unsigned long long *d2h = (unsigned long long *)(tmp + n * 16);
    unsigned long long *counts = (unsigned long long *)(tmp + n * 24);
    unsigned long long *total = counts + nb;
    int rc = grophecy_eval(s, pc, b, (uint64_t *)h2d, (uint64_t *)d2h, t, stream);
    if (rc) return rc;
    group_count<<<(unsigned)nb, G_THREADS, 0, st>>>(*b, counts);
    group_scan<<<1, 1024, 0, st>>>(counts, nb, total);
    group_reduce<<<(unsigned)nb, G_THREADS, 0, st>>>(*b, counts, t, h2d, d2h, device_out, capacity);
    count_launch(3);
    unsigned long long ng = 0;
    e = cudaGetLastError();
    if (e == cudaSuccess) e = cudaMemcpyAsync(&ng, total, 8, cudaMemcpyDeviceToHost, st);
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    if (e != cudaSuccess) return cuda_fail(e, "grophecy_group_best");
    *n_groups = ng;
    if (ng > capacity) {
        set_error("more groups than capacity (first `capacity` written)");
        return GROPHECY_ELIMIT;
    }
    return GROPHECY_OK;
}
