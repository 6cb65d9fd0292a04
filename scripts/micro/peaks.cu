// Microbenchmark of the per-GPU pipe peaks the op-bound roofline divides by
// (DESIGN.md §6): fp64 FMA-pipe operations/s (DFMA, DMUL, DADD each count 1),
// int32 IMAD operations/s and int->fp64 conversions/s (I2F.F64, XU pipe);
// the issue peak is nominal (1 warp instruction / clock / scheduler).  Each kernel runs many independent chains
// per thread over a persistent grid (every SM full), timed with CUDA events,
// best of 5.  Prints one JSON object.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o peaks peaks.cu
#include <cstdio>
#include <cuda_runtime.h>

constexpr int ILP = 8;

__global__ void k_dfma(double *out, double a, double b, int n)
{
    double x[ILP];
#pragma unroll
    for (int j = 0; j < ILP; j++) x[j] = a + threadIdx.x + j;
    for (int i = 0; i < n; i++)
#pragma unroll
        for (int j = 0; j < ILP; j++) x[j] = __fma_rn(x[j], b, a);
    double s = 0;
#pragma unroll
    for (int j = 0; j < ILP; j++) s += x[j];
    if (s == 12345.678) out[threadIdx.x] = s;
}

__global__ void k_imad(unsigned *out, unsigned a, unsigned b, int n)
{
    unsigned x[ILP];
#pragma unroll
    for (int j = 0; j < ILP; j++) x[j] = a + threadIdx.x + j;
    for (int i = 0; i < n; i++)
#pragma unroll
        for (int j = 0; j < ILP; j++) x[j] = x[j] * b + a;
    unsigned s = 0;
#pragma unroll
    for (int j = 0; j < ILP; j++) s ^= x[j];
    if (s == 0x12345u) out[threadIdx.x] = s;
}

__global__ void k_i2f(double *out, unsigned a, int n)
{
    unsigned long long h[ILP];
#pragma unroll
    for (int j = 0; j < ILP; j++) h[j] = 0ull;
    const unsigned x = a + threadIdx.x;
    for (int i = 0; i < n; i++) {
#pragma unroll
        for (int j = 0; j < ILP; j++)
            h[j] ^= (unsigned long long)__double_as_longlong(__uint2double_rn(x + (unsigned)(i * ILP + j)));
    }
    unsigned long long s = 0;
#pragma unroll
    for (int j = 0; j < ILP; j++) s ^= h[j];
    if (s == 0x12345ull) out[threadIdx.x] = (double)s;
}

template <class F>
static float best_ms(F launch)
{
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    launch();
    cudaDeviceSynchronize();
    float best = 1e30f;
    for (int r = 0; r < 5; r++) {
        cudaEventRecord(e0);
        launch();
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
    int dev = 0;
    cudaDeviceProp p;
    cudaGetDeviceProperties(&p, dev);
    int clk = 0;
    cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, dev);
    void *buf;
    cudaMalloc(&buf, 1 << 20);
    const int tpb = 256, blocks = p.multiProcessorCount * 8, n = 4000;
    const double thr = (double)blocks * tpb * n * ILP;
    float ms_dfma = best_ms([&] { k_dfma<<<blocks, tpb>>>((double *)buf, 1.0, 0.999999, n); });
    float ms_imad = best_ms([&] { k_imad<<<blocks, tpb>>>((unsigned *)buf, 3u, 1664525u, n); });
    float ms_i2f = best_ms([&] { k_i2f<<<blocks, tpb>>>((double *)buf, 3u, n / 4); });
    const double fp64 = thr / (ms_dfma * 1e-3);
    const double imad = thr / (ms_imad * 1e-3);
    const double i2f = thr / 4 / (ms_i2f * 1e-3);
    const double issue = (double)p.multiProcessorCount * 4.0 * clk * 1e3;   // 1 warp-inst/clk/scheduler
    printf("{\"gpu\": \"%s\", \"sms\": %d, \"sm_clock_mhz_attr\": %d, "
           "\"fp64_ops_per_s\": %.6e, \"int_imad_ops_per_s\": %.6e, "
           "\"i2f_f64_ops_per_s\": %.6e, \"issue_warp_inst_per_s_nominal\": %.6e, "
           "\"fp64_per_sm_per_clk\": %.2f, \"imad_per_sm_per_clk\": %.2f, \"i2f_per_sm_per_clk\": %.2f, "
           "\"method\": \"independent chains (ILP %d) x %d threads x %d blocks, CUDA events, best of 5; per-clk figures use the attribute clock\"}\n",
           p.name, p.multiProcessorCount, clk / 1000, fp64, imad, i2f, issue,
           fp64 / p.multiProcessorCount / (clk * 1e3), imad / p.multiProcessorCount / (clk * 1e3),
           i2f / p.multiProcessorCount / (clk * 1e3), ILP, tpb, blocks);
    return 0;
}
