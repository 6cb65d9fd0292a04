// Microbenchmark: dependent-chain latency and throughput of DFMA / DMUL / I2F.F64
// on this GPU (used to reason about the model's dependency chains).
#include <cstdio>
#include <cuda_runtime.h>

__global__ void chain(double *out, long long *cyc, double a, double b, int n)
{
    double x = a + threadIdx.x;
    long long t0 = clock64();
#pragma unroll 16
    for (int i = 0; i < n; i++) x = __fma_rn(x, b, a);
    long long t1 = clock64();
    out[threadIdx.x] = x;
    if (threadIdx.x == 0) cyc[0] = t1 - t0;
}

__global__ void chain_i2f(double *out, long long *cyc, unsigned a, int n)
{
    unsigned x = a + threadIdx.x;
    double acc = 0;
    long long t0 = clock64();
#pragma unroll 16
    for (int i = 0; i < n; i++) { double d = __uint2double_rn(x); x = (unsigned)__double2uint_rz(d) + 1u; }
    long long t1 = clock64();
    out[threadIdx.x] = x;
    if (threadIdx.x == 0) cyc[0] = t1 - t0;
}

template <int ILP>
__global__ void thru(double *out, double a, double b, int n)
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
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

int main()
{
    double *out; long long *cyc;
    cudaMalloc(&out, 1 << 26); cudaMalloc(&cyc, 8);
    long long h;
    int n = 4096;
    chain<<<1, 32>>>(out, cyc, 1.0, 0.999999, n); cudaDeviceSynchronize();
    chain<<<1, 32>>>(out, cyc, 1.0, 0.999999, n); cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost);
    printf("DFMA dependent latency: %.2f cycles\n", (double)h / n);
    chain_i2f<<<1, 32>>>(out, cyc, 7, n); cudaDeviceSynchronize();
    chain_i2f<<<1, 32>>>(out, cyc, 7, n); cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost);
    printf("I2F.F64+F2I+IADD dependent latency: %.2f cycles\n", (double)h / n);
    int dev; cudaGetDevice(&dev); cudaDeviceProp p; cudaGetDeviceProperties(&p, dev);
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    int blocks = p.multiProcessorCount * 8, tpb = 256, iters = 2000;
    thru<8><<<blocks, tpb>>>(out, 1.0, 0.999999, iters);
    cudaEventRecord(e0);
    thru<8><<<blocks, tpb>>>(out, 1.0, 0.999999, iters);
    cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    double ops = (double)blocks * tpb * iters * 8;
    printf("DFMA throughput: %.3f Tops/s (%.1f per SM per clk at %d MHz)\n", ops / ms / 1e9,
           ops / (ms * 1e-3) / p.multiProcessorCount / (p.clockRate * 1e3), p.clockRate / 1000);
    return 0;
}
