// PCIe calibration / validation subsystem (§III-C, P:L91-115;
// validation protocol §V-A).
//
// "GROPHECY++ automatically measures the values of the two parameters for
// each new system": alpha = mean time of a 1-byte transfer, beta =
// mean time of a 512 MB transfer / 512 MB, each averaged over ten runs
// (P:L113).  Transfers use pinned host memory (cudaHostAlloc).
// Each transfer is issued and waited for on its own (cudaMemcpyAsync +
// cudaStreamSynchronize) and timed with the host steady clock — the time a
// program observes; CUDA-event times are reported alongside (DESIGN.md
// reading 4).
#include <cuda_runtime.h>
#include <stdint.h>

#include <chrono>
#include <mutex>

#include "grophecy.h"
#include "internal.h"

namespace grophecy {

namespace {
struct XferBuffers {
    void *host = nullptr;
    void *dev = nullptr;
    size_t bytes = 0;
    cudaStream_t stream = nullptr;
    cudaEvent_t e0 = nullptr, e1 = nullptr;
};
constexpr int MAX_DEV = 64;
XferBuffers g_buf[MAX_DEV];
std::mutex g_mu[MAX_DEV];   // one per device: concurrent mode measures all GPUs at once

int ensure(int device, size_t bytes, XferBuffers *&out)
{
    if (device < 0 || device >= MAX_DEV) {
        set_error("device index out of range");
        return GROPHECY_EINVAL;
    }
    XferBuffers &b = g_buf[device];
    cudaError_t e;
    if (!b.stream) {
        if ((e = cudaStreamCreateWithFlags(&b.stream, cudaStreamNonBlocking)) != cudaSuccess)
            return cuda_fail(e, "cudaStreamCreate");
        cudaEventCreate(&b.e0);
        cudaEventCreate(&b.e1);
    }
    if (b.bytes < bytes) {
        if (b.host) cudaFreeHost(b.host);
        if (b.dev) cudaFree(b.dev);
        b.host = b.dev = nullptr;
        b.bytes = 0;
        if ((e = cudaHostAlloc(&b.host, bytes, cudaHostAllocDefault)) != cudaSuccess)
            return cuda_fail(e, "cudaHostAlloc");
        if ((e = cudaMalloc(&b.dev, bytes)) != cudaSuccess) return cuda_fail(e, "cudaMalloc");
        // touch both so first-use costs are not timed
        cudaMemset(b.dev, 0, bytes);
        for (size_t i = 0; i < bytes; i += 4096) ((volatile char *)b.host)[i] = 0;
        b.bytes = bytes;
    }
    out = &b;
    return GROPHECY_OK;
}
}  // namespace

}  // namespace grophecy

using namespace grophecy;

extern "C" {

int grophecy_measure_transfer(int device, int direction, uint64_t bytes, int reps, int warmup,
                              double *mean_wall_s, double *mean_event_s)
{
    if (!mean_wall_s || reps < 1 || warmup < 0 || bytes == 0 || bytes > (1ull << 31) ||
        (direction != GROPHECY_DIR_H2D && direction != GROPHECY_DIR_D2H)) {
        set_error("grophecy_measure_transfer: bad arguments");
        return GROPHECY_EINVAL;
    }
    if (device < 0 || device >= MAX_DEV) {
        set_error("device index out of range");
        return GROPHECY_EINVAL;
    }
    std::lock_guard<std::mutex> lock(g_mu[device]);
    int prev = 0;
    cudaGetDevice(&prev);
    cudaError_t e = cudaSetDevice(device);
    if (e != cudaSuccess) return cuda_fail(e, "cudaSetDevice");
    XferBuffers *b = nullptr;
    int rc = ensure(device, (size_t)bytes, b);
    if (rc) {
        cudaSetDevice(prev);
        return rc;
    }
    const cudaMemcpyKind kind =
        direction == GROPHECY_DIR_H2D ? cudaMemcpyHostToDevice : cudaMemcpyDeviceToHost;
    void *dst = direction == GROPHECY_DIR_H2D ? b->dev : b->host;
    const void *src = direction == GROPHECY_DIR_H2D ? b->host : b->dev;
    double wall = 0.0, ev = 0.0;
    for (int r = 0; r < warmup + reps; r++) {
        auto t0 = std::chrono::steady_clock::now();
        cudaEventRecord(b->e0, b->stream);
        e = cudaMemcpyAsync(dst, src, (size_t)bytes, kind, b->stream);
        cudaEventRecord(b->e1, b->stream);
        if (e == cudaSuccess) e = cudaStreamSynchronize(b->stream);
        auto t1 = std::chrono::steady_clock::now();
        if (e != cudaSuccess) {
            cudaSetDevice(prev);
            return cuda_fail(e, "transfer");
        }
        if (r >= warmup) {
            float ms = 0.f;
            cudaEventElapsedTime(&ms, b->e0, b->e1);
            wall += std::chrono::duration<double>(t1 - t0).count();
            ev += (double)ms * 1e-3;
        }
    }
    *mean_wall_s = wall / reps;
    if (mean_event_s) *mean_event_s = ev / reps;
    cudaSetDevice(prev);
    return GROPHECY_OK;
}

int grophecy_calibrate(int device, int reps, uint64_t large_bytes, grophecy_pcie *out)
{
    if (!out || reps < 1 || large_bytes == 0) {
        set_error("grophecy_calibrate: bad arguments");
        return GROPHECY_EINVAL;
    }
    for (int dir = 0; dir < 2; dir++) {
        double tS = 0.0, tL = 0.0;
        int rc = grophecy_measure_transfer(device, dir, 1, reps, 2, &tS, nullptr);
        if (rc) return rc;
        rc = grophecy_measure_transfer(device, dir, large_bytes, reps, 2, &tL, nullptr);
        if (rc) return rc;
        rc = grophecy_fit_pcie(tS, tL, large_bytes, dir == GROPHECY_DIR_H2D ? &out->h2d : &out->d2h);
        if (rc) return rc;
    }
    return GROPHECY_OK;
}

}  // extern "C"
