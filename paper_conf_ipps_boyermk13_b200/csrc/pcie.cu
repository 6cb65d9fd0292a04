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
#include <cstdlib>
#include <mutex>

#include "grophecy.h"
#include "internal.h"

namespace grophecy {

namespace {
struct XferBuffers {
    void *host = nullptr;
    void *pageable = nullptr;   // malloc'd host buffer (NEXT-4)
    size_t pbytes = 0;
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

int ensure_pageable(XferBuffers &b, size_t bytes)
{
    if (b.pbytes >= bytes) return GROPHECY_OK;
    std::free(b.pageable);
    b.pageable = std::malloc(bytes);
    b.pbytes = 0;
    if (!b.pageable) {
        set_error("malloc(pageable buffer) failed");
        return GROPHECY_ECUDA;
    }
    for (size_t i = 0; i < bytes; i += 4096) ((volatile char *)b.pageable)[i] = 0;   // fault in
    b.pbytes = bytes;
    return GROPHECY_OK;
}
}  // namespace

}  // namespace grophecy

using namespace grophecy;

extern "C" {

int grophecy_measure_transfer(int device, int direction, uint64_t bytes, int reps, int warmup,
                              double *mean_wall_s, double *mean_event_s)
{
    return grophecy_measure_transfer_mem(device, direction, GROPHECY_MEM_PINNED, bytes, reps,
                                         warmup, mean_wall_s, mean_event_s);
}

// Pinned (the paper's default) or pageable (malloc) host memory; the
// same per-transfer protocol (reading 4).
int grophecy_measure_transfer_mem(int device, int direction, int memory, uint64_t bytes, int reps,
                                  int warmup, double *mean_wall_s, double *mean_event_s)
{
    if (!mean_wall_s || reps < 1 || warmup < 0 || bytes == 0 || bytes > (1ull << 31) ||
        (direction != GROPHECY_DIR_H2D && direction != GROPHECY_DIR_D2H) ||
        (memory != GROPHECY_MEM_PINNED && memory != GROPHECY_MEM_PAGEABLE)) {
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
    if (memory == GROPHECY_MEM_PAGEABLE && (rc = ensure_pageable(*b, (size_t)bytes))) {
        cudaSetDevice(prev);
        return rc;
    }
    void *hbuf = memory == GROPHECY_MEM_PINNED ? b->host : b->pageable;
    const cudaMemcpyKind kind =
        direction == GROPHECY_DIR_H2D ? cudaMemcpyHostToDevice : cudaMemcpyDeviceToHost;
    void *dst = direction == GROPHECY_DIR_H2D ? b->dev : hbuf;
    const void *src = direction == GROPHECY_DIR_H2D ? hbuf : b->dev;
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

// Pinned allocation overhead: cudaHostAlloc and cudaFreeHost timed
// separately by the host steady clock; one discarded pair first.
int grophecy_measure_pin_alloc(int device, uint64_t bytes, int reps, double *mean_alloc_s,
                               double *mean_free_s)
{
    if (!mean_alloc_s || reps < 1 || bytes == 0 || bytes > (1ull << 34) || device < 0 ||
        device >= MAX_DEV) {
        set_error("grophecy_measure_pin_alloc: bad arguments");
        return GROPHECY_EINVAL;
    }
    std::lock_guard<std::mutex> lock(g_mu[device]);
    int prev = 0;
    cudaGetDevice(&prev);
    cudaError_t e = cudaSetDevice(device);
    if (e != cudaSuccess) return cuda_fail(e, "cudaSetDevice");
    double ta = 0.0, tf = 0.0;
    constexpr int WARM = 3;   // the driver's pinned pool grows on the first allocations
    for (int r = 0; r < reps + WARM; r++) {
        void *p = nullptr;
        auto t0 = std::chrono::steady_clock::now();
        e = cudaHostAlloc(&p, (size_t)bytes, cudaHostAllocDefault);
        auto t1 = std::chrono::steady_clock::now();
        if (e == cudaSuccess) e = cudaFreeHost(p);
        auto t2 = std::chrono::steady_clock::now();
        if (e != cudaSuccess) {
            cudaSetDevice(prev);
            return cuda_fail(e, "cudaHostAlloc / cudaFreeHost");
        }
        if (r >= WARM) {
            ta += std::chrono::duration<double>(t1 - t0).count();
            tf += std::chrono::duration<double>(t2 - t1).count();
        }
    }
    *mean_alloc_s = ta / reps;
    if (mean_free_s) *mean_free_s = tf / reps;
    cudaSetDevice(prev);
    return GROPHECY_OK;
}

// The paper's two-measurement protocol for each link of the memory
// model, plus the allocation line from a one-page and a large allocation.
int grophecy_calibrate_memory(int device, int reps, uint64_t large_bytes, grophecy_memory_model *out)
{
    if (!out || reps < 1 || large_bytes < 4096 || large_bytes > (1ull << 31)) {
        set_error("grophecy_calibrate_memory: bad arguments");
        return GROPHECY_EINVAL;
    }
    for (int mem = 0; mem < 2; mem++) {
        grophecy_pcie &pc = mem == GROPHECY_MEM_PINNED ? out->pinned : out->pageable;
        for (int dir = 0; dir < 2; dir++) {
            double tS = 0.0, tL = 0.0;
            int rc = grophecy_measure_transfer_mem(device, dir, mem, 1, reps, 2, &tS, nullptr);
            if (!rc) rc = grophecy_measure_transfer_mem(device, dir, mem, large_bytes, reps, 2, &tL, nullptr);
            if (!rc) rc = grophecy_fit_pcie(tS, tL, large_bytes, dir == GROPHECY_DIR_H2D ? &pc.h2d : &pc.d2h);
            if (rc) return rc;
        }
    }
    double aS = 0.0, fS = 0.0, aL = 0.0, fL = 0.0;
    int rc = grophecy_measure_pin_alloc(device, 4096, reps, &aS, &fS);
    if (!rc) rc = grophecy_measure_pin_alloc(device, large_bytes, reps, &aL, &fL);
    if (!rc) rc = grophecy_fit_pcie(aS + fS, aL + fL, large_bytes, &out->pin_alloc);
    return rc;
}

// DESIGN.md reading 17: per array, pinned = allocation + pinned transfers,
// pageable = pageable transfers (its malloc is the program's own); the
// cheaper wins, pinned on ties.  Sums left to right.
int grophecy_choose_memory(const grophecy_memory_model *m, uint64_t h2d_bytes, uint64_t d2h_bytes,
                           uint64_t footprint_bytes, grophecy_memory_choice *out)
{
    if (!m || !out || footprint_bytes < h2d_bytes || footprint_bytes < d2h_bytes) {
        set_error("grophecy_choose_memory: bad arguments");
        return GROPHECY_EINVAL;
    }
    const double a = (h2d_bytes || d2h_bytes) ? grophecy_pcie_time(&m->pin_alloc, footprint_bytes) : 0.0;
    const double pin = (a + grophecy_pcie_time(&m->pinned.h2d, h2d_bytes)) +
                       grophecy_pcie_time(&m->pinned.d2h, d2h_bytes);
    const double pg = grophecy_pcie_time(&m->pageable.h2d, h2d_bytes) +
                      grophecy_pcie_time(&m->pageable.d2h, d2h_bytes);
    out->t_pinned_s = pin;
    out->t_pageable_s = pg;
    out->memory = pin <= pg ? GROPHECY_MEM_PINNED : GROPHECY_MEM_PAGEABLE;
    out->reserved = 0;
    return GROPHECY_OK;
}

}  // extern "C"
