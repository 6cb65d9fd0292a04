/*
 * grophecy.h — C ABI of the B200-native GROPHECY++ projection engine.
 *
 * The engine is the data-parallel hot path of GROPHECY++ (Boyer, Meng,
 * Kumaran, "Improving GPU Performance Prediction with Data Transfer
 * Modeling", IPDPS 2013; /root/reference/PAPER.md, cited as P:Lnnn):
 * for every candidate (code skeleton x transformation x problem size) it
 *   1. analyses data usage across the kernel sequence to find the bytes that
 *      must cross PCIe in each direction           (§III-B),
 *   2. prices each per-array transfer with the two-measurement linear PCIe
 *      model T(d) = alpha + beta*d                  (§III-C, Eq. (1)),
 *   3. projects every kernel's GPU time with an MWP/CWP model (GROPHECY [15],
 *      Hong & Kim [6]; P:L13, L67, L123 — formula read in DESIGN.md §3 N5),
 * sums them and selects the fastest candidate.
 *
 * Conventions
 *  - extern "C", plain pointers and sizes; no exceptions cross the ABI.
 *  - Every call returns a grophecy_status (0 = OK) unless it returns a value;
 *    grophecy_last_error() returns a thread-local message for the last
 *    non-OK status on the calling thread.
 *  - Bytes are uint64; times are double seconds (IEEE-754 binary64, evaluated
 *    in the fixed order of DESIGN.md §3 — results are bitwise reproducible
 *    and bitwise equal to the CPU oracle's).
 *  - "DEVICE" pointers are CUDA global-memory pointers on the space's device;
 *    "HOST" pointers are host memory (pinned where stated for speed).
 *  - cuda_stream is a cudaStream_t passed as void* (NULL = legacy default
 *    stream).  Asynchronous calls return the LAUNCH status only.
 *  - A grophecy_space is not thread-safe and its best-mode scratch is shared:
 *    use one space per host thread / per concurrently-used stream.
 */
#ifndef GROPHECY_H
#define GROPHECY_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define GROPHECY_ABI_VERSION 4

typedef enum {
    GROPHECY_OK = 0,
    GROPHECY_EINVAL = -1,       /* bad argument / malformed descriptor */
    GROPHECY_ELIMIT = -2,       /* a documented size limit is exceeded */
    GROPHECY_ECUDA = -3,        /* CUDA runtime error (message has details) */
    GROPHECY_ENCCL = -4,        /* NCCL missing or an NCCL call failed */
    GROPHECY_ENOFEASIBLE = -5,  /* best: no valid candidate with finite time */
    GROPHECY_EBADCAND = -6,     /* some records were invalid (see n_invalid) */
    GROPHECY_EINTERNAL = -7     /* internal consistency check failed (a bug) */
} grophecy_status;

/* ---------------------------------------------------------------------- */
/* PCIe model — §III-C                                                     */
/* ---------------------------------------------------------------------- */

/* T(d) = alpha + beta*d for d > 0 bytes; T(0) = 0 (no transfer).  Eq. (1). */
typedef struct { double alpha_s, beta_s_per_byte; } grophecy_link;
/* Separate links per direction (Figs. 2/4 measure each direction). */
typedef struct { grophecy_link h2d, d2h; } grophecy_pcie;

/* The paper's two-measurement fit: alpha = t_small (time of a 1-byte
 * transfer), beta = t_large / large_bytes (paper: 512 MB, read as 2^29 B).
 * Pure host function.  EINVAL if out == NULL, t_small < 0, t_large <= 0,
 * large_bytes == 0, or either time is not finite. */
int grophecy_fit_pcie(double t_small_s, double t_large_s, uint64_t large_bytes,
                      grophecy_link *out);

/* Eq. (1) on the host: 0 for bytes == 0, else alpha + beta*(double)bytes. */
double grophecy_pcie_time(const grophecy_link *link, uint64_t bytes);

/* ---------------------------------------------------------------------- */
/* Design-space description                                                */
/* ---------------------------------------------------------------------- */

/* A size-affine integer: v = c0 + floor((c1*nx + c2*ny + c3*nx*ny) / 8),
 * evaluated in int64 (eighths keep halves/quarters of a dimension integral).
 * |c1|,|c2|,|c3| <= 2^15. */
typedef struct { int32_t c0, c1, c2, c3; } grophecy_affine8;

enum { GROPHECY_ARRAY_LIVEOUT = 1u };   /* written data goes back to the CPU;
                                           clear = "temporary" hint */
enum { GROPHECY_R = 1u, GROPHECY_W = 2u };   /* region mode bits; R|W = read-modify-write */
enum { GROPHECY_REGION_WHOLE = 1u };    /* irregular access: the whole array may be
                                           referenced.  With W in the mode it
                                           is a "may-write": the kernel may write any
                                           element, so it counts as a whole-array read
                                           + write (reading 10) */
enum { GROPHECY_KERNEL_PER_ITER = 1u }; /* runs every iteration; else once */

/* An array of planes x rows x cols elements (row-major), extents clamped at
 * 0.  planes = {1, 0, 0, 0} for the 2-D arrays of the paper's workloads;
 * rank-3 arrays (N4r) have any other planes
 * expression.  56 bytes. */
typedef struct {
    grophecy_affine8 rows, cols;
    uint32_t elem_bytes, flags;
    grophecy_affine8 planes;
} grophecy_array_desc;

/* A bounded regular section (Havlak-Kennedy [5]) of `array` accessed
 * by `kernel` (program order index): rows r0, r0 + r_step, ... and columns
 * c0, c0 + c_step, ... inside the box [r0, r1) x [c0, c1) clamped to the
 * array (the lattice stays anchored at the unclamped r0 / c0; lo >= hi is
 * empty).  r_step / c_step: 0 or 1 = dense, else <= GROPHECY_MAX_STEP and the
 * least common multiple of one array's row (column) steps must be
 * <= GROPHECY_MAX_STEP_LCM.  Planes [p0, p1) (dense, clamped to the array's
 * planes; 2-D arrays: {0,0,0,0} and {1,0,0,0}).  WHOLE regions ignore the box,
 * the planes and the steps.  104 bytes. */
typedef struct {
    uint8_t kernel, array, mode, flags;
    grophecy_affine8 r0, r1, c0, c1;
    uint16_t r_step, c_step;
    grophecy_affine8 p0, p1;
} grophecy_region_desc;

typedef struct { grophecy_affine8 work_items; uint32_t flags; } grophecy_kernel_desc;

/* Characteristics of one kernel under one transformation, as GROPHECY's
 * characteristic synthesis would supply them (DESIGN.md §3 N5):
 * threads per block, work items per thread, registers per thread, shared
 * memory per block, and per-thread instruction counts (total, coalesced /
 * uncoalesced memory, uncoalesced transactions per memory warp, bytes per
 * warp load, synchronisations). */
typedef struct {
    uint32_t tpb, ipt, regs_per_thread, smem_per_block;
    double total_insts, coal_insts, uncoal_insts, uncoal_per_mw, load_bytes_per_warp,
        synch_insts;
} grophecy_kx_desc;

/* Skeleton flags.  HULL: data usage by the approximate BRS algebra instead of
 * exact element sets — per array, a read section is "previously written"
 * when one write section of an earlier kernel contains it, and the UNIONs of
 * the remaining read sections (-> H2D) and of all write sections (-> D2H) are
 * Havlak-Kennedy hulls [min l : max u : gcd] per dimension ([5];
 * DESIGN.md N4h).  Never smaller than the exact counts; equal for
 * whole-array workloads. */
enum { GROPHECY_SKEL_HULL = 1u };

/* One code skeleton: a kernel sequence, its arrays and access regions, and
 * the characteristics table kx[x * n_kernels + k] for n_xforms
 * transformations; flags: GROPHECY_SKEL_*; reserved must be 0. */
typedef struct {
    uint32_t n_kernels, n_arrays, n_regions, n_xforms;
    const grophecy_kernel_desc *kernels;
    const grophecy_array_desc *arrays;
    const grophecy_region_desc *regions;
    const grophecy_kx_desc *kx;
    uint32_t flags, reserved;
} grophecy_skeleton_desc;

/* The modelled GPU ("configured to reflect different GPU architectures"). */
typedef struct {
    uint32_t n_sm, warp_size, max_threads_per_block, max_blocks_per_sm, max_threads_per_sm,
        regs_per_sm, smem_per_sm;
    double freq_hz, mem_bw_Bps, mem_ld_cycles, dep_del_coal, dep_del_uncoal, issue_cycles;
} grophecy_gpu_model;

/* Limits checked by grophecy_space_validate / _create (ELIMIT / EINVAL):
 *   1 <= n_skels <= 65536; 1 <= n_xforms <= 65536; 1 <= n_kernels <= 32;
 *   n_arrays <= 16; n_regions <= 256; <= 32 regions per array;
 *   region.kernel < n_kernels, region.array < n_arrays, mode in {R, W, R|W},
 *   region steps <= 64, lcm of one array's row (column) steps <= 64;
 *   skeleton flags within GROPHECY_SKEL_HULL;
 *   1 <= tpb <= 65536, 1 <= ipt <= 65536; instruction counts finite, >= 0,
 *   total >= coal + uncoal, uncoal_per_mw >= 1, load_bytes_per_warp > 0;
 *   GPU integers >= 1 and GPU doubles finite and > 0; elem_bytes >= 1. */
#define GROPHECY_MAX_SKELS 65536u
#define GROPHECY_MAX_XFORMS 65536u
#define GROPHECY_MAX_KERNELS 32u
#define GROPHECY_MAX_ARRAYS 16u
#define GROPHECY_MAX_REGIONS 256u
#define GROPHECY_MAX_REGIONS_PER_ARRAY 32u
#define GROPHECY_MAX_DIM (1u << 20)
#define GROPHECY_MAX_STEP 64u
#define GROPHECY_MAX_STEP_LCM 64u

/* Pure host validation of a design space (no CUDA). */
int grophecy_space_validate(const grophecy_skeleton_desc *skels, uint32_t n_skels,
                            const grophecy_gpu_model *gpu);

typedef struct grophecy_space grophecy_space;   /* opaque; owns device tables + scratch */

/* Validate, precompute per-(kernel, transformation) constants on the host and
 * upload the tables to `device`.  Copies its inputs: the caller may free
 * them on return.  On error *out is NULL. */
int grophecy_space_create(const grophecy_skeleton_desc *skels, uint32_t n_skels,
                          const grophecy_gpu_model *gpu, int device, grophecy_space **out);
void grophecy_space_destroy(grophecy_space *space);

/* ---------------------------------------------------------------------- */
/* Candidate batches                                                       */
/* ---------------------------------------------------------------------- */

/* Struct-of-arrays candidate records, DEVICE pointers, length n, 16-byte
 * aligned.  skx = (skeleton << 16) | transformation.  Global index of
 * record i (used for tie-breaking and reported by best): index_base + i when
 * stripe_len == 0; otherwise the batch is a rank's stripes of a larger
 * workload stored back to back and record i is
 *   index_base + (i / stripe_len) * stripe_stride + i % stripe_len
 * (stripe_stride >= stripe_len, else EINVAL; an increasing map, so ties still
 * resolve to the lowest global index).  The map only changes reported
 * indices: eval outputs stay positional, group_best rejects striped batches.
 * A record is valid iff skeleton < n_skels, transformation < that
 * skeleton's n_xforms, 1 <= nx, ny <= 2^20 and iters >= 1. */
typedef struct {
    const uint32_t *skx, *nx, *ny, *iters;
    uint64_t n, index_base;
    uint64_t stripe_len, stripe_stride;   /* 0, 0: contiguous */
} grophecy_batch;

/* Project every candidate.  Outputs are DEVICE arrays of length n owned by
 * the caller: h2d_bytes[i], d2h_bytes[i] (exact), t_total_s[i] (+inf when a
 * transformation cannot run: zero occupancy).  Invalid records produce
 * (0, 0, NaN) and are counted in the space's invalid counter.  Async. */
int grophecy_eval(const grophecy_space *space, const grophecy_pcie *pcie,
                  const grophecy_batch *batch, uint64_t *h2d_bytes, uint64_t *d2h_bytes,
                  double *t_total_s, void *cuda_stream);

/* Components of each projected time (DEVICE arrays of length n, each may be
 * NULL): t_iter_s = sum of per-iteration kernel times, t_once_s = sum of
 * run-once kernel times, t_h2d_s / t_d2h_s = summed per-array transfer times,
 * so that  t_total_s = ((t_once + iters * t_iter) + t_h2d) + t_d2h  exactly
 * (P:L77, L147, L167).  "Kernel only" = t_once + iters * t_iter and
 * "transfer only" = t_h2d + t_d2h are the paper's Table II predictors
 * (P:L251); iteration sweeps follow in closed form (Figs. 8/10/12).
 * Invalid records get NaN in every component. */
typedef struct { double *t_iter_s, *t_once_s, *t_h2d_s, *t_d2h_s; } grophecy_parts;

/* grophecy_eval plus the time components of every candidate.  Async. */
int grophecy_eval_parts(const grophecy_space *space, const grophecy_pcie *pcie,
                        const grophecy_batch *batch, uint64_t *h2d_bytes, uint64_t *d2h_bytes,
                        double *t_total_s, const grophecy_parts *parts, void *cuda_stream);

/* Synchronise the stream, return the number of invalid records seen by
 * grophecy_eval on this space since the last call, and reset the counter. */
int grophecy_invalid_count(grophecy_space *space, uint64_t *count, void *cuda_stream);

/* The selected candidate: minimum (t_total_s, index) over valid records with
 * finite time, ties to the lowest global index.  48 bytes. */
typedef struct {
    double t_total_s;      /* +inf when none */
    uint64_t index;        /* global index; UINT64_MAX when none */
    uint64_t h2d_bytes, d2h_bytes;   /* of the selected candidate */
    uint64_t n_invalid;    /* invalid records in the batch */
    uint64_t n_valid;      /* valid records (finite or not) */
} grophecy_best_result;

/* Fused projection + argmin; writes one result to HOST memory and
 * synchronises the stream.  Returns ENOFEASIBLE if nothing qualifies
 * (result still filled), EBADCAND if n_invalid > 0 (result still filled). */
int grophecy_best(grophecy_space *space, const grophecy_pcie *pcie,
                  const grophecy_batch *batch, grophecy_best_result *host_out,
                  void *cuda_stream);

/* Asynchronous variant: one launch; the result lands in DEVICE memory.
 * If accumulate != 0 the batch's result is merged (min-loc, counters summed)
 * into the existing *device_out instead of overwriting it. */
int grophecy_best_async(grophecy_space *space, const grophecy_pcie *pcie,
                        const grophecy_batch *batch, grophecy_best_result *device_out,
                        int accumulate, void *cuda_stream);

/* Min-loc combine of `count` results (e.g. one per rank after an all-gather):
 * device_in and device_out are DEVICE pointers; one tiny launch. */
int grophecy_best_combine(const grophecy_best_result *device_in, uint32_t count,
                          grophecy_best_result *device_out, void *cuda_stream);
/* The same combine on the host (pure C, no CUDA). */
int grophecy_best_combine_host(const grophecy_best_result *in, uint32_t count,
                               grophecy_best_result *out);

/* Cross-GPU min-loc: every rank calls this with
 * its shard (batch.index_base = the global index of its first record) and
 * an ncclComm_t of the ranks (one rank per GPU); the fused best kernel runs
 * on the shard, the ranks' results are all-gathered by NCCL on cuda_stream,
 * and every rank receives the global best (lexicographic min of (t, global
 * index)) in host_out.  Synchronises the stream.  NCCL is resolved at run
 * time (libnccl.so.2, or the path in GROPHECY_NCCL_LIB): ENCCL if missing or
 * on an NCCL error; status otherwise as grophecy_best for the global result. */
int grophecy_best_allreduce(grophecy_space *space, const grophecy_pcie *pcie,
                            const grophecy_batch *batch, void *nccl_comm,
                            grophecy_best_result *host_out, void *cuda_stream);
/* The same min-loc for a result already in DEVICE memory (e.g. accumulated
 * by several grophecy_best_async launches over a rank's batches): NCCL
 * all-gather of the ranks' device_in on cuda_stream, combine, global best to
 * host_out on every rank.  Synchronises the stream; errors as above. */
int grophecy_best_allreduce_result(grophecy_space *space, const grophecy_best_result *device_in,
                                   void *nccl_comm, grophecy_best_result *host_out,
                                   void *cuda_stream);
/* Communicator helpers (same run-time NCCL): a 128-byte ncclUniqueId for rank
 * 0 to broadcast; ncclCommInitRank on `device` (comm_out: ncclComm_t);
 * ncclCommDestroy. */
int grophecy_nccl_unique_id(void *id_out);
int grophecy_nccl_comm_init(int nranks, int rank, const void *id, int device, void **comm_out);
int grophecy_nccl_comm_destroy(void *comm);

/* Best transformation per projection point (the predicted kernel time
 * "is the predicted time of the best-performing version").  A group is a
 * maximal run of consecutive records with equal (skeleton, nx, ny, iters);
 * per group: first global index, size, and the argmin (t, index) over valid
 * records with finite time (ties to the lowest index; best_index UINT64_MAX
 * and best_t_s +inf when none) with that candidate's bytes.  48 bytes. */
typedef struct {
    double best_t_s;
    uint64_t first, count, best_index, h2d_bytes, d2h_bytes;
} grophecy_group_result;

/* Groups of the batch into DEVICE array device_out (capacity entries, in
 * record order); *n_groups (HOST) receives the number of groups.  ELIMIT if
 * n_groups > capacity (the first `capacity` are written).  Synchronous. */
int grophecy_group_best(grophecy_space *space, const grophecy_pcie *pcie,
                        const grophecy_batch *batch, grophecy_group_result *device_out,
                        uint64_t capacity, uint64_t *n_groups, void *cuda_stream);

/* Cross-batch fix-up of a group split between two consecutive batches (e.g.
 * the last group of shard r and the first group of shard r + 1 when their
 * boundary records share (skeleton, nx, ny, iters)): out = the group of both
 * halves — first = a->first, count = a->count + b->count, the better
 * (t, index) of the two bests with its bytes.  `a` must precede `b`.  out may
 * alias a or b.  EINVAL on NULL or if a->first + a->count != b->first.  Pure
 * host function. */
int grophecy_group_merge_host(const grophecy_group_result *a, const grophecy_group_result *b,
                              grophecy_group_result *out);

/* Predicted speedup per group, S_g = t_cpu[g] / groups[g].best_t_s (P:L147:
 * "the total CPU time divided by the total GPU time"), in DEVICE memory:
 * groups (n entries), t_cpu (n doubles; the caller's CPU time of the group's
 * projection point), out (n doubles).  Groups without a feasible candidate
 * (best_t_s = +inf) give t_cpu / inf = 0.  Async, one launch. */
int grophecy_group_speedup(const grophecy_group_result *groups, const double *t_cpu, uint64_t n,
                           double *out, void *cuda_stream);

/* Break-even iteration count per candidate (the
 * iteration sweeps of P:L167, L215-239): with F = (t_once + t_h2d) + t_d2h
 * (one-time GPU cost) and c = the CPU time of one iteration, the GPU run with
 * `it` iterations, F + it * t_iter, beats the CPU run it * c iff
 * it * (c - t_iter) > F, so
 *     n_be      = F / (c - t_iter)        if c > t_iter, else +inf
 *     iters_min = 1 if n_be < 1, floor(n_be) + 1 if finite, else UINT64_MAX
 * (n_be in IEEE binary64 in that order; iters_min exact from n_be; NaN inputs
 * — invalid records — give NaN / UINT64_MAX; iters_min saturates at
 * UINT64_MAX for n_be >= 2^64).  Inputs: grophecy_eval_parts outputs (DEVICE,
 * n each) and either t_cpu_iter (DEVICE, n doubles) or, if it is NULL, the
 * scalar c for every candidate.  Outputs DEVICE n_be (may be NULL) and
 * iters_min (may be NULL).  Async, one launch. */
int grophecy_crossover(const double *t_iter, const double *t_once, const double *t_h2d,
                       const double *t_d2h, const double *t_cpu_iter, double t_cpu_iter_scalar,
                       uint64_t n, double *n_be, uint64_t *iters_min, void *cuda_stream);

/* GPU speedup = total CPU time / total GPU time. */
double grophecy_speedup(double t_cpu_s, double t_gpu_s);
/* Error magnitude |predicted - measured| / measured (Table II applies
 * it to predicted vs measured speedups).  Pure host functions. */
double grophecy_error_magnitude(double predicted, double measured);
/* Arithmetic mean of n values, summed in order (the paper's averages of
 * error magnitudes).  NaN for n = 0.  Pure host. */
double grophecy_mean(const double *values, uint64_t n);

/* End-to-end entry point: host_batch's record arrays are HOST memory
 * (pinned for full speed; index_base / stripes as in grophecy_batch).  The
 * records stream to the device in chunks, copies overlapped with the fused
 * projection + argmin, and the result returns in host memory.  Synchronous.
 * Same status rules as grophecy_best. */
int grophecy_best_host(grophecy_space *space, const grophecy_pcie *pcie,
                       const grophecy_batch *host_batch, grophecy_best_result *host_out,
                       void *cuda_stream);

/* ---------------------------------------------------------------------- */
/* PCIe calibration / validation subsystem      */
/* ---------------------------------------------------------------------- */

enum { GROPHECY_DIR_H2D = 0, GROPHECY_DIR_D2H = 1 };

/* Time `reps` pinned cudaMemcpyAsync transfers of `bytes` in one direction on
 * `device` (after `warmup` discarded ones).  Each transfer is issued and
 * waited for individually.  mean_wall_s: mean host steady-clock time per
 * transfer (what a program sees); mean_event_s: mean CUDA-event time (may be
 * NULL).  bytes <= 2^31. */
int grophecy_measure_transfer(int device, int direction, uint64_t bytes, int reps,
                              int warmup, double *mean_wall_s, double *mean_event_s);

/* The paper's automatic calibration: per direction, t_S = mean
 * of `reps` 1-byte transfers and t_L = mean of `reps` transfers of
 * large_bytes (paper: 512 MB = 2^29 B), then grophecy_fit_pcie. */
int grophecy_calibrate(int device, int reps, uint64_t large_bytes, grophecy_pcie *out);

/* ---------------------------------------------------------------------- */
/* Pinned vs pageable memory ("we may extend  */
/* our framework to automatically explore the tradeoff between the two types */
/* of memory", "account for the overhead of memory allocation";       */
/* DESIGN.md reading 17)                                                    */
/* ---------------------------------------------------------------------- */

enum { GROPHECY_MEM_PINNED = 0, GROPHECY_MEM_PAGEABLE = 1 };

/* grophecy_measure_transfer with the host buffer's memory type: PINNED
 * (cudaHostAlloc, as grophecy_measure_transfer) or PAGEABLE (malloc'd,
 * touched before timing).  Same protocol, outputs and limits. */
int grophecy_measure_transfer_mem(int device, int direction, int memory, uint64_t bytes,
                                  int reps, int warmup, double *mean_wall_s,
                                  double *mean_event_s);

/* Mean host steady-clock time of cudaHostAlloc(bytes) (mean_alloc_s) and of
 * the matching cudaFreeHost (mean_free_s, may be NULL) over `reps` pairs
 * after three discarded pairs; the buffer is not touched.  1 <= bytes <= 2^34. */
int grophecy_measure_pin_alloc(int device, uint64_t bytes, int reps, double *mean_alloc_s,
                               double *mean_free_s);

/* The memory model: Eq. (1) links per direction for pinned and for pageable
 * host memory, and the pinned allocation overhead in the same two-parameter
 * form, A(F) = alpha + beta * F for a pinned buffer of F bytes (allocation +
 * release; F = 0 -> 0). */
typedef struct {
    grophecy_pcie pinned, pageable;
    grophecy_link pin_alloc;
} grophecy_memory_model;

/* Automatic calibration of the whole model with the paper's protocol
 * (P:L113): per direction and memory type t_S (1 byte) and t_L (large_bytes),
 * each the mean of `reps` transfers; A from a one-page and a large_bytes
 * pinned allocation (alloc + free), alpha = t(4096), beta = t(large) / large. */
int grophecy_calibrate_memory(int device, int reps, uint64_t large_bytes,
                              grophecy_memory_model *out);

/* The per-array choice (reading 17): with h2d / d2h the array's transfer
 * bytes and footprint its full host buffer,
 *   pinned   = (A(footprint) if h2d + d2h > 0 else 0) + T_pin,h2d(h2d) + T_pin,d2h(d2h)
 *   pageable = T_page,h2d(h2d) + T_page,d2h(d2h)
 * (sums left to right, Eq. (1) with T(0) = 0); memory = PINNED iff
 * pinned <= pageable.  Pure host function.  EINVAL on NULL arguments or
 * footprint < max(h2d, d2h). */
typedef struct {
    double t_pinned_s, t_pageable_s;
    int32_t memory;
    int32_t reserved;
} grophecy_memory_choice;
int grophecy_choose_memory(const grophecy_memory_model *model, uint64_t h2d_bytes,
                           uint64_t d2h_bytes, uint64_t footprint_bytes,
                           grophecy_memory_choice *out);

/* The batched projection with the per-array memory choice (reading 17):
 * grophecy_eval_parts / grophecy_best where every array with a transfer is
 * priced pinned — t_h2d gets A(footprint) + T_pin,h2d, t_d2h gets T_pin,d2h —
 * or pageable — T_page,h2d / T_page,d2h — whichever grophecy_choose_memory
 * picks for it (footprint = planes * rows * cols * elem_bytes at the
 * candidate's size).  Bytes, kernel times and everything else as in
 * grophecy_eval / grophecy_best; same layouts, ownership and errors (parts
 * may be NULL).  Runs on the general projection path. */
int grophecy_eval_mem(const grophecy_space *space, const grophecy_memory_model *model,
                      const grophecy_batch *batch, uint64_t *h2d_bytes, uint64_t *d2h_bytes,
                      double *t_total_s, const grophecy_parts *parts, void *cuda_stream);
int grophecy_best_mem(grophecy_space *space, const grophecy_memory_model *model,
                      const grophecy_batch *batch, grophecy_best_result *host_out,
                      void *cuda_stream);

/* ---------------------------------------------------------------------- */
/* Synthetic workloads (bench / tests) — not part of the method             */
/* ---------------------------------------------------------------------- */

/* Per-skeleton size rule for the counter-based generator (synth/records.py
 * documents the closed form; this is an independent CUDA implementation). */
typedef struct { uint32_t kind, lo, hi, it_lo, it_hi, pad; } grophecy_synth_rule;
enum { GROPHECY_SYNTH_SQUARE = 0, GROPHECY_SYNTH_INDEP = 1, GROPHECY_SYNTH_ONED = 2,
       GROPHECY_SYNTH_FIXED = 3 };

/* Generate records [start, start + count) of an n_total-record workload into
 * DEVICE arrays.  rules is a HOST array of n_rules entries.  Async. */
int grophecy_synth_records(const grophecy_synth_rule *rules, uint32_t n_rules,
                           uint64_t n_total, uint32_t n_xforms, uint64_t seed, uint64_t start,
                           uint64_t count, uint32_t *skx, uint32_t *nx, uint32_t *ny,
                           uint32_t *iters, void *cuda_stream);

/* Diagnostic: evaluate on the HOST the usage plan that grophecy_space_create
 * compiles for `skel` (for sizes inside the plan's domain nx >= *plan_tx,
 * ny >= *plan_ty: the residue-class byte polynomials the kernel evaluates,
 * cross-checked against the band programs they are derived from).  Fills
 * per-array H2D / D2H bytes (arrays of skel->n_arrays).  Returns ELIMIT if
 * the skeleton has no plan or (nx, ny) is outside its domain (the kernel then
 * uses the general cell sweep), EINTERNAL if polynomial and program disagree.
 * Pure host function. */
int grophecy_plan_usage_host(const grophecy_skeleton_desc *skel, int64_t nx, int64_t ny,
                             uint64_t *h2d_per_array, uint64_t *d2h_per_array,
                             uint32_t *plan_tx, uint32_t *plan_ty);

/* Diagnostic: size of the usage plan compiled for `skel`: stats[0] =
 * expressions, [1] = program words, [2] = terms, [3] = terms, [4] = max terms
 * of one array program, [5] = max words of one program, [6] = coefficients
 * per byte polynomial (4 bilinear, 10 otherwise), [7] = distinct residue
 * classes among the 64 polynomial sets, [8] = polynomial table bytes.
 * `stats` holds 9 entries.
 * ELIMIT if the skeleton has no plan.  Pure host function. */
int grophecy_plan_stats(const grophecy_skeleton_desc *skel, uint32_t *stats);

/* Diagnostic: per-phase warp-cycle sums of the sweep kernel (8 entries:
 * waiting for staged records, phase A, barrier, phase B, barrier, phase C),
 * copied to HOST out8 and reset.  Only in builds with GROPHECY_PHASE_TIMING=1
 * (scripts/phase_timing.py); EINVAL otherwise. */
int grophecy_debug_phase_cycles(uint64_t *out8);

/* Number of CUDA kernel launches issued by this library since load (for
 * the bench's gpu_launches count). */
uint64_t grophecy_launch_count(void);

const char *grophecy_last_error(void);
int grophecy_abi_version(void);

#ifdef __cplusplus
}
#endif
#endif /* GROPHECY_H */
