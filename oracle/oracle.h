/*
 * GROPHECY++ CPU ORACLE — TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, obviously-correct CPU implementation of the projection the
 * CUDA path computes.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load it.  It shares no code,
 * header or table with paper_conf_ipps_boyermk13_b200/ (the product), and
 * the product never loads it.
 *
 * Source of truth: /root/reference/PAPER.md ("P:Lnnn" = line nnn) and the
 * readings recorded in DESIGN.md §3.
 *
 * Arithmetic (N1): byte counts are exact 64-bit integers; times are IEEE-754
 * binary64 evaluated in exactly the written order (compiled with
 * -ffp-contract=off, no fast-math).
 *
 * Parity status per function:
 *   oracle_fit_pcie / oracle_pcie_time ... pinned (Eq. 1 closed form)
 *   oracle_usage ......................... pinned (bitmap brute force, Table I sizes,
 *                                           invariants)
 *   oracle_bitmap_usage .................. pinned (hand-counted tiny cases)
 *   oracle_kernel_time ................... pinned only to hand-derived closed forms
 *                                           of OUR reading (H&K MWP/CWP): the paper
 *                                           prints no kernel-model formula
 *                                           ("parity unpinned" by the paper itself)
 *   oracle_eval_one / oracle_best ........ pinned (composition identities, brute-force min)
 *   validation helpers ................... pinned (Table II arithmetic)
 *   oracle_op_tally[_one] ................ pinned to hand counts of its own stated
 *                                           rule: a measurement
 *                                           convention, not a paper quantity
 *   oracle_choose_memory ................. pinned to closed forms of OUR reading 17
 *                                           (pinned vs pageable + allocation, NEXT-4);
 *                                           the paper only names the tradeoff (P:L93,
 *                                           L296): "parity unpinned" by the paper
 */
#ifndef GROPHECY_ORACLE_H
#define GROPHECY_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct { int32_t c0, c1, c2, c3; } or_affine8;   /* c0 + floor((c1 nx + c2 ny + c3 nx ny)/8) */

/* planes: extent of a leading third dimension (rank-3 arrays, SURVEY §8(f)
 * NEXT-3; N4r); 1 for the 2-D arrays of the paper's workloads. */
typedef struct { or_affine8 rows, cols; uint32_t elem_bytes, liveout; or_affine8 planes; } or_array;
/* mode: bit0 = read, bit1 = write.  whole != 0: irregular access, the whole
 * array may be referenced; an irregular write is a "may-write" and
 * counts as read + write of the whole array (reading 10).
 * r_step / c_step: the strides of the bounded regular section [l:u:s]
 * ([5]); 0 or 1 = dense.  A strided region covers rows r0 + i*r_step
 * inside the clamped box (the lattice is anchored at the unclamped r0). */
typedef struct {
    uint32_t kernel, array, mode, whole;
    or_affine8 r0, r1, c0, c1;
    uint32_t r_step, c_step;
    or_affine8 p0, p1;             /* planes [p0, p1) (dense); whole: all planes */
} or_region;
typedef struct { or_affine8 work; uint32_t per_iter; } or_kernel;
typedef struct {
    uint32_t tpb, ipt, regs, smem;
    double total, coal, uncoal, upm, lbpw, synch;
} or_kx;
typedef struct {
    uint32_t n_kernels, n_arrays, n_regions, n_xforms;
    const or_kernel *kernels;
    const or_array *arrays;
    const or_region *regions;
    const or_kx *kx;               /* [n_xforms][n_kernels] */
    uint32_t hull;                 /* 1: Havlak-Kennedy approximate UNION (N4h) */
} or_skeleton;
typedef struct {
    uint32_t n_sm, warp_size, max_tpb, max_bps, max_tps, regs_sm, smem_sm;
    double freq, mem_bw, mem_ld, dd_coal, dd_uncoal, issue;
} or_gpu;
typedef struct { double alpha, beta; } or_link;

/* §III-C, Eq. (1) and P:L113 */
int     oracle_fit_pcie(double t_small, double t_large, uint64_t large_bytes, or_link *out);
double  oracle_pcie_time(const or_link *l, uint64_t bytes);

/* NEXT-4 (reading 17): per-array pinned vs pageable
 * choice.  pinned = (A(footprint) if any transfer else 0) + T_pin,h2d(h) +
 * T_pin,d2h(d); pageable = T_page,h2d(h) + T_page,d2h(d); *memory = 0 (pinned)
 * iff pinned <= pageable.  Returns -1 if footprint < max(h, d). */
int oracle_choose_memory(const or_link *pin_h2d, const or_link *pin_d2h,
                         const or_link *page_h2d, const or_link *page_d2h,
                         const or_link *pin_alloc, uint64_t h2d, uint64_t d2h,
                         uint64_t footprint, double *t_pinned, double *t_pageable,
                         int *memory);

int64_t oracle_affine8(const or_affine8 *a, int64_t nx, int64_t ny);

/* §III-B: per-array H2D / D2H bytes, cell method and literal bitmap. */
void oracle_usage(const or_skeleton *s, int64_t nx, int64_t ny,
                  uint64_t *h2d_per_array, uint64_t *d2h_per_array);
int  oracle_bitmap_usage(const or_skeleton *s, int64_t nx, int64_t ny,
                         uint64_t *h2d_per_array, uint64_t *d2h_per_array);
/* The approximate mode: BRS lists merged with the
 * Havlak-Kennedy UNION (per dimension [min l : max u : gcd]); a read is
 * "previously written" when one earlier write section contains it.
 * oracle_usage dispatches here when s->hull != 0. */
void oracle_usage_hull(const or_skeleton *s, int64_t nx, int64_t ny,
                       uint64_t *h2d_per_array, uint64_t *d2h_per_array);

/* Kernel-time projection (GROPHECY [15] / Hong & Kim [6] reading). */
double oracle_kernel_time(const or_skeleton *s, const or_gpu *g, uint32_t xform,
                          uint32_t k, int64_t nx, int64_t ny, int *regime);

/* Components of one candidate's time:
 * t = ((t_once + iters * t_iter) + t_h2d) + t_d2h.  Returns 1 if valid
 * (else all components NaN). */
/* NEXT-4: one candidate with the per-array pinned / pageable choice
 * (reading 17); also returns the two transfer components. */
int oracle_eval_mem_one(const or_skeleton *skels, uint32_t n_skels, const or_gpu *g,
                        const or_link *pin_h2d, const or_link *pin_d2h,
                        const or_link *page_h2d, const or_link *page_d2h,
                        const or_link *pin_alloc,
                        uint32_t skx, uint32_t nx, uint32_t ny, uint32_t iters,
                        uint64_t *h2d, uint64_t *d2h, double *t, double *t_h2d, double *t_d2h);

int oracle_eval_parts_one(const or_skeleton *skels, uint32_t n_skels, const or_gpu *g,
                          const or_link *h2d_link, const or_link *d2h_link,
                          uint32_t skx, uint32_t nx, uint32_t ny, uint32_t iters,
                          double *t_iter, double *t_once, double *t_h2d, double *t_d2h);

/* Best transformation per group: groups are maximal runs of
 * consecutive records with equal (skeleton, nx, ny, iters); per group the
 * first index, the size, and the argmin (t, index) over valid records with
 * finite t (best_index UINT64_MAX, best_t +inf when none).  Returns the number
 * of groups (results beyond `capacity` are not written). */
uint64_t oracle_group_best(const or_skeleton *skels, uint32_t n_skels, const or_gpu *g,
                           const or_link *h2d_link, const or_link *d2h_link,
                           const uint32_t *skx, const uint32_t *nx, const uint32_t *ny,
                           const uint32_t *iters, uint64_t n, uint64_t index_base,
                           uint64_t capacity, uint64_t *first, uint64_t *count,
                           uint64_t *best_index, double *best_t);

/* One candidate.  Returns 1 if the record is valid. */
int oracle_eval_one(const or_skeleton *skels, uint32_t n_skels, const or_gpu *g,
                    const or_link *h2d_link, const or_link *d2h_link,
                    uint32_t skx, uint32_t nx, uint32_t ny, uint32_t iters,
                    uint64_t *h2d, uint64_t *d2h, double *t);

void oracle_eval(const or_skeleton *skels, uint32_t n_skels, const or_gpu *g,
                 const or_link *h2d_link, const or_link *d2h_link,
                 const uint32_t *skx, const uint32_t *nx, const uint32_t *ny,
                 const uint32_t *iters, uint64_t n, int nthreads,
                 uint64_t *h2d, uint64_t *d2h, double *t);

typedef struct {
    double t_total_s;
    uint64_t index, h2d_bytes, d2h_bytes, n_invalid, n_valid;
} or_best;

/* argmin over valid, finite records of (t, index_base + i).
 * Returns 0 if a best exists, -1 if none (index = UINT64_MAX). */
int oracle_best(const or_skeleton *skels, uint32_t n_skels, const or_gpu *g,
                const or_link *h2d_link, const or_link *d2h_link,
                const uint32_t *skx, const uint32_t *nx, const uint32_t *ny,
                const uint32_t *iters, uint64_t n, uint64_t index_base,
                int nthreads, or_best *out);

/* Algorithmic op tally of one candidate under the amortisation rule of
 * DESIGN.md §6 (oracle.c states it in full): fp64 operations (a division by a
 * space constant counts 2), integer operations and int->fp64 conversions per
 * record, usage charged once per design point of X records.  Returns 1 if the
 * record is valid.  oracle_op_tally: means over a batch (mean3 = {fp64, int,
 * cvt}), returns the number of valid records. */
int oracle_op_tally_one(const or_skeleton *skels, uint32_t n_skels, const or_gpu *g,
                        uint32_t skx, uint32_t nx, uint32_t ny, uint32_t iters, uint32_t X,
                        double *fp64, double *ints, double *cvt);
uint64_t oracle_op_tally(const or_skeleton *skels, uint32_t n_skels, const or_gpu *g,
                         const uint32_t *skx, const uint32_t *nx, const uint32_t *ny,
                         const uint32_t *iters, uint64_t n, uint32_t X, double *mean3);

/* Validation helpers (Table II). */
double oracle_error_magnitude(double predicted, double measured);
double oracle_mean(const double *v, uint64_t n);
double oracle_speedup(double t_cpu, double t_gpu);
double oracle_speedup_error(double s_pred, double s_meas);

/* Break-even iteration count (NEXT-2; "transfers once, kernels every
 * iteration"; reading N9): the GPU run with `it` iterations costs
 * F + it*t_iter with F = (t_once + t_h2d) + t_d2h, the CPU run it*c; the GPU
 * wins iff it*(c - t_iter) > F.  *n_be = F/(c - t_iter) (c > t_iter) else
 * +inf; *iters_min = smallest integer it >= 1 with it > *n_be (UINT64_MAX if
 * none representable); NaN inputs give NaN / UINT64_MAX. */
void oracle_crossover(double t_iter, double t_once, double t_h2d, double t_d2h, double c,
                      double *n_be, uint64_t *iters_min);

#ifdef __cplusplus
}
#endif
#endif
