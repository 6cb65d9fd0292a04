/*
 * GROPHECY++ CPU ORACLE — TEST INFRASTRUCTURE ONLY (see oracle.h).
 * Plain C11; build: gcc -O2 -std=c11 -ffp-contract=off -fno-fast-math -fPIC -shared -pthread
 * Every function cites the PAPER.md passage (P:Lnnn) or DESIGN.md reading it follows.
 */
#include "oracle.h"

#include <math.h>
#include <pthread.h>
#include <stdlib.h>
#include <string.h>

#define OR_INF_K 0x7fffffff   /* "no kernel" = +infinity for fr / fw */

/* min(a, b) = a < b ? a : b  (N1; never fmin) */
static double dmin(double a, double b) { return a < b ? a : b; }
static int64_t imin64(int64_t a, int64_t b) { return a < b ? a : b; }
static int64_t imax64(int64_t a, int64_t b) { return a > b ? a : b; }
static uint64_t umin64(uint64_t a, uint64_t b) { return a < b ? a : b; }

/* ------------------------------------------------------------------------ */
/* PCIe model — §III-C.  Eq. (1): T(d) = alpha + beta*d.           */
/* Fit: alpha = t_S (1-byte transfer), beta = t_L / s_L.            */
/* ------------------------------------------------------------------------ */
int oracle_fit_pcie(double t_small, double t_large, uint64_t large_bytes, or_link *out)
{
    if (!out || !isfinite(t_small) || !isfinite(t_large) || t_small < 0.0 ||
        t_large <= 0.0 || large_bytes == 0)
        return -1;
    out->alpha = t_small;
    out->beta = t_large / (double)large_bytes;
    return 0;
}

/* Eq. (1); a zero-byte "transfer" is no transfer (reading 9). */
double oracle_pcie_time(const or_link *l, uint64_t bytes)
{
    if (bytes == 0) return 0.0;
    return l->alpha + l->beta * (double)bytes;
}

/* Pinned vs pageable (NEXT-4, reading 17): the paper's future work
 * "explore the tradeoff between the two types of memory" and
 * "account for the overhead of memory allocation".  Written out:
 * both candidates priced with Eq. (1), the allocation of the whole host
 * buffer in the same linear form, the cheaper one chosen (pinned on ties). */
int oracle_choose_memory(const or_link *pin_h2d, const or_link *pin_d2h,
                         const or_link *page_h2d, const or_link *page_d2h,
                         const or_link *pin_alloc, uint64_t h2d, uint64_t d2h,
                         uint64_t footprint, double *t_pinned, double *t_pageable,
                         int *memory)
{
    if (footprint < h2d || footprint < d2h) return -1;
    double alloc = 0.0;
    if (h2d > 0 || d2h > 0) alloc = oracle_pcie_time(pin_alloc, footprint);
    double pinned = alloc;
    pinned = pinned + oracle_pcie_time(pin_h2d, h2d);
    pinned = pinned + oracle_pcie_time(pin_d2h, d2h);
    double pageable = oracle_pcie_time(page_h2d, h2d);
    pageable = pageable + oracle_pcie_time(page_d2h, d2h);
    *t_pinned = pinned;
    *t_pageable = pageable;
    *memory = pinned <= pageable ? 0 : 1;
    return 0;
}

/* Size-affine value (N2): c0 + floor((c1 nx + c2 ny + c3 nx ny) / 8). */
int64_t oracle_affine8(const or_affine8 *a, int64_t nx, int64_t ny)
{
    int64_t num = (int64_t)a->c1 * nx + (int64_t)a->c2 * ny + (int64_t)a->c3 * nx * ny;
    int64_t q = num / 8;
    if (num % 8 != 0 && num < 0) q -= 1;   /* floor, not truncation */
    return (int64_t)a->c0 + q;
}

/* ------------------------------------------------------------------------ */
/* Data usage — §III-B, N4.                            */
/* ------------------------------------------------------------------------ */

/* The BRS of one region instantiated at (nx, ny), clamped to the array. */
static void region_box(const or_region *g, int64_t R, int64_t C, int64_t nx, int64_t ny,
                       int64_t *r0, int64_t *r1, int64_t *c0, int64_t *c1)
{
    if (g->whole) {                     /* irregular: whole array */
        *r0 = 0; *r1 = R; *c0 = 0; *c1 = C;
        return;
    }
    *r0 = imin64(imax64(oracle_affine8(&g->r0, nx, ny), 0), R);
    *r1 = imin64(imax64(oracle_affine8(&g->r1, nx, ny), 0), R);
    *c0 = imin64(imax64(oracle_affine8(&g->c0, nx, ny), 0), C);
    *c1 = imin64(imax64(oracle_affine8(&g->c1, nx, ny), 0), C);
}

/* The region's plane range (rank-3 arrays, N4r), clamped to [0, P). */
static void region_pbox(const or_region *g, int64_t P, int64_t nx, int64_t ny, int64_t *p0,
                        int64_t *p1)
{
    if (g->whole) {
        *p0 = 0; *p1 = P;
        return;
    }
    *p0 = imin64(imax64(oracle_affine8(&g->p0, nx, ny), 0), P);
    *p1 = imin64(imax64(oracle_affine8(&g->p1, nx, ny), 0), P);
}

/* Strides of a region (whole regions are dense). */
static int64_t row_step(const or_region *g) { return (!g->whole && g->r_step > 1) ? g->r_step : 1; }
static int64_t col_step(const or_region *g) { return (!g->whole && g->c_step > 1) ? g->c_step : 1; }

/* Lattice anchors: the unclamped lower bounds (the section's l). */
static int64_t row_anchor(const or_region *g, int64_t nx, int64_t ny)
{
    return g->whole ? 0 : oracle_affine8(&g->r0, nx, ny);
}
static int64_t col_anchor(const or_region *g, int64_t nx, int64_t ny)
{
    return g->whole ? 0 : oracle_affine8(&g->c0, nx, ny);
}

/* x mod m in [0, m) */
static int64_t pmod(int64_t x, int64_t m) { return ((x % m) + m) % m; }

/* Effective access mode: an irregular ("may") write needs the original data
 * on the GPU and returns the whole array, i.e. it reads and writes every
 * element (reading 10). */
static uint32_t eff_mode(const or_region *g)
{
    return (g->whole && (g->mode & 2u)) ? (g->mode | 1u) : g->mode;
}

static int64_t gcd64(int64_t a, int64_t b)
{
    if (a < 0) a = -a;
    if (b < 0) b = -b;
    while (b) { int64_t t = a % b; a = b; b = t; }
    return a;
}

static int cmp_i64(const void *a, const void *b)
{
    int64_t x = *(const int64_t *)a, y = *(const int64_t *)b;
    return (x > y) - (x < y);
}

static int sort_unique(int64_t *v, int n)
{
    qsort(v, (size_t)n, sizeof(int64_t), cmp_i64);
    int m = 0;
    for (int i = 0; i < n; i++)
        if (m == 0 || v[i] != v[m - 1]) v[m++] = v[i];
    return m;
}

/* #{ r in [a, b) : r mod L == rho } */
static int64_t count_residue(int64_t a, int64_t b, int64_t rho, int64_t L)
{
    int64_t first = a + pmod(rho - a, L);
    return first < b ? (b - 1 - first) / L + 1 : 0;
}

/*
 * For every element e of array a:  fr(e) = first kernel reading e,
 * fw(e) = first kernel writing e (program order).
 *   H2D_a = elem_bytes * |{e : fr(e) < inf and fr(e) <= fw(e)}|
 *           ("read but not previously written"; a kernel's reads see the
 *            state before its own writes, reading 7)
 *   D2H_a = [live-out] * elem_bytes * |{e : fw(e) < inf}|
 *           ("union of all written BRSs", minus temporaries)
 * Cell method: the row/column breakpoints of all boxes cut the array into
 * slabs that every box either contains or misses; with strides, rows of a
 * slab are further split by their residue modulo L = lcm of the row strides
 * (a region with stride s covers row r of a slab it contains iff
 * (r - l) mod s == 0, which depends on r mod L only).  fr / fw are constant
 * per (row slab, row residue) x (column slab, column residue) cell.
 */
void oracle_usage(const or_skeleton *s, int64_t nx, int64_t ny,
                  uint64_t *h2d_per_array, uint64_t *d2h_per_array)
{
    if (s->hull) {
        oracle_usage_hull(s, nx, ny, h2d_per_array, d2h_per_array);
        return;
    }
    int nreg = (int)s->n_regions;
    int64_t *rb = (int64_t *)malloc(sizeof(int64_t) * (size_t)(2 * nreg + 2));
    int64_t *cb = (int64_t *)malloc(sizeof(int64_t) * (size_t)(2 * nreg + 2));
    int64_t *pb = (int64_t *)malloc(sizeof(int64_t) * (size_t)(2 * nreg + 2));
    int64_t *box = (int64_t *)malloc(sizeof(int64_t) * (size_t)(8 * nreg + 8));
    for (uint32_t a = 0; a < s->n_arrays; a++) {
        const or_array *A = &s->arrays[a];
        int64_t R = imax64(0, oracle_affine8(&A->rows, nx, ny));
        int64_t C = imax64(0, oracle_affine8(&A->cols, nx, ny));
        int64_t Pl = imax64(0, oracle_affine8(&A->planes, nx, ny));
        int nr = 0, nc = 0, np = 0;
        int64_t Lr = 1, Lc = 1;
        rb[nr++] = 0; rb[nr++] = R;
        cb[nc++] = 0; cb[nc++] = C;
        pb[np++] = 0; pb[np++] = Pl;
        for (int j = 0; j < nreg; j++) {
            const or_region *g = &s->regions[j];
            if (g->array != a) continue;
            int64_t *b = &box[8 * j];
            region_box(g, R, C, nx, ny, &b[0], &b[1], &b[2], &b[3]);
            b[4] = row_anchor(g, nx, ny);
            b[5] = col_anchor(g, nx, ny);
            region_pbox(g, Pl, nx, ny, &b[6], &b[7]);
            rb[nr++] = b[0]; rb[nr++] = b[1];
            cb[nc++] = b[2]; cb[nc++] = b[3];
            pb[np++] = b[6]; pb[np++] = b[7];
            Lr = Lr / gcd64(Lr, row_step(g)) * row_step(g);
            Lc = Lc / gcd64(Lc, col_step(g)) * col_step(g);
        }
        nr = sort_unique(rb, nr);
        nc = sort_unique(cb, nc);
        np = sort_unique(pb, np);
        uint64_t h = 0, d = 0;
        /* rank-3: the plane breakpoints cut the planes into slabs as well */
        for (int k = 0; k + 1 < np; k++) {
        int64_t z0 = pb[k], z1 = pb[k + 1];
        for (int i = 0; i + 1 < nr; i++)
            for (int64_t rho = 0; rho < Lr; rho++) {
                int64_t y0 = rb[i], y1 = rb[i + 1];
                int64_t hgt = count_residue(y0, y1, rho, Lr);
                if (hgt == 0) continue;
                for (int jj = 0; jj + 1 < nc; jj++)
                    for (int64_t sig = 0; sig < Lc; sig++) {
                        int64_t x0 = cb[jj], x1 = cb[jj + 1];
                        int64_t wid = count_residue(x0, x1, sig, Lc);
                        if (wid == 0) continue;
                        int fr = OR_INF_K, fw = OR_INF_K;
                        for (int j = 0; j < nreg; j++) {
                            const or_region *g = &s->regions[j];
                            if (g->array != a) continue;
                            const int64_t *b = &box[8 * j];
                            if (b[6] <= z0 && z1 <= b[7] &&
                                b[0] <= y0 && y1 <= b[1] && b[2] <= x0 && x1 <= b[3] &&
                                pmod(rho - b[4], row_step(g)) == 0 &&
                                pmod(sig - b[5], col_step(g)) == 0) {
                                uint32_t m = eff_mode(g);
                                if ((m & 1u) && (int)g->kernel < fr) fr = (int)g->kernel;
                                if ((m & 2u) && (int)g->kernel < fw) fw = (int)g->kernel;
                            }
                        }
                        uint64_t area = (uint64_t)(z1 - z0) * (uint64_t)hgt * (uint64_t)wid;
                        if (fr != OR_INF_K && fr <= fw) h += area;
                        if (fw != OR_INF_K) d += area;
                    }
            }
        }
        h2d_per_array[a] = h * A->elem_bytes;
        d2h_per_array[a] = A->liveout ? d * A->elem_bytes : 0;
    }
    free(rb); free(cb); free(pb); free(box);
}

/* The literal per-element definition (test-only; R*C <= 2^20 per array). */
int oracle_bitmap_usage(const or_skeleton *s, int64_t nx, int64_t ny,
                        uint64_t *h2d_per_array, uint64_t *d2h_per_array)
{
    for (uint32_t a = 0; a < s->n_arrays; a++) {
        const or_array *A = &s->arrays[a];
        int64_t R = imax64(0, oracle_affine8(&A->rows, nx, ny));
        int64_t C = imax64(0, oracle_affine8(&A->cols, nx, ny));
        int64_t Pl = imax64(0, oracle_affine8(&A->planes, nx, ny));
        if (R * C * Pl > (1 << 20)) return -1;
        uint64_t h = 0, d = 0;
        for (int64_t p = 0; p < Pl; p++)
        for (int64_t r = 0; r < R; r++) {
            for (int64_t c = 0; c < C; c++) {
                int fr = OR_INF_K, fw = OR_INF_K;
                for (uint32_t j = 0; j < s->n_regions; j++) {
                    const or_region *g = &s->regions[j];
                    if (g->array != a) continue;
                    int64_t r0, r1, c0, c1, p0, p1;
                    region_box(g, R, C, nx, ny, &r0, &r1, &c0, &c1);
                    region_pbox(g, Pl, nx, ny, &p0, &p1);
                    if (p0 <= p && p < p1 && r0 <= r && r < r1 && c0 <= c && c < c1 &&
                        pmod(r - row_anchor(g, nx, ny), row_step(g)) == 0 &&
                        pmod(c - col_anchor(g, nx, ny), col_step(g)) == 0) {
                        uint32_t m = eff_mode(g);
                        if ((m & 1u) && (int)g->kernel < fr) fr = (int)g->kernel;
                        if ((m & 2u) && (int)g->kernel < fw) fw = (int)g->kernel;
                    }
                }
                if (fr != OR_INF_K && fr <= fw) h += 1;
                if (fw != OR_INF_K) d += 1;
            }
        }
        h2d_per_array[a] = h * A->elem_bytes;
        d2h_per_array[a] = A->liveout ? d * A->elem_bytes : 0;
    }
    return 0;
}

/* ------------------------------------------------------------------------ */
/* Approximate mode: BRS lists with the Havlak-Kennedy UNION ([5]; */
/* SURVEY §8(f) NEXT-3; N4h).                                      */
/* ------------------------------------------------------------------------ */

/* One dimension of a section: {l, l+s, ..., u}; s == 0 iff l == u; empty iff l > u. */
typedef struct { int64_t l, u, s; } or_sec1;
/* A section (planes x rows x columns); empty iff any dimension is. */
typedef struct { or_sec1 r, c, p; } or_sec;

static int sec1_empty(or_sec1 a) { return a.l > a.u; }

/* The elements of the lattice anchor + i*step inside [lo, hi). */
static or_sec1 sec1_make(int64_t lo, int64_t hi, int64_t anchor, int64_t step)
{
    or_sec1 v = {1, 0, 0};
    int64_t first = lo + pmod(anchor - lo, step);
    if (first >= hi) return v;
    v.l = first;
    v.u = first + ((hi - 1 - first) / step) * step;
    v.s = v.l == v.u ? 0 : step;
    return v;
}

/* HK UNION: [min l : max u : gcd(s_a, s_b, |l_a - l_b|)] */
static or_sec1 sec1_union(or_sec1 a, or_sec1 b)
{
    if (sec1_empty(a)) return b;
    if (sec1_empty(b)) return a;
    or_sec1 v;
    v.l = imin64(a.l, b.l);
    v.u = imax64(a.u, b.u);
    v.s = gcd64(gcd64(a.s, b.s), a.l - b.l);
    if (v.l == v.u) v.s = 0;
    return v;
}

/* every element of x is an element of w */
static int sec1_contains(or_sec1 w, or_sec1 x)
{
    if (sec1_empty(x)) return 1;
    if (sec1_empty(w)) return 0;
    if (w.s == 0) return x.l == w.l && x.u == w.l;
    return x.l >= w.l && x.u <= w.u && pmod(x.l - w.l, w.s) == 0 && x.s % w.s == 0;
}

static uint64_t sec1_count(or_sec1 a)
{
    if (sec1_empty(a)) return 0;
    return a.s == 0 ? 1 : (uint64_t)((a.u - a.l) / a.s) + 1;
}

static int sec_empty(or_sec x) { return sec1_empty(x.r) || sec1_empty(x.c) || sec1_empty(x.p); }

static or_sec sec_union(or_sec a, or_sec b)
{
    if (sec_empty(a)) return b;
    if (sec_empty(b)) return a;
    or_sec v = {sec1_union(a.r, b.r), sec1_union(a.c, b.c), sec1_union(a.p, b.p)};
    return v;
}

static int sec_contains(or_sec w, or_sec x)
{
    if (sec_empty(x)) return 1;
    if (sec_empty(w)) return 0;
    return sec1_contains(w.r, x.r) && sec1_contains(w.c, x.c) && sec1_contains(w.p, x.p);
}

static uint64_t sec_count(or_sec a)
{
    return sec_empty(a) ? 0 : sec1_count(a.r) * sec1_count(a.c) * sec1_count(a.p);
}

static or_sec region_sec(const or_region *g, int64_t R, int64_t C, int64_t Pl, int64_t nx,
                         int64_t ny)
{
    int64_t r0, r1, c0, c1, p0, p1;
    region_box(g, R, C, nx, ny, &r0, &r1, &c0, &c1);
    region_pbox(g, Pl, nx, ny, &p0, &p1);
    or_sec v = {sec1_make(r0, r1, row_anchor(g, nx, ny), row_step(g)),
                sec1_make(c0, c1, col_anchor(g, nx, ny), col_step(g)),
                sec1_make(p0, p1, p0, 1)};
    return v;
}

/*
 * Per array, kernels in program order: "we maintain a list of
 * BRSs that are read but are not previously written" — a read section of
 * kernel k is dropped when ONE write section of a kernel < k contains it
 * (reads see the state before the kernel's own writes, reading 7);
 * "the UNION of all such BRSs is data that needs to be transferred to the
 * GPU.  The UNION of all written BRSs is data that needs to be transferred
 * back" — UNION = Havlak-Kennedy hull.  Bytes = elements of the hull.
 */
void oracle_usage_hull(const or_skeleton *s, int64_t nx, int64_t ny,
                       uint64_t *h2d_per_array, uint64_t *d2h_per_array)
{
    or_sec *wl = (or_sec *)malloc(sizeof(or_sec) * (size_t)(s->n_regions + 1));
    for (uint32_t a = 0; a < s->n_arrays; a++) {
        const or_array *A = &s->arrays[a];
        int64_t R = imax64(0, oracle_affine8(&A->rows, nx, ny));
        int64_t C = imax64(0, oracle_affine8(&A->cols, nx, ny));
        int64_t Pl = imax64(0, oracle_affine8(&A->planes, nx, ny));
        or_sec hr = {{1, 0, 0}, {1, 0, 0}, {1, 0, 0}}, hw = {{1, 0, 0}, {1, 0, 0}, {1, 0, 0}};
        int nw = 0;                                   /* writes of kernels < k */
        for (uint32_t k = 0; k < s->n_kernels; k++) {
            for (uint32_t j = 0; j < s->n_regions; j++) {   /* reads of kernel k */
                const or_region *g = &s->regions[j];
                if (g->array != a || g->kernel != k || !(eff_mode(g) & 1u)) continue;
                or_sec x = region_sec(g, R, C, Pl, nx, ny);
                if (sec_empty(x)) continue;
                int written = 0;
                for (int q = 0; q < nw; q++)
                    if (sec_contains(wl[q], x)) written = 1;
                if (!written) hr = sec_union(hr, x);
            }
            for (uint32_t j = 0; j < s->n_regions; j++) {   /* then its writes */
                const or_region *g = &s->regions[j];
                if (g->array != a || g->kernel != k || !(eff_mode(g) & 2u)) continue;
                or_sec x = region_sec(g, R, C, Pl, nx, ny);
                if (sec_empty(x)) continue;
                wl[nw++] = x;
                hw = sec_union(hw, x);
            }
        }
        h2d_per_array[a] = sec_count(hr) * A->elem_bytes;
        d2h_per_array[a] = A->liveout ? sec_count(hw) * A->elem_bytes : 0;
    }
    free(wl);
}

/* ------------------------------------------------------------------------ */
/* Kernel-time projection.  The paper defers to GROPHECY [15] (P:L13, L67,   */
/* L123) whose GPU model is Hong & Kim's MWP/CWP model [6].   */
/* The formula is absent from PAPER.md; DESIGN.md §3 N5 writes down the      */
/* reading implemented here, step by step, in H&K's notation.               */
/* regime: 0 = no work, 1/2/3 = H&K case, 4 = no memory insts, -1 = infeasible */
/* ------------------------------------------------------------------------ */
double oracle_kernel_time(const or_skeleton *s, const or_gpu *g, uint32_t xform,
                          uint32_t k, int64_t nx, int64_t ny, int *regime)
{
    const or_kx *c = &s->kx[(size_t)xform * s->n_kernels + k];
    int dummy;
    if (!regime) regime = &dummy;

    /* occupancy: active blocks per SM (no allocation granularity) */
    uint64_t occ;
    if (c->tpb > g->max_tpb) {
        occ = 0;
    } else {
        occ = umin64(g->max_bps, g->max_tps / c->tpb);
        if (c->regs > 0) occ = umin64(occ, g->regs_sm / ((uint64_t)c->regs * c->tpb));
        if (c->smem > 0) occ = umin64(occ, g->smem_sm / c->smem);
    }
    uint64_t wpb = c->tpb / g->warp_size + (c->tpb % g->warp_size != 0);
    uint64_t ipb = (uint64_t)c->tpb * c->ipt;
    double mem = c->coal + c->uncoal;                   /* #Mem_insts */
    double comp = g->issue * c->total;                  /* Comp_cycles */

    int64_t Wi = oracle_affine8(&s->kernels[k].work, nx, ny);
    uint64_t W = Wi > 0 ? (uint64_t)Wi : 0;             /* work items */
    if (occ == 0) { *regime = -1; return INFINITY; }
    uint64_t blocks = W / ipb + (W % ipb != 0);
    if (blocks == 0) { *regime = 0; return 0.0; }
    uint64_t asm_ = umin64(g->n_sm, blocks);            /* #Active_SMs */
    uint64_t abps = umin64(occ, blocks / asm_ + (blocks % asm_ != 0)); /* active blocks/SM */
    double N = (double)(abps * wpb);                    /* active warps per SM */
    double rep = (double)blocks / (double)(abps * asm_);/* #Rep */
    double cyc;
    if (mem == 0.0) {
        cyc = comp * N * rep;
        *regime = 4;
    } else {
        double mlu = g->mem_ld + (c->upm - 1.0) * g->dd_uncoal;   /* Mem_L_Uncoal */
        double mlc = g->mem_ld;                                   /* Mem_L_Coal */
        double wu = c->uncoal / mem;
        double wc = c->coal / mem;
        double ml = mlu * wu + mlc * wc;                          /* Mem_L */
        double dd = (g->dd_uncoal * c->upm) * wu + g->dd_coal * wc; /* Departure_delay */
        double mwp0 = ml / dd;                                    /* MWP_Without_BW */
        double bwpw = g->freq * c->lbpw / ml;                     /* BW_per_warp */
        double bwr = g->mem_bw / bwpw;
        double mpk = bwr / (double)asm_;                          /* MWP_peak_BW */
        double memc = mlu * c->uncoal + mlc * c->coal;            /* Mem_cycles */
        double cwpf = (memc + comp) / comp;                       /* CWP_full */
        double cpm = comp / mem;
        double mwp = dmin(dmin(mwp0, mpk), N);
        double cwp = dmin(cwpf, N);
        if (mwp == N && cwp == N) {
            cyc = (memc + comp + cpm * (mwp - 1.0)) * rep;
            *regime = 1;
        } else if (cwp >= mwp || comp > memc) {
            cyc = (memc * N / mwp + cpm * (mwp - 1.0)) * rep;
            *regime = 2;
        } else {
            cyc = (ml + comp * N) * rep;
            *regime = 3;
        }
        cyc = cyc + dd * (mwp - 1.0) * c->synch * (double)abps * rep;  /* Synch_cost */
    }
    return cyc / g->freq;
}

/* ------------------------------------------------------------------------ */
/* One candidate: total GPU time = kernels + transfers;        */
/* transfers happen once, per-iteration kernels repeat.            */
/* ------------------------------------------------------------------------ */
int oracle_eval_one(const or_skeleton *skels, uint32_t n_skels, const or_gpu *g,
                    const or_link *h2d_link, const or_link *d2h_link,
                    uint32_t skx, uint32_t nx, uint32_t ny, uint32_t iters,
                    uint64_t *h2d, uint64_t *d2h, double *t)
{
    uint32_t skel = skx >> 16, xform = skx & 0xffffu;
    if (skel >= n_skels || xform >= skels[skel].n_xforms || nx < 1 || nx > (1u << 20) ||
        ny < 1 || ny > (1u << 20) || iters < 1) {
        *h2d = 0; *d2h = 0; *t = NAN;
        return 0;
    }
    const or_skeleton *s = &skels[skel];
    uint64_t hpa[64], dpa[64];
    oracle_usage(s, nx, ny, hpa, dpa);

    double t_iter = 0.0, t_once = 0.0;
    for (uint32_t k = 0; k < s->n_kernels; k++) {
        double tk = oracle_kernel_time(s, g, xform, k, nx, ny, NULL);
        if (s->kernels[k].per_iter) t_iter = t_iter + tk;
        else t_once = t_once + tk;
    }
    double t_kern = t_once + (double)iters * t_iter;

    /* each array is transferred separately */
    double t_h = 0.0, t_d = 0.0;
    uint64_t H = 0, D = 0;
    for (uint32_t a = 0; a < s->n_arrays; a++) {
        if (hpa[a] > 0) t_h = t_h + oracle_pcie_time(h2d_link, hpa[a]);
        H += hpa[a];
    }
    for (uint32_t a = 0; a < s->n_arrays; a++) {
        if (dpa[a] > 0) t_d = t_d + oracle_pcie_time(d2h_link, dpa[a]);
        D += dpa[a];
    }
    *h2d = H;
    *d2h = D;
    *t = (t_kern + t_h) + t_d;
    return 1;
}

/* ------------------------------------------------------------------------ */
/* Algorithmic op tally of one candidate (DESIGN.md §6,     */
/* "op-bound roofline").  Counts the arithmetic the definition N4-N6 needs   */
/* per candidate under the stated amortisation rule:                         */
/*  R1  size-independent quantities are computed once per design space and   */
/*      charge nothing per candidate: N5 part A, the saturated-grid          */
/*      constants (E, S, D: on a saturated grid #Active_SMs = n_sm and        */
/*      active blocks/SM = occupancy, so MWP, CWP, the H&K case and the       */
/*      synch factor are fixed) and the times of the finitely many grids     */
/*      below saturation (blocks < sat: a per-(kernel, transformation)       */
/*      table);                                                               */
/*  R2  data usage depends only on (skeleton, nx, ny) (N4, reading 11): it is */
/*      charged once per design point of X transformations, 1/X per record:   */
/*      per kernel its work count (affine8: 3 mul + 2 add + 1 shift = 6 int), */
/*      per array and direction its byte count (a bilinear form: 6 int) and,  */
/*      when the bytes are non-zero, Eq. (1) priced and summed (1 int->fp64   */
/*      conversion, 1 mul, 2 add);                                           */
/*  R3  exact identities cost nothing: a product with an exact zero (S = 0),  */
/*      a division by a power of two (rep = blocks * 2^-k folds into E), and  */
/*      a kernel with zero occupancy (its sum is +inf);                       */
/*  R4  a candidate whose transformation has a zero-occupancy kernel has a    */
/*      non-finite total and takes no part in the argmin (N7): beyond its     */
/*      share of the design point's work (R2) it costs nothing.               */
/* Per (candidate, kernel) on a saturated grid: blocks = ceil(W / ipb) by a  */
/* multiply-high and a shift (2 int), 1 conversion, rep = blocks / D (a      */
/* division), cyc = E rep (+ S rep: mul + add), t = cyc / freq (a division),  */
/* the running sum (1 add); below saturation 2 int + the running sum.  Per   */
/* candidate: iters * t_iter (mul), + t_once (add, when the skeleton has     */
/* run-once kernels), + t_h2d, + t_d2h (2 add), the argmin compare (1).       */
/* fp64 counts each add / mul / compare as 1 and each division by a space    */
/* constant as 2 (its cheapest exact evaluation, x*zh + RN(x*zl): the        */
/* two-product form).  Returns 1 for a valid record (0: all counts 0).        */
static uint64_t occupancy_of(const or_gpu *g, const or_kx *c)
{
    if (c->tpb > g->max_tpb) return 0;
    uint64_t occ = umin64(g->max_bps, g->max_tps / c->tpb);
    if (c->regs > 0) occ = umin64(occ, g->regs_sm / ((uint64_t)c->regs * c->tpb));
    if (c->smem > 0) occ = umin64(occ, g->smem_sm / c->smem);
    return occ;
}

int oracle_op_tally_one(const or_skeleton *skels, uint32_t n_skels, const or_gpu *g,
                        uint32_t skx, uint32_t nx, uint32_t ny, uint32_t iters, uint32_t X,
                        double *fp64, double *ints, double *cvt)
{
    uint32_t skel = skx >> 16, xform = skx & 0xffffu;
    *fp64 = *ints = *cvt = 0.0;
    if (skel >= n_skels || xform >= skels[skel].n_xforms || nx < 1 || nx > (1u << 20) ||
        ny < 1 || ny > (1u << 20) || iters < 1 || X < 1)
        return 0;
    const or_skeleton *s = &skels[skel];
    double f = 0.0, in = 0.0, cv = 0.0;
    int has_once = 0, feasible = 1;
    for (uint32_t k = 0; k < s->n_kernels; k++) {
        const or_kx *c = &s->kx[(size_t)xform * s->n_kernels + k];
        if (occupancy_of(g, c) == 0) feasible = 0;
    }
    for (uint32_t k = 0; k < s->n_kernels; k++) {
        const or_kx *c = &s->kx[(size_t)xform * s->n_kernels + k];
        if (!s->kernels[k].per_iter) has_once = 1;
        in += 6.0 / X;                                   /* work count (R2) */
        if (!feasible) continue;                         /* R3, R4 */
        const uint64_t occ = occupancy_of(g, c);
        uint64_t ipb = (uint64_t)c->tpb * c->ipt;
        int64_t Wi = oracle_affine8(&s->kernels[k].work, nx, ny);
        uint64_t W = Wi > 0 ? (uint64_t)Wi : 0;
        uint64_t blocks = W / ipb + (W % ipb != 0);
        in += 2.0;                                       /* ceil division */
        f += 1.0;                                        /* running sum */
        uint64_t asm_ = umin64(g->n_sm, blocks ? blocks : 1);
        uint64_t abps = blocks ? umin64(occ, blocks / asm_ + (blocks % asm_ != 0)) : 0;
        if (!(asm_ == g->n_sm && abps == occ)) continue; /* below saturation: tabulated (R1) */
        cv += 1.0;
        uint64_t D = occ * g->n_sm;
        if (D & (D - 1)) f += 2.0;                       /* rep = blocks / D */
        f += 1.0;                                        /* E * rep */
        /* S = Departure_delay * (MWP - 1) * #synch * occupancy at saturation */
        double mem = c->coal + c->uncoal, S = 0.0;
        if (mem != 0.0) {
            double mlu = g->mem_ld + (c->upm - 1.0) * g->dd_uncoal, mlc = g->mem_ld;
            double wu = c->uncoal / mem, wc = c->coal / mem;
            double ml = mlu * wu + mlc * wc;
            double dd = (g->dd_uncoal * c->upm) * wu + g->dd_coal * wc;
            double bwr = g->mem_bw / (g->freq * c->lbpw / ml);
            double N = (double)(occ * (c->tpb / g->warp_size + (c->tpb % g->warp_size != 0)));
            double mwp = dmin(dmin(ml / dd, bwr / (double)g->n_sm), N);
            S = dd * (mwp - 1.0) * c->synch * (double)occ;
        }
        if (S != 0.0) f += 2.0;                          /* + S * rep */
        f += 2.0;                                        /* / freq */
    }
    /* usage of the design point (R2) */
    uint64_t hpa[64], dpa[64];
    oracle_usage(s, nx, ny, hpa, dpa);
    for (uint32_t a = 0; a < s->n_arrays; a++) {
        in += 12.0 / X;
        if (hpa[a]) { f += 3.0 / X; cv += 1.0 / X; }
        if (dpa[a]) { f += 3.0 / X; cv += 1.0 / X; }
    }
    if (feasible) f += 1.0 + (has_once ? 1.0 : 0.0) + 2.0 + 1.0;   /* totals + argmin */
    *fp64 = f;
    *ints = in;
    *cvt = cv;
    return 1;
}

/* Mean tally over a batch (single thread).  Returns the valid record count. */
uint64_t oracle_op_tally(const or_skeleton *skels, uint32_t n_skels, const or_gpu *g,
                         const uint32_t *skx, const uint32_t *nx, const uint32_t *ny,
                         const uint32_t *iters, uint64_t n, uint32_t X, double *mean3)
{
    double sf = 0.0, si = 0.0, sc = 0.0;
    uint64_t v = 0;
    for (uint64_t i = 0; i < n; i++) {
        double f, in, cv;
        if (oracle_op_tally_one(skels, n_skels, g, skx[i], nx[i], ny[i], iters[i], X, &f, &in, &cv)) {
            sf += f; si += in; sc += cv; v++;
        }
    }
    mean3[0] = v ? sf / (double)v : 0.0;
    mean3[1] = v ? si / (double)v : 0.0;
    mean3[2] = v ? sc / (double)v : 0.0;
    return v;
}

/* The projection with the per-array memory choice (NEXT-4, DESIGN.md
 * reading 17): every array with a transfer is priced as pinned (its
 * allocation A(footprint) + pinned transfers) or pageable, whichever
 * oracle_choose_memory picks; the pinned H2D term carries the allocation.
 * footprint = planes * rows * cols * elem_bytes (the whole host buffer). */
int oracle_eval_mem_one(const or_skeleton *skels, uint32_t n_skels, const or_gpu *g,
                        const or_link *pin_h2d, const or_link *pin_d2h,
                        const or_link *page_h2d, const or_link *page_d2h,
                        const or_link *pin_alloc,
                        uint32_t skx, uint32_t nx, uint32_t ny, uint32_t iters,
                        uint64_t *h2d, uint64_t *d2h, double *t, double *t_h2d, double *t_d2h)
{
    uint32_t skel = skx >> 16, xform = skx & 0xffffu;
    if (skel >= n_skels || xform >= skels[skel].n_xforms || nx < 1 || nx > (1u << 20) ||
        ny < 1 || ny > (1u << 20) || iters < 1) {
        *h2d = 0; *d2h = 0; *t = NAN; *t_h2d = NAN; *t_d2h = NAN;
        return 0;
    }
    const or_skeleton *s = &skels[skel];
    uint64_t hpa[64], dpa[64];
    oracle_usage(s, nx, ny, hpa, dpa);
    double t_iter = 0.0, t_once = 0.0;
    for (uint32_t k = 0; k < s->n_kernels; k++) {
        double tk = oracle_kernel_time(s, g, xform, k, nx, ny, NULL);
        if (s->kernels[k].per_iter) t_iter = t_iter + tk;
        else t_once = t_once + tk;
    }
    double t_kern = t_once + (double)iters * t_iter;
    double t_h = 0.0, t_d = 0.0;
    uint64_t H = 0, D = 0;
    for (uint32_t a = 0; a < s->n_arrays; a++) {
        const or_array *A = &s->arrays[a];
        H += hpa[a];
        D += dpa[a];
        if (hpa[a] == 0 && dpa[a] == 0) continue;
        uint64_t P = (uint64_t)imax64(0, oracle_affine8(&A->planes, nx, ny));
        uint64_t R = (uint64_t)imax64(0, oracle_affine8(&A->rows, nx, ny));
        uint64_t C = (uint64_t)imax64(0, oracle_affine8(&A->cols, nx, ny));
        uint64_t F = P * R * C * A->elem_bytes;
        double tp, tg;
        int m;
        oracle_choose_memory(pin_h2d, pin_d2h, page_h2d, page_d2h, pin_alloc, hpa[a], dpa[a], F,
                             &tp, &tg, &m);
        if (m == 0) {
            t_h = t_h + (oracle_pcie_time(pin_alloc, F) + oracle_pcie_time(pin_h2d, hpa[a]));
            t_d = t_d + oracle_pcie_time(pin_d2h, dpa[a]);
        } else {
            t_h = t_h + oracle_pcie_time(page_h2d, hpa[a]);
            t_d = t_d + oracle_pcie_time(page_d2h, dpa[a]);
        }
    }
    *h2d = H;
    *d2h = D;
    *t_h2d = t_h;
    *t_d2h = t_d;
    *t = (t_kern + t_h) + t_d;
    return 1;
}

/* The same computation, returning the four components. */
int oracle_eval_parts_one(const or_skeleton *skels, uint32_t n_skels, const or_gpu *g,
                          const or_link *h2d_link, const or_link *d2h_link,
                          uint32_t skx, uint32_t nx, uint32_t ny, uint32_t iters,
                          double *t_iter, double *t_once, double *t_h2d, double *t_d2h)
{
    uint32_t skel = skx >> 16, xform = skx & 0xffffu;
    if (skel >= n_skels || xform >= skels[skel].n_xforms || nx < 1 || nx > (1u << 20) ||
        ny < 1 || ny > (1u << 20) || iters < 1) {
        *t_iter = *t_once = *t_h2d = *t_d2h = NAN;
        return 0;
    }
    const or_skeleton *s = &skels[skel];
    uint64_t hpa[64], dpa[64];
    oracle_usage(s, nx, ny, hpa, dpa);
    double ti = 0.0, to = 0.0;
    for (uint32_t k = 0; k < s->n_kernels; k++) {
        double tk = oracle_kernel_time(s, g, xform, k, nx, ny, NULL);
        if (s->kernels[k].per_iter) ti = ti + tk;
        else to = to + tk;
    }
    double th = 0.0, td = 0.0;
    for (uint32_t a = 0; a < s->n_arrays; a++)
        if (hpa[a] > 0) th = th + oracle_pcie_time(h2d_link, hpa[a]);
    for (uint32_t a = 0; a < s->n_arrays; a++)
        if (dpa[a] > 0) td = td + oracle_pcie_time(d2h_link, dpa[a]);
    *t_iter = ti; *t_once = to; *t_h2d = th; *t_d2h = td;
    return 1;
}

/* Plain loop: runs of equal (skeleton, nx, ny, iters); per run the argmin of
 * (t, index) over valid records with finite t ("the predicted time of the
 * best-performing version"). */
uint64_t oracle_group_best(const or_skeleton *skels, uint32_t n_skels, const or_gpu *g,
                           const or_link *h2d_link, const or_link *d2h_link,
                           const uint32_t *skx, const uint32_t *nx, const uint32_t *ny,
                           const uint32_t *iters, uint64_t n, uint64_t index_base,
                           uint64_t capacity, uint64_t *first, uint64_t *count,
                           uint64_t *best_index, double *best_t)
{
    uint64_t ng = 0, i = 0;
    while (i < n) {
        uint64_t j = i;
        double bt = INFINITY;
        uint64_t bi = UINT64_MAX;
        while (j < n && (skx[j] >> 16) == (skx[i] >> 16) && nx[j] == nx[i] && ny[j] == ny[i] &&
               iters[j] == iters[i]) {
            uint64_t h, d; double t;
            if (oracle_eval_one(skels, n_skels, g, h2d_link, d2h_link, skx[j], nx[j], ny[j],
                                iters[j], &h, &d, &t) && isfinite(t)) {
                if (bi == UINT64_MAX || t < bt) { bt = t; bi = index_base + j; }
            }
            j++;
        }
        if (ng < capacity) {
            first[ng] = index_base + i; count[ng] = j - i;
            best_index[ng] = bi; best_t[ng] = bt;
        }
        ng++;
        i = j;
    }
    return ng;
}

/* ------------------------------------------------------------------------ */
/* Batch drivers: a static partition over host threads (plain loop inside). */
/* ------------------------------------------------------------------------ */
typedef struct {
    const or_skeleton *skels; uint32_t n_skels; const or_gpu *g;
    const or_link *hl, *dl;
    const uint32_t *skx, *nx, *ny, *iters;
    uint64_t lo, hi, index_base;
    uint64_t *h2d, *d2h; double *t;         /* eval mode (may be NULL) */
    or_best best;                           /* best mode partial */
} or_job;

static void *eval_worker(void *p)
{
    or_job *j = (or_job *)p;
    for (uint64_t i = j->lo; i < j->hi; i++)
        oracle_eval_one(j->skels, j->n_skels, j->g, j->hl, j->dl, j->skx[i], j->nx[i],
                        j->ny[i], j->iters[i], &j->h2d[i], &j->d2h[i], &j->t[i]);
    return NULL;
}

/* (t, index) lexicographic: is (ta, ia) < (tb, ib)?  (the best) */
static int better(double ta, uint64_t ia, double tb, uint64_t ib)
{
    return ta < tb || (ta == tb && ia < ib);
}

static void *best_worker(void *p)
{
    or_job *j = (or_job *)p;
    or_best b = {INFINITY, UINT64_MAX, 0, 0, 0, 0};
    for (uint64_t i = j->lo; i < j->hi; i++) {
        uint64_t h, d; double t;
        if (!oracle_eval_one(j->skels, j->n_skels, j->g, j->hl, j->dl, j->skx[i], j->nx[i],
                             j->ny[i], j->iters[i], &h, &d, &t)) {
            b.n_invalid++;
            continue;
        }
        b.n_valid++;
        if (!isfinite(t)) continue;
        uint64_t gi = j->index_base + i;
        if (b.index == UINT64_MAX || better(t, gi, b.t_total_s, b.index)) {
            b.t_total_s = t; b.index = gi; b.h2d_bytes = h; b.d2h_bytes = d;
        }
    }
    j->best = b;
    return NULL;
}

static void run_jobs(or_job *jobs, int nthreads, void *(*fn)(void *))
{
    if (nthreads <= 1) { fn(&jobs[0]); return; }
    pthread_t *th = (pthread_t *)malloc(sizeof(pthread_t) * (size_t)nthreads);
    for (int i = 0; i < nthreads; i++) pthread_create(&th[i], NULL, fn, &jobs[i]);
    for (int i = 0; i < nthreads; i++) pthread_join(th[i], NULL);
    free(th);
}

static or_job *make_jobs(int nthreads, uint64_t n, or_job proto)
{
    or_job *jobs = (or_job *)malloc(sizeof(or_job) * (size_t)nthreads);
    for (int i = 0; i < nthreads; i++) {
        jobs[i] = proto;
        jobs[i].lo = n * (uint64_t)i / (uint64_t)nthreads;
        jobs[i].hi = n * (uint64_t)(i + 1) / (uint64_t)nthreads;
    }
    return jobs;
}

void oracle_eval(const or_skeleton *skels, uint32_t n_skels, const or_gpu *g,
                 const or_link *h2d_link, const or_link *d2h_link,
                 const uint32_t *skx, const uint32_t *nx, const uint32_t *ny,
                 const uint32_t *iters, uint64_t n, int nthreads,
                 uint64_t *h2d, uint64_t *d2h, double *t)
{
    if (nthreads < 1) nthreads = 1;
    or_job proto;
    memset(&proto, 0, sizeof proto);
    proto.skels = skels; proto.n_skels = n_skels; proto.g = g;
    proto.hl = h2d_link; proto.dl = d2h_link;
    proto.skx = skx; proto.nx = nx; proto.ny = ny; proto.iters = iters;
    proto.h2d = h2d; proto.d2h = d2h; proto.t = t;
    or_job *jobs = make_jobs(nthreads, n, proto);
    run_jobs(jobs, nthreads, eval_worker);
    free(jobs);
}

int oracle_best(const or_skeleton *skels, uint32_t n_skels, const or_gpu *g,
                const or_link *h2d_link, const or_link *d2h_link,
                const uint32_t *skx, const uint32_t *nx, const uint32_t *ny,
                const uint32_t *iters, uint64_t n, uint64_t index_base,
                int nthreads, or_best *out)
{
    if (nthreads < 1) nthreads = 1;
    or_job proto;
    memset(&proto, 0, sizeof proto);
    proto.skels = skels; proto.n_skels = n_skels; proto.g = g;
    proto.hl = h2d_link; proto.dl = d2h_link;
    proto.skx = skx; proto.nx = nx; proto.ny = ny; proto.iters = iters;
    proto.index_base = index_base;
    or_job *jobs = make_jobs(nthreads, n, proto);
    run_jobs(jobs, nthreads, best_worker);
    or_best b = {INFINITY, UINT64_MAX, 0, 0, 0, 0};
    for (int i = 0; i < nthreads; i++) {
        or_best *p = &jobs[i].best;
        b.n_invalid += p->n_invalid;
        b.n_valid += p->n_valid;
        if (p->index != UINT64_MAX &&
            (b.index == UINT64_MAX || better(p->t_total_s, p->index, b.t_total_s, b.index))) {
            b.t_total_s = p->t_total_s; b.index = p->index;
            b.h2d_bytes = p->h2d_bytes; b.d2h_bytes = p->d2h_bytes;
        }
    }
    free(jobs);
    *out = b;
    return b.index == UINT64_MAX ? -1 : 0;
}

/* ------------------------------------------------------------------------ */
/* Validation helpers.                                                       */
/* ------------------------------------------------------------------------ */
/* "error magnitude ... absolute value of the percent difference between the
 * predicted and measured values" — returned as a fraction. */
double oracle_error_magnitude(double predicted, double measured)
{
    return fabs(predicted - measured) / measured;
}

/* arithmetic mean */
double oracle_mean(const double *v, uint64_t n)
{
    double s = 0.0;
    for (uint64_t i = 0; i < n; i++) s = s + v[i];
    return s / (double)n;
}

/* "The GPU speedup is the total CPU time divided by the total GPU time" */
double oracle_speedup(double t_cpu, double t_gpu) { return t_cpu / t_gpu; }

/* Error magnitude of a predicted speedup (Table II). */
double oracle_speedup_error(double s_pred, double s_meas)
{
    return oracle_error_magnitude(s_pred, s_meas);
}

/* Break-even iteration count (oracle.h; N9), written as the
 * definition. */
void oracle_crossover(double t_iter, double t_once, double t_h2d, double t_d2h, double c,
                      double *n_be, uint64_t *iters_min)
{
    double F = (t_once + t_h2d) + t_d2h;
    double den = c - t_iter;
    double v;
    if (isnan(F) || isnan(den)) v = NAN;
    else if (den > 0.0) v = F / den;
    else v = INFINITY;
    *n_be = v;
    if (isnan(v) || v >= 18446744073709551616.0) {   /* also +inf */
        *iters_min = UINT64_MAX;
        return;
    }
    /* smallest integer it >= 1 with it > v: 1 if v < 1, else floor(v) + 1 */
    *iters_min = v < 1.0 ? 1 : (uint64_t)floor(v) + 1;
}
