// The projection hot path for sm_100a: grophecy_eval[_parts|_mem] /
// grophecy_best[_async|_mem|_host] / grophecy_best_combine.
//
// Best mode: one cooperative launch of sweep_kernel.  CTA sweep tiles of
// 4096 records = 256 design points x 16 transformations of one skeleton are
// staged in shared memory by TMA bulk copies one tile ahead; per warp (lane =
// design point) phase A checks the canonical layout, phase B computes the
// kernels' work counts and the data usage from the skeleton's residue-class
// byte polynomials (plan.cpp; usage depends only on (skeleton, nx, ny),
// DESIGN.md reading 11) staged in shared memory; then CTA-wide phase C: a
// warp takes a transformation and its lanes run its program (the feasible
// kernels in summation order, each with its class of the saturated model) on
// 8 design points each, so every (kernel, transformation) record and code
// path is warp-uniform.  Tiles that are not canonical (any other layout,
// mixed skeletons, keys off the polynomial domain, strided / hull / rank-3
// skeletons, huge work counts) are listed and, after a grid barrier, drained
// by the same CTAs with general_tile: 128-record warp tiles, runs of equal
// keys, usage per distinct key (plans, else the warp-cooperative
// coordinate-compressed sweep or the HK hull), the model per record.  Eval
// mode: canon_kernel (warp tiles, lane = (transformation, half), coalesced
// stores) then general_kernel over the list.  The kernel-time model runs from
// per-(kernel, transformation) constants the host precomputed in the
// definition's operation order; on saturated grids the two remaining IEEE
// divisions use the two-product method (x * zh + RN(x * zl), exact for the
// divisors used: space.cpp div2_ok), small grids come from a table computed
// step by step at space creation.  Best mode fuses the argmin (lane -> warp
// -> CTA -> grid, last-block pattern).
//
// Compiled with -fmad=false: no contraction anywhere; FMAs appear only as the
// explicit __fma_rn of the divisions.
#include <cooperative_groups.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <type_traits>
#include <cmath>

#include "grophecy.h"
#include "internal.h"

namespace grophecy {

constexpr unsigned FULL = 0xffffffffu;
#ifndef GROPHECY_THREADS
#define GROPHECY_THREADS 256
#endif
constexpr int THREADS = GROPHECY_THREADS;
constexpr int WARPS = THREADS / 32;
constexpr int RPT = 4;                       // records per lane
constexpr int WTILE = 32 * RPT;              // records per warp tile
constexpr int SLOT_CAP = 16;                 // distinct keys resident per warp chunk
constexpr int MAXK = GROPHECY_MAX_KERNELS;   // kernels per skeleton
constexpr long long BIG = 0x7fffffffffffffffLL;
#ifndef GROPHECY_MINB
#define GROPHECY_MINB 2
#endif

// c0 + floor((c1 nx + c2 ny + c3 nx ny) / 8); nx, ny <= 2^20 (so the 32x32->64
// products are exact), nxny = nx * ny precomputed.
__device__ __forceinline__ long long aff8n(int4 c, int nx, int ny, long long nxny)
{
    const long long num = (long long)c.y * nx + (long long)c.z * ny + (long long)c.w * nxny;
    return (long long)c.x + (num >> 3);   // arithmetic shift: floor(num / 8)
}

__device__ __forceinline__ long long aff8(int4 c, long long nx, long long ny)
{
    return aff8n(c, (int)nx, (int)ny, nx * ny);
}

__device__ __forceinline__ long long clampll(long long v, long long hi)
{
    return v < 0 ? 0 : (v > hi ? hi : v);
}

__device__ __forceinline__ double dmin(double a, double b) { return a < b ? a : b; }

// Correctly rounded a / b given rb = RN(1/b) (Markstein).
__device__ __forceinline__ double div_rn(double a, double b, double rb)
{
    double q = __dmul_rn(a, rb);
    double r = __fma_rn(-q, b, a);
    return __fma_rn(r, rb, q);
}

struct SweepScratch {
    long long box[32][4];
    long long rs_h[64];
    long long cs_w[64];
    long long rs_a[64];         // slab starts (strided arrays)
    long long cs_a[64];
    unsigned rs_m[64];
    unsigned cs_m[64];
    unsigned pr_m[64];          // strided arrays: regions whose row lattice hits residue rho
    unsigned pc_m[64];
    unsigned upto[32];
    // strided arrays: (slab, residue) units aggregated by coverage mask,
    // [0] rows / [1] columns (open addressing, key 0 = empty)
    unsigned agg_key[2][64];
    unsigned long long agg_sum[2][64];
    unsigned agg_over;
};

constexpr int MAX_SEG = 8;                   // keys per warp pass (plan path)

struct PlanScratch {
    alignas(16) double T[MAX_SEG][2 * GROPHECY_MAX_ARRAYS + 2];  // per-array transfer times of the pass's keys
};

union WarpScratch {
    SweepScratch sw;                    // general cell sweep (one key per warp)
    PlanScratch pl;                     // usage plans: up to MAX_SEG keys per pass
};

struct Usage {
    unsigned long long h, d;
    double th, td;
};

__device__ __forceinline__ unsigned long long warp_sum_u64(unsigned long long v)
{
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(FULL, v, o);
    return v;
}

// How transfers are priced: the pinned links of `pc` (the paper's model), or
// with mem set the per-array pinned / pageable choice of DESIGN.md reading 17
// (NEXT-4, grophecy_choose_memory's rule; general path only).
struct Price {
    grophecy_pcie pc;
    grophecy_memory_model mm;
    int mem;
};

__device__ __forceinline__ double link_time(const grophecy_link &l, unsigned long long b)
{
    return b ? __dadd_rn(l.alpha_s, __dmul_rn(l.beta_s_per_byte, __ull2double_rn(b))) : 0.0;
}

// Reading 17 for one array with transfer bytes (h, d) and host footprint F:
// the H2D / D2H terms it adds (the pinned H2D term carries the allocation).
__device__ __forceinline__ void mem_terms(const grophecy_memory_model &m, unsigned long long h,
                                          unsigned long long d, unsigned long long F, double &th,
                                          double &td)
{
    th = td = 0.0;
    if (!h && !d) return;
    const double a = link_time(m.pin_alloc, F);
    const double ph = __dadd_rn(a, link_time(m.pinned.h2d, h)), pd = link_time(m.pinned.d2h, d);
    const double gh = link_time(m.pageable.h2d, h), gd = link_time(m.pageable.d2h, d);
    if (__dadd_rn(ph, pd) <= __dadd_rn(gh, gd)) {
        th = ph;
        td = pd;
    } else {
        th = gh;
        td = gd;
    }
}

// Host footprint of an array at (nx, ny): planes * rows * cols * elem_bytes.
__device__ __forceinline__ unsigned long long footprint(const ArrayDev &A, long long nx, long long ny)
{
    long long R = aff8(A.rows, nx, ny), C = aff8(A.cols, nx, ny);
    long long Pl = A.rank3 ? aff8(A.planes, nx, ny) : 1;
    R = R > 0 ? R : 0;
    C = C > 0 ? C : 0;
    Pl = Pl > 0 ? Pl : 0;
    return (unsigned long long)Pl * (unsigned long long)R * (unsigned long long)C *
           (unsigned long long)A.elem_bytes;
}

// Per-array byte counts -> totals and per-array PCIe times in array order
// (Eq. (1), one transfer per array).  Warp-uniform.
__device__ __forceinline__ void add_array(Usage &o, const ArrayDev &A, unsigned long long h,
                                          unsigned long long d, const Price &pr, long long nx,
                                          long long ny)
{
    const unsigned long long ha = h * (unsigned long long)A.elem_bytes;
    const unsigned long long da = A.liveout ? d * (unsigned long long)A.elem_bytes : 0ull;
    if (pr.mem) {
        double th, td;
        mem_terms(pr.mm, ha, da, footprint(A, nx, ny), th, td);
        o.th = __dadd_rn(o.th, th);
        o.td = __dadd_rn(o.td, td);
    } else {
        const grophecy_pcie &pc = pr.pc;
        if (ha) o.th = __dadd_rn(o.th, __dadd_rn(pc.h2d.alpha_s,
                                                 __dmul_rn(pc.h2d.beta_s_per_byte, (double)ha)));
        if (da) o.td = __dadd_rn(o.td, __dadd_rn(pc.d2h.alpha_s,
                                                 __dmul_rn(pc.d2h.beta_s_per_byte, (double)da)));
    }
    o.h += ha;
    o.d += da;
}

// Work-item count as stored for the model's fast path: W if 0 < W < 2^30,
// 0 if W <= 0 (blocks = 0: the small-grid table gives t = 0), W_HUGE above
// (the general path recomputes W from the key).
constexpr uint32_t W_HUGE = 0xffffffffu;
__device__ __forceinline__ uint32_t w_store(long long w)
{
    return w <= 0 ? 0u : (w < 0x40000000LL ? (uint32_t)w : W_HUGE);
}

// One residue-class byte polynomial P(a, b) (plan.cpp; internal.h layout),
// wrapping 64-bit arithmetic; a, b < 2^18.
template <bool BIQ>
__device__ __forceinline__ unsigned long long poly_eval(const unsigned long long *c, uint32_t a,
                                                        uint32_t b)
{
    const ulonglong2 c01 = __ldg(reinterpret_cast<const ulonglong2 *>(c));
    const ulonglong2 c23 = __ldg(reinterpret_cast<const ulonglong2 *>(c) + 1);
    unsigned long long v = c01.x + c01.y * a + (c23.x + c23.y * a) * b;
    if (BIQ) {
        const ulonglong2 c45 = __ldg(reinterpret_cast<const ulonglong2 *>(c) + 2);
        const ulonglong2 c67 = __ldg(reinterpret_cast<const ulonglong2 *>(c) + 3);
        const unsigned long long c8 = __ldg(c + 8);
        v += (unsigned long long)a * (a * (c45.x + b * (c67.x + b * c8))) +
             (unsigned long long)b * (b * (c45.y + a * c67.y));
    }
    return v;
}

// Usage of one key from its skeleton's residue-class byte polynomials
// (plan.cpp), by a segment of L lanes (32/L keys per warp pass).  Lane sl
// evaluates the H2D and D2H polynomials of arrays sl, sl+L, ... (bytes, with
// elem_bytes and live-out folded in) and prices each transfer with Eq. (1)
// into T[2a + dir]; byte totals are an integer tree sum over the segment, and
// the segment's lane 0 adds the transfer times in array order (N6).  The
// kernels' work-item counts go to w_out.  Results: *res (segment lane 0).
__device__ __forceinline__ void plan_usage(const SpaceDev &S, bool active, unsigned long long key,
                                           const Price &pr, double *T, int sl, int L,
                                           Usage *res, uint32_t *w_out)
{
    const grophecy_pcie &pc = pr.pc;
    uint32_t n_arrays = 0, K = 0, kb = 0, stride = 4, a_base = 0;
    uint32_t nx = 0, ny = 0;
    const unsigned long long *P = S.poly;
    if (active) {
        const SkelInfo &I = S.skel[(uint32_t)(key >> 42)];
        n_arrays = I.n_arrays;
        a_base = I.a_base;
        K = I.n_kernels;
        kb = I.k_base;
        stride = I.poly_stride;
        nx = (uint32_t)((key >> 21) & 0x1fffffull);
        ny = (uint32_t)(key & 0x1fffffull);
        P += I.poly_base + (size_t)((nx & 7u) * 8u + (ny & 7u)) * (2u * n_arrays * stride);
    }
    const uint32_t a8 = nx >> 3, b8 = ny >> 3;
    unsigned long long hs = 0, ds = 0;
    for (uint32_t a = sl; a < n_arrays; a += L) {
#pragma unroll
        for (int dir = 0; dir < 2; dir++) {
            const unsigned long long *c = P + (2 * a + dir) * stride;
            const unsigned long long bytes = stride > 4 ? poly_eval<true>(c, a8, b8)
                                                        : poly_eval<false>(c, a8, b8);
            const grophecy_link lk = dir ? pc.d2h : pc.h2d;
            T[2 * a + dir] = bytes ? __dadd_rn(lk.alpha_s, __dmul_rn(lk.beta_s_per_byte,
                                                                    __ull2double_rn(bytes)))
                                   : 0.0;
            if (dir) ds += bytes; else hs += bytes;
        }
        if (pr.mem) {   // reading 17: this array's pinned / pageable terms
            const unsigned long long *c = P + (2 * a) * stride;
            const unsigned long long bh = stride > 4 ? poly_eval<true>(c, a8, b8) : poly_eval<false>(c, a8, b8);
            const unsigned long long bd = stride > 4 ? poly_eval<true>(c + stride, a8, b8)
                                                     : poly_eval<false>(c + stride, a8, b8);
            mem_terms(pr.mm, bh, bd, footprint(S.arrays[a_base + a], nx, ny), T[2 * a], T[2 * a + 1]);
        }
    }
    {
        const long long nxny = (long long)((unsigned long long)nx * ny);
        for (uint32_t q = sl; q < K; q += L)
            w_out[q] = w_store(aff8n(__ldg(&S.kern_work[kb + q]), (int)nx, (int)ny, nxny));
    }
    for (int off = 1; off < L; off <<= 1) {
        hs += __shfl_xor_sync(FULL, hs, off);
        ds += __shfl_xor_sync(FULL, ds, off);
    }
    __syncwarp();
    if (active && sl == 0) {
        double th = 0.0, td = 0.0;   // arrays without transfer add +0.0
        for (uint32_t a = 0; a < n_arrays; a++) {
            const double2 t2 = *reinterpret_cast<const double2 *>(&T[2 * a]);
            th = __dadd_rn(th, t2.x);
            td = __dadd_rn(td, t2.y);
        }
        Usage o;
        o.h = hs;
        o.d = ds;
        o.th = th;
        o.td = td;
        *res = o;
    }
}


// x mod m in [0, m) for m >= 1
__device__ __forceinline__ long long pmodll(long long x, long long m)
{
    const long long r = x % m;
    return r < 0 ? r + m : r;
}

// #{ r in [a, a + len) : r mod L == rho }, a >= 0, 0 <= rho < L
__device__ __forceinline__ unsigned long long count_residue(long long a, long long len, unsigned rho,
                                                           unsigned L)
{
    if (L == 1) return (unsigned long long)len;
    if (((unsigned long long)a | (unsigned long long)(a + len)) < (1ull << 31)) {   // 32-bit
        const unsigned ua = (unsigned)a, ub = (unsigned)(a + len);
        const unsigned first = ua + (rho + L - ua % L) % L;
        return first < ub ? (unsigned long long)((ub - 1u - first) / L) + 1ull : 0ull;
    }
    const long long first = a + pmodll((long long)rho - a, L);
    const long long b = a + len;
    return first < b ? (unsigned long long)((b - 1 - first) / L) + 1ull : 0ull;
}

// Rank-3 arrays (N4r): the planes [0, P) are cut into slabs at
// every region's plane bounds; f(pm, depth) is called per slab with the mask
// of the (valid) regions covering it.  2-D arrays: one slab [0, 1).
template <class F>
__device__ __forceinline__ void plane_slabs(bool valid, long long p0, long long p1, long long P, F &&f)
{
    if (P == 1) {   // 2-D arrays (and one-plane rank-3 ones): every valid region
        const unsigned pm = __ballot_sync(FULL, valid);
        if (pm) f(pm, 1ull);
        return;
    }
    long long z = 0;
    while (z < P) {
        long long c = P;
        if (valid && p0 > z && p0 < c) c = p0;
        if (valid && p1 > z && p1 < c) c = p1;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            const long long t = __shfl_xor_sync(FULL, c, o);
            c = t < c ? t : c;
        }
        const unsigned pm = __ballot_sync(FULL, valid && p0 <= z && c <= p1);
        if (pm) f(pm, (unsigned long long)(c - z));
        z = c;
    }
}

// Strided arrays (BRS [l:u:s]): the slabs of the sweep
// are split by row residue rho mod Lr and column residue sigma mod Lc (Lr, Lc
// = lcm of the array's steps); a region covers a (slab, residue) unit iff it
// covers the slab and its lattice hits the residue: (rho - l) mod step == 0.
// The first-reader / first-writer rule per cell is the dense sweep's.
__device__ __forceinline__ void strided_cells(SweepScratch &ws, unsigned Lr, unsigned Lc, int Sr, int Sc, int n,
                              long long ar, long long ac, unsigned rs, unsigned cs, unsigned Rm,
                              unsigned Wm, int lane, unsigned long long &h, unsigned long long &d,
                              bool valid, long long pl0, long long pl1, long long P)
{
    // residue masks: lane q marks the residues its lattice hits (phase,
    // phase + step, ... < L), then one ballot per residue transposes them
    // into pr_m[rho] / pc_m[sigma] = the regions hitting that residue
    unsigned long long rbits = 0, cbits = 0;
    if (lane < n) {
        for (unsigned r = (unsigned)pmodll(ar, rs); r < Lr; r += rs) rbits |= 1ull << r;
        for (unsigned c = (unsigned)pmodll(ac, cs); c < Lc; c += cs) cbits |= 1ull << c;
    }
    for (unsigned rho = 0; rho < Lr; rho++) {
        const unsigned m = __ballot_sync(FULL, (rbits >> rho) & 1ull);
        if (lane == 0) ws.pr_m[rho] = m;
    }
    for (unsigned sig = 0; sig < Lc; sig++) {
        const unsigned m = __ballot_sync(FULL, (cbits >> sig) & 1ull);
        if (lane == 0) ws.pc_m[sig] = m;
    }
    __syncwarp();
    // Aggregate the row units (slab i, residue rho) by coverage mask — their
    // heights add up, the first-reader / first-writer rule only sees the mask —
    // and the column units likewise; then classify each (row mask, column
    // mask) pair once with area = (sum of heights) x (sum of widths).  Far
    // fewer cells than the units' product; a table overflow (> 64 distinct
    // masks in a dimension) falls back to the product.
    for (int q = lane; q < 128; q += 32) {
        ws.agg_key[q >> 6][q & 63] = 0u;
        ws.agg_sum[q >> 6][q & 63] = 0ull;
    }
    if (lane == 0) ws.agg_over = 0u;
    __syncwarp();
    auto insert = [&](int dim, unsigned m, unsigned long long v) {
        unsigned slot = (m * 0x9E3779B1u) >> 26;
        for (int probe = 0; probe < 64; probe++, slot = (slot + 1) & 63u) {
            const unsigned old = atomicCAS(&ws.agg_key[dim][slot], 0u, m);
            if (old == 0u || old == m) {
                atomicAdd(&ws.agg_sum[dim][slot], v);
                return;
            }
        }
        ws.agg_over = 1u;
    };
    const int Ur = Sr * (int)Lr, Uc = Sc * (int)Lc;
    for (int u = lane; u < Ur; u += 32) {
        const int i = u / (int)Lr;
        const unsigned rho = (unsigned)(u - i * (int)Lr);
        const unsigned m = ws.rs_m[i] & ws.pr_m[rho];
        if (!m) continue;
        const unsigned long long hg = count_residue(ws.rs_a[i], ws.rs_h[i], rho, Lr);
        if (hg) insert(0, m, hg);
    }
    for (int u = lane; u < Uc; u += 32) {
        const int j = u / (int)Lc;
        const unsigned sig = (unsigned)(u - j * (int)Lc);
        const unsigned m = ws.cs_m[j] & ws.pc_m[sig];
        if (!m) continue;
        const unsigned long long wd = count_residue(ws.cs_a[j], ws.cs_w[j], sig, Lc);
        if (wd) insert(1, m, wd);
    }
    __syncwarp();
    if (!ws.agg_over) {
        // occupied slots as bit lists (ballots over the 64 slots)
        const unsigned long long occ_r =
            (unsigned long long)__ballot_sync(FULL, ws.agg_key[0][lane] != 0u) |
            (unsigned long long)__ballot_sync(FULL, ws.agg_key[0][lane + 32] != 0u) << 32;
        const unsigned long long occ_c =
            (unsigned long long)__ballot_sync(FULL, ws.agg_key[1][lane] != 0u) |
            (unsigned long long)__ballot_sync(FULL, ws.agg_key[1][lane + 32] != 0u) << 32;
        // compact into the (now free) slab arrays: masks -> rs_m / cs_m,
        // summed heights / widths -> rs_h / cs_w
        const unsigned long long below = (1ull << lane) - 1ull;
        const unsigned kr0 = ws.agg_key[0][lane], kr1 = ws.agg_key[0][lane + 32];
        const unsigned kc0 = ws.agg_key[1][lane], kc1 = ws.agg_key[1][lane + 32];
        const unsigned long long sr0 = ws.agg_sum[0][lane], sr1 = ws.agg_sum[0][lane + 32];
        const unsigned long long sc0 = ws.agg_sum[1][lane], sc1 = ws.agg_sum[1][lane + 32];
        __syncwarp();
        if (kr0) { const int q = __popcll(occ_r & below); ws.rs_m[q] = kr0; ws.rs_h[q] = (long long)sr0; }
        if (kr1) { const int q = __popcll(occ_r & (below << 32 | 0xffffffffull)); ws.rs_m[q] = kr1; ws.rs_h[q] = (long long)sr1; }
        if (kc0) { const int q = __popcll(occ_c & below); ws.cs_m[q] = kc0; ws.cs_w[q] = (long long)sc0; }
        if (kc1) { const int q = __popcll(occ_c & (below << 32 | 0xffffffffull)); ws.cs_m[q] = kc1; ws.cs_w[q] = (long long)sc1; }
        __syncwarp();
        const int nr = __popcll(occ_r), nc = __popcll(occ_c);
        plane_slabs(valid, pl0, pl1, P, [&](unsigned pm, unsigned long long depth) {
            const unsigned Rp = Rm & pm, Wp = Wm & pm;
            unsigned long long hs = 0, ds = 0;
            for (int p = lane; p < nr * nc; p += 32) {
                const int i = p / nc, j = p - i * nc;
                const unsigned m = ws.rs_m[i] & ws.cs_m[j];
                if (m) {
                    const unsigned long long area =
                        (unsigned long long)ws.rs_h[i] * (unsigned long long)ws.cs_w[j];
                    const unsigned mr = m & Rp, mw = m & Wp;
                    if (mr && (!mw || (mr & ws.upto[__ffs(mw) - 1]))) hs += area;
                    if (mw) ds += area;
                }
            }
            h += depth * hs;
            d += depth * ds;
        });
        return;
    }
    plane_slabs(valid, pl0, pl1, P, [&](unsigned pm, unsigned long long depth) {
    const unsigned Rp = Rm & pm, Wp = Wm & pm;
    unsigned long long hs = 0, ds = 0;
    for (int i = 0; i < Sr; i++) {
        const unsigned sm = ws.rs_m[i];
        if (!sm) continue;
        const long long ra = ws.rs_a[i], rh = ws.rs_h[i];
        for (unsigned rho = 0; rho < Lr; rho++) {
            const unsigned rm = sm & ws.pr_m[rho];
            if (!rm) continue;
            const unsigned long long hg = count_residue(ra, rh, rho, Lr);
            if (!hg) continue;
            for (int u = lane; u < Uc; u += 32) {
                const int j = u / (int)Lc;
                const unsigned sig = (unsigned)(u - j * (int)Lc);
                const unsigned m = rm & ws.cs_m[j] & ws.pc_m[sig];
                if (m) {
                    const unsigned long long area =
                        hg * count_residue(ws.cs_a[j], ws.cs_w[j], sig, Lc);
                    const unsigned mr = m & Rp, mw = m & Wp;
                    if (mr && (!mw || (mr & ws.upto[__ffs(mw) - 1]))) hs += area;
                    if (mw) ds += area;
                }
            }
        }
    }
    h += depth * hs;
    d += depth * ds;
    });
}

// Data usage of one (skeleton, nx, ny) key by the general coordinate-compressed
// sweep over the whole warp (DESIGN.md §3 N4; §III-B), plus
// the per-array PCIe transfer times in array order.  Used for keys outside
// their skeleton's plan domain.
__device__ __forceinline__ Usage warp_usage_sweep(const SpaceDev &S, const SkelInfo &I, long long nx, long long ny,
                                  const Price &pc, WarpScratch &wsu, int lane)
{
    SweepScratch &ws = wsu.sw;
    Usage o = {0ull, 0ull, 0.0, 0.0};
    const unsigned lt = (1u << lane) - 1u;
    for (uint32_t a = 0; a < I.n_arrays; a++) {
        const ArrayDev A = S.arrays[I.a_base + a];
        long long R = aff8(A.rows, nx, ny);
        long long C = aff8(A.cols, nx, ny);
        R = R > 0 ? R : 0;
        C = C > 0 ? C : 0;
        long long P = 1;                       // planes (rank-3 arrays, N4r)
        if (A.rank3) {
            P = aff8(A.planes, nx, ny);
            P = P > 0 ? P : 0;
        }
        const int n = (int)A.r_count;
        unsigned long long h = 0, d = 0;
        if (n > 0 && R > 0 && C > 0 && P > 0) {
            long long r0 = 0, r1 = 0, c0 = 0, c1 = 0, p0 = 0, p1 = 0;
            long long ar = 0, ac = 0;          // lattice anchors (unclamped lower bounds)
            bool valid = false;
            unsigned mode = 0, up = 0, rs = 1, cs = 1;
            if (lane < n) {
                const RegionDev &g = S.regions[A.r_base + lane];
                if (g.whole) {
                    r1 = R;
                    c1 = C;
                    p1 = P;
                } else {
                    ar = aff8(g.r0, nx, ny);
                    ac = aff8(g.c0, nx, ny);
                    r0 = clampll(ar, R);
                    r1 = clampll(aff8(g.r1, nx, ny), R);
                    c0 = clampll(ac, C);
                    c1 = clampll(aff8(g.c1, nx, ny), C);
                    if (A.rank3) {
                        p0 = clampll(aff8(g.p0, nx, ny), P);
                        p1 = clampll(aff8(g.p1, nx, ny), P);
                    } else {
                        p1 = 1;
                    }
                }
                valid = r0 < r1 && c0 < c1 && p0 < p1;
                mode = g.mode;
                up = g.upto;
                rs = g.rs;
                cs = g.cs;
            }
            const bool strided = A.lr > 1 || A.lc > 1;
            const unsigned vm = __ballot_sync(FULL, valid);
            const unsigned Rm = __ballot_sync(FULL, valid && (mode & GROPHECY_R));
            const unsigned Wm = __ballot_sync(FULL, valid && (mode & GROPHECY_W));
            if (vm) {
                const bool full = valid && r0 == 0 && r1 == R && c0 == 0 && c1 == C && rs == 1 &&
                                  cs == 1 && p0 == 0 && p1 == P;
                const unsigned fm = __ballot_sync(FULL, full);
                if (fm == vm) {
                    // every access covers the whole array: one cell
                    const int fwl = Wm ? __ffs(Wm) - 1 : 0;
                    const unsigned upw = __shfl_sync(FULL, up, fwl);
                    const unsigned long long area =
                        (unsigned long long)P * (unsigned long long)R * (unsigned long long)C;
                    if (Rm && (!Wm || (Rm & upw))) h = area;
                    if (Wm) d = area;
                } else {
                    if (lane < n) {
                        ws.box[lane][0] = r0;
                        ws.box[lane][1] = r1;
                        ws.box[lane][2] = c0;
                        ws.box[lane][3] = c1;
                        ws.upto[lane] = up;
                    }
                    __syncwarp();
                    // elementary slabs: for each breakpoint value, is it the
                    // first occurrence, the next larger breakpoint, and which
                    // boxes cover [value, next)
                    long long rn0 = BIG, rn1 = BIG, cn0 = BIG, cn1 = BIG;
                    bool rd0 = false, rd1 = false, cd0 = false, cd1 = false;
                    unsigned rm0 = 0, rm1 = 0, cm0 = 0, cm1 = 0;
                    for (int i = 0; i < n; i++) {
                        if (!((vm >> i) & 1u)) continue;
                        const long long b0 = ws.box[i][0], b1 = ws.box[i][1];
                        const long long b2 = ws.box[i][2], b3 = ws.box[i][3];
                        const bool before = i < lane;
                        rd0 |= before && (b0 == r0 || b1 == r0);
                        rd1 |= (i <= lane && b0 == r1) || (before && b1 == r1);
                        cd0 |= before && (b2 == c0 || b3 == c0);
                        cd1 |= (i <= lane && b2 == c1) || (before && b3 == c1);
                        if (b0 > r0 && b0 < rn0) rn0 = b0;
                        if (b1 > r0 && b1 < rn0) rn0 = b1;
                        if (b0 > r1 && b0 < rn1) rn1 = b0;
                        if (b1 > r1 && b1 < rn1) rn1 = b1;
                        if (b2 > c0 && b2 < cn0) cn0 = b2;
                        if (b3 > c0 && b3 < cn0) cn0 = b3;
                        if (b2 > c1 && b2 < cn1) cn1 = b2;
                        if (b3 > c1 && b3 < cn1) cn1 = b3;
                        const unsigned bit = 1u << i;
                        if (b0 <= r0 && r0 < b1) rm0 |= bit;
                        if (b0 <= r1 && r1 < b1) rm1 |= bit;
                        if (b2 <= c0 && c0 < b3) cm0 |= bit;
                        if (b2 <= c1 && c1 < b3) cm1 |= bit;
                    }
                    const bool sr0 = valid && !rd0 && rn0 != BIG;
                    const bool sr1 = valid && !rd1 && rn1 != BIG;
                    const bool sc0 = valid && !cd0 && cn0 != BIG;
                    const bool sc1 = valid && !cd1 && cn1 != BIG;
                    const unsigned br0 = __ballot_sync(FULL, sr0), br1 = __ballot_sync(FULL, sr1);
                    const unsigned bc0 = __ballot_sync(FULL, sc0), bc1 = __ballot_sync(FULL, sc1);
                    __syncwarp();
                    if (sr0) {
                        int p = __popc(br0 & lt);
                        ws.rs_h[p] = rn0 - r0;
                        ws.rs_m[p] = rm0;
                        ws.rs_a[p] = r0;
                    }
                    if (sr1) {
                        int p = __popc(br0) + __popc(br1 & lt);
                        ws.rs_h[p] = rn1 - r1;
                        ws.rs_m[p] = rm1;
                        ws.rs_a[p] = r1;
                    }
                    if (sc0) {
                        int p = __popc(bc0 & lt);
                        ws.cs_w[p] = cn0 - c0;
                        ws.cs_m[p] = cm0;
                        ws.cs_a[p] = c0;
                    }
                    if (sc1) {
                        int p = __popc(bc0) + __popc(bc1 & lt);
                        ws.cs_w[p] = cn1 - c1;
                        ws.cs_m[p] = cm1;
                        ws.cs_a[p] = c1;
                    }
                    __syncwarp();
                    const int Sr = __popc(br0) + __popc(br1);
                    const int Sc = __popc(bc0) + __popc(bc1);
                    if (strided) {
                        strided_cells(ws, A.lr, A.lc, Sr, Sc, n, ar, ac, rs, cs, Rm, Wm, lane, h, d,
                                      valid, p0, p1, P);
                    } else
                    plane_slabs(valid, p0, p1, P, [&](unsigned pm, unsigned long long depth) {
                        const unsigned Rp = Rm & pm, Wp = Wm & pm;
                        unsigned long long hs = 0, ds = 0;
                        for (int i = 0; i < Sr; i++) {
                            const unsigned rm = ws.rs_m[i] & pm;
                            if (!rm) continue;
                            const unsigned long long hg = (unsigned long long)ws.rs_h[i];
                            for (int j = lane; j < Sc; j += 32) {
                                const unsigned m = rm & ws.cs_m[j];
                                if (m) {
                                    const unsigned mr = m & Rp, mw = m & Wp;
                                    const unsigned long long area = hg * (unsigned long long)ws.cs_w[j];
                                    if (mr && (!mw || (mr & ws.upto[__ffs(mw) - 1]))) hs += area;
                                    if (mw) ds += area;
                                }
                            }
                        }
                        h += depth * hs;
                        d += depth * ds;
                    });
                    h = warp_sum_u64(h);
                    d = warp_sum_u64(d);
                    __syncwarp();
                }
            }
        }
        add_array(o, A, h, d, pc, nx, ny);
    }
    return o;
}

// ---- approximate mode: BRS algebra with the Havlak-Kennedy UNION ----------
// ([5]; N4h).  One dimension of a
// section {l, l+s, ..., u}: s == 0 iff one element, empty iff l > u.
struct Sec1 {
    long long l, u, s;
};

__device__ __forceinline__ bool sec1_empty(const Sec1 &a) { return a.l > a.u; }

__device__ __forceinline__ long long gcdll(long long a, long long b)
{
    a = a < 0 ? -a : a;
    b = b < 0 ? -b : b;
    while (b) {
        const long long t = a % b;
        a = b;
        b = t;
    }
    return a;
}

// lattice anchor + i*step inside [lo, hi)
__device__ __forceinline__ Sec1 sec1_make(long long lo, long long hi, long long anchor, long long step)
{
    Sec1 v = {1, 0, 0};
    const long long first = lo + pmodll(anchor - lo, step);
    if (first >= hi) return v;
    v.l = first;
    v.u = first + ((hi - 1 - first) / step) * step;
    v.s = v.l == v.u ? 0 : step;
    return v;
}

__device__ __forceinline__ Sec1 sec1_union(const Sec1 &a, const Sec1 &b)
{
    if (sec1_empty(a)) return b;
    if (sec1_empty(b)) return a;
    Sec1 v;
    v.l = a.l < b.l ? a.l : b.l;
    v.u = a.u > b.u ? a.u : b.u;
    v.s = gcdll(gcdll(a.s, b.s), a.l - b.l);
    if (v.l == v.u) v.s = 0;
    return v;
}

// every element of x (non-empty) is one of w (non-empty)
__device__ __forceinline__ bool sec1_contains(const Sec1 &w, const Sec1 &x)
{
    if (w.s == 0) return x.l == w.l && x.u == w.l;
    return x.l >= w.l && x.u <= w.u && pmodll(x.l - w.l, w.s) == 0 && x.s % w.s == 0;
}

__device__ __forceinline__ unsigned long long sec1_count(const Sec1 &a)
{
    if (sec1_empty(a)) return 0ull;
    return a.s == 0 ? 1ull : (unsigned long long)((a.u - a.l) / a.s) + 1ull;
}

// One dimension (rows: dim 0, columns: dim 1) of a region's section.
__device__ __forceinline__ Sec1 region_sec1(const RegionDev &g, int dim, long long nx, long long ny,
                                            long long E, bool rank3 = false)
{
    if (g.whole) return sec1_make(0, E, 0, 1);
    if (dim == 2) {   // planes (rank-3 arrays, N4r): dense [p0, p1); 2-D arrays [0, 1)
        if (!rank3) return sec1_make(0, E, 0, 1);
        const long long q0 = clampll(aff8(g.p0, nx, ny), E);
        return sec1_make(q0, clampll(aff8(g.p1, nx, ny), E), q0, 1);
    }
    const int4 lo = dim ? g.c0 : g.r0, hi = dim ? g.c1 : g.r1;
    const long long an = aff8(lo, nx, ny);
    return sec1_make(clampll(an, E), clampll(aff8(hi, nx, ny), E), an, dim ? g.cs : g.rs);
}

// Usage of one key in the approximate mode: lane a works on array a.  Its
// regions are sorted by kernel, so the write sections of earlier kernels are
// the write regions before the first region of the current kernel.  Pass 1
// marks the kept reads (not inside one earlier write section, both
// dimensions); the hulls are then built one dimension at a time (the HK
// UNION works per dimension), which keeps the live state small.
__device__ __forceinline__ Usage warp_usage_hull(const SpaceDev &S, const SkelInfo &I, long long nx,
                                                 long long ny, const Price &pc, int lane)
{
    unsigned long long h = 0, d = 0;
    if ((uint32_t)lane < I.n_arrays) {
        const ArrayDev &A = S.arrays[I.a_base + lane];
        long long E[3] = {aff8(A.rows, nx, ny), aff8(A.cols, nx, ny),
                          A.rank3 ? aff8(A.planes, nx, ny) : 1};
        E[0] = E[0] > 0 ? E[0] : 0;
        E[1] = E[1] > 0 ? E[1] : 0;
        E[2] = E[2] > 0 ? E[2] : 0;
        const bool r3 = A.rank3 != 0;
        const RegionDev *G = S.regions + A.r_base;
        const uint32_t n = A.r_count;
        uint32_t nonempty = 0, keep = 0, wmask = 0;
        for (uint32_t j = 0; j < n; j++) {
            const Sec1 xr = region_sec1(G[j], 0, nx, ny, E[0]);
            const Sec1 xc = region_sec1(G[j], 1, nx, ny, E[1]);
            const Sec1 xp = region_sec1(G[j], 2, nx, ny, E[2], r3);
            if (sec1_empty(xr) || sec1_empty(xc) || sec1_empty(xp)) continue;
            nonempty |= 1u << j;
            if (G[j].mode & GROPHECY_W) wmask |= 1u << j;
            if (!(G[j].mode & GROPHECY_R)) continue;
            bool written = false;
            for (uint32_t q = 0; q < j && !written; q++) {
                if (!((wmask >> q) & 1u) || G[q].kernel >= G[j].kernel) continue;
                written = sec1_contains(region_sec1(G[q], 0, nx, ny, E[0]), xr) &&
                          sec1_contains(region_sec1(G[q], 1, nx, ny, E[1]), xc) &&
                          (!r3 || sec1_contains(region_sec1(G[q], 2, nx, ny, E[2], r3), xp));
            }
            if (!written) keep |= 1u << j;
        }
        unsigned long long cr = 1, cw = 1;
        for (int dim = 0; dim < (r3 ? 3 : 2); dim++) {   // 2-D arrays: one plane
            Sec1 hr = {1, 0, 0}, hw = {1, 0, 0};
            for (uint32_t j = 0; j < n; j++) {
                if (!((nonempty >> j) & 1u)) continue;
                const Sec1 x = region_sec1(G[j], dim, nx, ny, E[dim], r3);
                if ((keep >> j) & 1u) hr = sec1_union(hr, x);
                if ((wmask >> j) & 1u) hw = sec1_union(hw, x);
            }
            cr *= sec1_count(hr);
            cw *= sec1_count(hw);
        }
        h = keep ? cr : 0ull;
        d = wmask ? cw : 0ull;
    }
    Usage o = {0ull, 0ull, 0.0, 0.0};
    for (uint32_t a = 0; a < I.n_arrays; a++) {   // transfer times in array order
        const unsigned long long ha = __shfl_sync(FULL, h, a), da = __shfl_sync(FULL, d, a);
        add_array(o, S.arrays[I.a_base + a], ha, da, pc, nx, ny);
    }
    return o;
}

// Usage of one key off the plan path (outside the plan's domain, strided
// sections, the hull mode) and its kernels' work counts, by the whole warp.
__device__ __forceinline__ void slow_usage(const SpaceDev *gS, unsigned long long k, const Price &pc,
                                        WarpScratch *scr, Usage *res, uint32_t *w_out, int lane)
{
    const SpaceDev &S = *gS;
    const SkelInfo &I = S.skel[(uint32_t)(k >> 42)];
    const long long kx_ = (long long)((k >> 21) & 0x1fffffull);
    const long long ky_ = (long long)(k & 0x1fffffull);
    const Usage r = (I.flags & GROPHECY_SKEL_HULL) ? warp_usage_hull(S, I, kx_, ky_, pc, lane)
                                                   : warp_usage_sweep(S, I, kx_, ky_, pc, *scr, lane);
    if (lane == 0) *res = r;
    if (w_out && (uint32_t)lane < I.n_kernels)
        w_out[lane] = w_store(aff8(__ldg(&S.kern_work[I.k_base + lane]), kx_, ky_));
}

// Kernel time of one kernel (DESIGN.md §3 N5) from its work-item count Wi and
// its (kernel, transformation) constants J / kxi.
__device__ __forceinline__ double kernel_time(const SpaceDev &S, long long Wi, const KxJ &J,
                                              uint32_t kxi)
{
    const unsigned long long W = Wi > 0 ? (unsigned long long)Wi : 0ull;
    if (J.flags & KXF_INFEASIBLE) return __longlong_as_double(0x7ff0000000000000LL);
    const KxI II = S.kx_i[kxi];
    unsigned long long blocks;
    if (W < (1ull << 32)) {
        const unsigned long long q = II.magic ? __umul64hi(II.magic, W) : W;
        blocks = q + (q * J.ipb != W);
    } else {
        blocks = W / J.ipb + (W % J.ipb != 0);
    }
    if (blocks == 0) return 0.0;
    if (blocks >= II.sat_blocks) {
        const KxES es = S.kx_es[kxi];
        const KxD dd = S.kx_d[kxi];
        const double rep = div_rn(__ull2double_rn(blocks), dd.D, dd.rD);
        const double cyc = __dadd_rn(__dmul_rn(es.E, rep), __dmul_rn(es.S, rep));
        return div_rn(cyc, S.freq, S.rfreq);
    }
    // general (small) grid: the definition step by step
    const KxG G = S.kx_g[kxi];
    const unsigned long long nsm = S.n_sm;
    const unsigned long long asm_ = nsm < blocks ? nsm : blocks;
    unsigned long long abps = blocks / asm_ + (blocks % asm_ != 0);
    if ((unsigned long long)J.occ < abps) abps = J.occ;
    const double N = __ull2double_rn(abps * (unsigned long long)J.wpb);
    // integer denominators: RN(1/d) by __drcp_rn, then Markstein's correction
    const double dden = __ull2double_rn(abps * asm_);
    const double rep = div_rn(__ull2double_rn(blocks), dden, __drcp_rn(dden));
    double cyc;
    if (J.flags & KXF_NOMEM) {
        cyc = __dmul_rn(__dmul_rn(G.comp, N), rep);
    } else {
        const double dasm = __ull2double_rn(asm_);
        const double mpk = div_rn(G.bwr, dasm, __drcp_rn(dasm));
        const double mwp = dmin(dmin(G.mwp0, mpk), N);
        const double cwp = dmin(G.cwpf, N);
        const double cpm_term = __dmul_rn(G.cpm, __dsub_rn(mwp, 1.0));
        if (mwp == N && cwp == N)
            cyc = __dmul_rn(__dadd_rn(__dadd_rn(G.memc, G.comp), cpm_term), rep);
        else if (cwp >= mwp || G.comp > G.memc)
            cyc = __dmul_rn(__dadd_rn(__ddiv_rn(__dmul_rn(G.memc, N), mwp), cpm_term), rep);
        else
            cyc = __dmul_rn(__dadd_rn(G.ml, __dmul_rn(G.comp, N)), rep);
        const double sync = __dmul_rn(
            __dmul_rn(__dmul_rn(__dmul_rn(G.dd, __dsub_rn(mwp, 1.0)), G.synch),
                      __ull2double_rn(abps)),
            rep);
        cyc = __dadd_rn(cyc, sync);
    }
    return div_rn(cyc, S.freq, S.rfreq);
}

// Total projected time of one candidate: kernels (run-once
// plus iters x per-iteration) + transfers.  val = the key's plan values
// (work counts at 0..K-1) or NULL to evaluate the work expressions here.
__device__ __forceinline__ double candidate_time(const SpaceDev &S, uint32_t s, uint32_t x,
                                                 long long nx, long long ny, uint32_t it,
                                                 const long long *val, const Usage &u)
{
    const SkelInfo &I = S.skel[s];
    const uint32_t K = I.n_kernels, X = I.n_xforms, kb = I.k_base;
    uint32_t kxi = I.kx_base + x;
    double t_iter = 0.0, t_once = 0.0;
    for (uint32_t k = 0; k < K; k++, kxi += X) {
        const long long Wi = val ? val[k] : aff8(__ldg(&S.kern_work[kb + k]), nx, ny);
        const KxJ J = S.kx_j[kxi];
        const double tk = kernel_time(S, Wi, J, kxi);
        if (J.flags & KXF_PER_ITER) t_iter = __dadd_rn(t_iter, tk);
        else t_once = __dadd_rn(t_once, tk);
    }
    const double t_kern = __dadd_rn(t_once, __dmul_rn((double)it, t_iter));
    return __dadd_rn(__dadd_rn(t_kern, u.th), u.td);
}

struct Best {
    double t;
    unsigned long long i, h, d, ninv, nval;
};

__device__ __forceinline__ bool better(double ta, unsigned long long ia, double tb,
                                       unsigned long long ib)
{
    return ta < tb || (ta == tb && ia < ib);
}

__device__ __forceinline__ void merge(Best &a, const Best &b)
{
    if (better(b.t, b.i, a.t, a.i)) {
        a.t = b.t;
        a.i = b.i;
        a.h = b.h;
        a.d = b.d;
    }
    a.ninv += b.ninv;
    a.nval += b.nval;
}

__device__ __forceinline__ Best shfl_best(const Best &b, int src_xor)
{
    Best o;
    o.t = __shfl_xor_sync(FULL, b.t, src_xor);
    o.i = __shfl_xor_sync(FULL, b.i, src_xor);
    o.h = __shfl_xor_sync(FULL, b.h, src_xor);
    o.d = __shfl_xor_sync(FULL, b.d, src_xor);
    o.ninv = __shfl_xor_sync(FULL, b.ninv, src_xor);
    o.nval = __shfl_xor_sync(FULL, b.nval, src_xor);
    return o;
}

__device__ __forceinline__ Best warp_best(Best b)
{
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) merge(b, shfl_best(b, o));
    return b;
}

__device__ __forceinline__ Best none_best()
{
    Best b;
    b.t = __longlong_as_double(0x7ff0000000000000LL);
    b.i = ~0ull;
    b.h = b.d = b.ninv = b.nval = 0;
    return b;
}

__device__ __forceinline__ Best from_result(const grophecy_best_result &r)
{
    Best b;
    b.t = r.t_total_s;
    b.i = r.index;
    b.h = r.h2d_bytes;
    b.d = r.d2h_bytes;
    b.ninv = r.n_invalid;
    b.nval = r.n_valid;
    return b;
}

__device__ __forceinline__ void to_result(grophecy_best_result &r, const Best &b)
{
    r.t_total_s = b.t;
    r.index = b.i;
    r.h2d_bytes = b.h;
    r.d2h_bytes = b.d;
    r.n_invalid = b.ninv;
    r.n_valid = b.nval;
}

// Canonical tiles: CX consecutive records per group, 32 groups per tile (one
// group per lane in phases A/B).  Phase C maps lane = (transformation x,
// half h): the lane models transformation x of groups h, h + 2, ..., CG
// groups per pass, so one (kernel, x) constant load serves CG records.
// Work counters after P.tile_count (the space's 128-byte counter block):
// the pass-1 and pass-2 tile claims.  (Separate 32-byte sectors, with the
// pass-1 claim issued a tile further ahead, measured 2 % slower on C4.)
constexpr int CLAIM1 = 2, CLAIM2 = 1;
constexpr int CX = 16;
constexpr int CTILE = 32 * CX;
#ifndef GROPHECY_AU32
#define GROPHECY_AU32 4
#endif
#ifndef GROPHECY_CG
#define GROPHECY_CG 8
#endif
constexpr int CG = GROPHECY_CG;   // groups per lane per model pass (divides 16)
#ifndef GROPHECY_CMINB
#define GROPHECY_CMINB 2
#endif

// Per-warp shared memory of the general kernel (dynamic; > 48 KB per CTA
// needs the opt-in attribute).
struct WarpSmem {
    WarpScratch scratch;                        // usage plans / general sweep
    unsigned long long slot_key[SLOT_CAP];      // distinct keys of the chunk
    Usage res[SLOT_CAP];                        // their usage
    uint32_t slot_w[SLOT_CAP][MAXK + 1];        // their work-item counts (w_store; padded row)
    unsigned long long rec_key[WTILE];          // the tile's records after phase A
    uint32_t rec_skx[WTILE], rec_it[WTILE];
    int rec_slot[WTILE];
    uint8_t plan_pos[MAX_SEG];                  // plan keys of the current slot group
    unsigned long long best_h[32], best_d[32];  // bytes of each lane's running best
};
// ... and of the canonical kernel.  Per group g (= lane of phase A/B):
// work counts at cw[k][g & 1][g >> 1] (a phase-C lane of half h reads its
// groups h, h + 2, ... as consecutive words), usage and iterations at [g].
// The work counts follow the struct in the warp's slice, sized by the
// space's largest kernel count (canon_warp_bytes): shared memory left to L1,
// which the usage polynomials and the constants live in.
struct alignas(128) CanonSmem {
    alignas(128) uint32_t rec[4][CTILE];        // the tile's SoA records (TMA bulk copies)
    // per group g at index (g & 1) * 16 + (g >> 1): a phase-C lane's groups
    // (h, h + 2, ...) are consecutive (vector loads)
    alignas(16) double th[32], td[32], it[32];  // transfer times, (double) iters
    unsigned long long uh[32], ud[32];          // transfer bytes
    unsigned long long best_h[32], best_d[32];
    unsigned long long mbar;                    // completion of the rec copies
};
constexpr uint32_t CW_BYTES_PER_KERNEL = 2 * 16 * sizeof(uint32_t);   // cw[k][2][16] (w_store)
__host__ __device__ constexpr uint32_t canon_warp_bytes(uint32_t kmax)
{
    return (uint32_t)((sizeof(CanonSmem) + kmax * CW_BYTES_PER_KERNEL + 127) / 128 * 128);
}
struct CtaSmem {
    WarpSmem w[WARPS];
};

// Saturated-grid kernel time (DESIGN.md §3 N5, saturated reduction) of one
// (record, kernel) from the packed constants (sat, sh = satsh fields) and
// the stored work count w (w_store, < 2^30 here): blocks = ceil(w / ipb) by
// one 32x32+64 multiply-add and a shift, cyc = E rep + S rep, rep = blocks /
// D, t = cyc / freq, both divisions by the two-product method (x * zh +
// RN(x * zl) with zh + zl = 1/divisor; one DMUL + one DFMA, bitwise the IEEE
// quotient: DESIGN.md §5).  gen is set when the grid is not saturated — the
// returned value is then meaningless and the general branch decides.
__device__ __forceinline__ double fast_time(const KxFast &f, uint32_t sat, uint32_t sh, uint32_t w,
                                            double rfh, double rfl, bool &gen, uint32_t &blocks)
{
    const unsigned long long p = (unsigned long long)w * f.m + f.cc;
    blocks = (uint32_t)(p >> 32) >> sh;
    gen = blocks < sat;
    const double bb = __uint2double_rn(blocks);
    const double rep = __fma_rn(bb, f.rDh, __dmul_rn(bb, f.rDl));
    const double cyc = __dadd_rn(__dmul_rn(f.E, rep), __dmul_rn(f.S, rep));
    return __fma_rn(cyc, rfh, __dmul_rn(cyc, rfl));
}

// Kernel time off the saturated path: the small-grid table when the pair is
// tabulated (space.cpp), else the definition step by step (infeasible pairs,
// grids beyond the table, huge work counts).  Wi() recomputes the work count.
template <class WiF>
__device__ __forceinline__ double gen_time(const SpaceDev &S, uint32_t kxi, uint32_t sat32,
                                           double E, uint32_t w, uint32_t blocks, WiF Wi)
{
    if (sat32 <= S.small_stride && w != W_HUGE)
        return __ldg(&S.small_t[(size_t)kxi * S.small_stride + blocks]);
    if (E == __longlong_as_double(0x7ff0000000000000LL)) return E;   // infeasible: +inf
    return kernel_time(S, Wi(), S.kx_j[kxi], kxi);
}

// Model of NJ records of one skeleton at once (NJ independent dependency
// chains per thread).  W[j] = the work-item counts of record j's key (shared
// memory, one row per distinct key).  The saturated-grid formula is computed
// for every record; the rare general-grid cases are recomputed by kernel_time.
template <int NJ, bool SAMEX>
__device__ __forceinline__ void model_n(const SpaceDev &S, uint32_t s, const uint32_t *x,
                                        const int *ls, const WarpSmem &ws, double *t_iter,
                                        double *t_once)
{
    const SkelInfo &I = S.skel[s];
    const uint32_t K = I.n_kernels, X = I.n_xforms, pim = I.per_iter_mask;
    double ti[NJ], to[NJ];
#pragma unroll
    for (int j = 0; j < NJ; j++) ti[j] = to[j] = 0.0;
    uint32_t kb = I.kx_base;
    for (uint32_t k = 0; k < K; k++, kb += X) {
        double tk[NJ];
        bool gen[NJ];
        KxFast F0;
        if (SAMEX) F0 = S.kx_f[kb + x[0]];   // one constant load shared by the NJ records
        uint32_t w[NJ], blocks[NJ], sat[NJ];
        double E[NJ];
#pragma unroll
        for (int j = 0; j < NJ; j++) {
            const KxFast F = SAMEX ? F0 : S.kx_f[kb + x[j]];
            w[j] = ws.slot_w[ls[j]][k];
            sat[j] = F.satsh & KXF_SAT_MASK;
            tk[j] = fast_time(F, sat[j], F.satsh >> KXF_SAT_BITS, w[j], S.rfh, S.rfl, gen[j],
                              blocks[j]);
            gen[j] |= w[j] == W_HUGE;
            E[j] = F.E;
        }
        bool any = false;
#pragma unroll
        for (int j = 0; j < NJ; j++) any |= gen[j];
        if (any) {
#pragma unroll
            for (int j = 0; j < NJ; j++)
                if (gen[j]) {
                    const unsigned long long kk = ws.slot_key[ls[j]];
                    tk[j] = gen_time(S, kb + x[j], sat[j], E[j], w[j], blocks[j], [&] {
                        return aff8(__ldg(&S.kern_work[I.k_base + k]),
                                    (long long)((kk >> 21) & 0x1fffffull), (long long)(kk & 0x1fffffull));
                    });
                }
        }
        if ((pim >> k) & 1u) {
#pragma unroll
            for (int j = 0; j < NJ; j++) ti[j] = __dadd_rn(ti[j], tk[j]);
        } else {
#pragma unroll
            for (int j = 0; j < NJ; j++) to[j] = __dadd_rn(to[j], tk[j]);
        }
    }
    // infeasible kernels (fast path: a finite 0): that sum is +inf (xinf)
#pragma unroll
    for (int j = 0; j < NJ; j++) {
        const uint32_t xf = __ldg(&S.xinf[I.kx_base + x[j]]);
        const double inf = __longlong_as_double(0x7ff0000000000000LL);
        t_iter[j] = (xf & XINF_ITER) ? inf : ti[j];
        t_once[j] = (xf & XINF_ONCE) ? inf : to[j];
    }
}


struct Params {
    SpaceDev S;
    const SpaceDev *gS;   // device copy of S (out-of-line paths)
    grophecy_pcie pc;
    Price pr;             // general path pricing (pc, or the memory choice)
    const uint32_t *skx, *nx, *ny, *iters;
    unsigned long long n, base;
    unsigned long long *h2d;
    unsigned long long *d2h;
    double *t;
    double *p_iter, *p_once, *p_h2d, *p_d2h;   // optional component outputs (eval)
    grophecy_best_result *partials;
    unsigned int *ticket;
    grophecy_best_result *out;
    int accumulate;
    int aligned;    // record arrays 16-byte aligned -> vector loads
    uint32_t *tile_list;      // pass 1 -> pass 2: tiles left to the general path
    unsigned int *tile_count;
    uint32_t canon_warp_bytes; // pass 1: shared memory per warp (canon_warp_bytes(kmax))
    uint32_t sweep_kmax;       // sweep kernel: the space's largest work-slot count (smem layout)
    int direct;                // pass 2 takes every warp tile of the batch (no pass 1, no list)
    int reset_counters;        // best mode: pass 2 leaves the tile counters zeroed for the next call
    int fused;                 // best mode: the sweep kernel runs pass 2 itself (cooperative launch)
    // striped batches (grophecy_batch.stripe_len != 0): kernels work with
    // batch-local indices (base = the launch's local offset) and the final
    // best index is mapped to map_base + (i / map_len) * map_stride + i % map_len
    unsigned long long map_len, map_stride, map_base;
};

// Record validity (include/grophecy.h) and its usage key (skeleton, nx, ny).
// n_xf = the skeleton's n_xforms (looked up by the caller).
__device__ __forceinline__ unsigned long long key_of(const SpaceDev &S, uint32_t skx, uint32_t nx,
                                                     uint32_t ny, uint32_t it, bool has, uint32_t n_xf)
{
    const uint32_t skel = skx >> 16, x = skx & 0xffffu;
    const bool valid = has && skel < S.n_skels && nx - 1u < GROPHECY_MAX_DIM &&
                       ny - 1u < GROPHECY_MAX_DIM && it >= 1 && x < n_xf;
    return valid ? ((unsigned long long)skel << 42) | ((unsigned long long)nx << 21) | ny : ~0ull;
}

// Persistent kernel; every warp works alone on tiles of 128 consecutive
// records (no CTA barriers on the hot loop):
//   A  lane l loads records 4l..4l+3 (one 16-byte load per SoA array), checks
//      them, and run heads of equal keys get slot ids by a warp scan;
//   B  usage of each distinct key once (plan: 32/L keys per pass; else sweep);
//   C  lane l models records l, l+32, l+64, l+96 — the same transformation
//      when candidates come in groups of 16 — sharing one constant load per
//      kernel, then writes outputs / keeps its running argmin.
// One general tile: 128 consecutive records from tb (any layout, ragged
// tail, invalid records), processed by one warp:
//   A  lane l loads records l + 32 j, checks them, and run heads of equal
//      keys get slot ids by a warp scan;
//   B  usage of each distinct key once (plan: 8 keys per pass; else sweep);
//   C  lane l models records l, l+32, l+64, l+96 — the same transformation
//      when candidates come in groups of 16 — sharing one constant load per
//      kernel, then writes outputs / keeps its running argmin.
template <bool BEST>
__device__ __forceinline__ void general_tile(const Params &P, WarpSmem &ws, unsigned long long tb,
                                             int lane, double &best_t, unsigned long long &best_i,
                                             uint32_t &cnt_inv, uint32_t &cnt_val)
{
    const SpaceDev &S = P.S;
    const unsigned lt = (1u << lane) - 1u;
        // ---- A: records q = lane + 32 j (coalesced 32-bit loads), keys, one
        //      slot per distinct key of each 32 records (match + ballots) ----
        uint32_t skx[RPT], nx[RPT], ny[RPT], it[RPT];
#pragma unroll
        for (int j = 0; j < RPT; j++) {
            const unsigned long long i = tb + lane + 32 * j;
            const bool h = i < P.n;
            skx[j] = h ? __ldcs(P.skx + i) : 0u;
            nx[j] = h ? __ldcs(P.nx + i) : 0u;
            ny[j] = h ? __ldcs(P.ny + i) : 0u;
            it[j] = h ? __ldcs(P.iters + i) : 0u;
        }
        unsigned long long key[RPT];
        {
            // one n_xforms lookup per distinct skeleton among the lane's records
            uint32_t nxf = 0, last = 0xffffffffu;
#pragma unroll
            for (int j = 0; j < RPT; j++) {
                const uint32_t sj = skx[j] >> 16;
                if (sj != last && sj < S.n_skels) {
                    nxf = S.skel[sj].n_xforms;
                    last = sj;
                }
                key[j] = key_of(S, skx[j], nx[j], ny[j], it[j], tb + lane + 32 * j < P.n,
                                sj == last ? nxf : 0u);
            }
        }
        unsigned n_invalid = 0, n_valid = 0;
        unsigned nslots = 0;
        const unsigned le = (2u << lane) - 1u;   // lanes <= this one
#pragma unroll
        for (int j = 0; j < RPT; j++) {
            // one slot per distinct key of the 32 records lane + 32 j (equal keys
            // need not be adjacent: any order of a design point's records),
            // its lowest lane the head; slots in head order
            const unsigned mk = __match_any_sync(FULL, key[j]);
            const int leader = __ffs(mk) - 1;
            const bool head = key[j] != ~0ull && lane == leader;
            const unsigned hb = __ballot_sync(FULL, head);
            const int hslot = (int)(nslots + __popc(hb & le)) - 1;
            const int lslot = __shfl_sync(FULL, hslot, leader);   // (every lane: FULL mask)
            const int slot = key[j] == ~0ull ? -1 : lslot;
            nslots += __popc(hb);
            const int q = lane + 32 * j;
            ws.rec_skx[q] = skx[j];
            ws.rec_it[q] = it[j];
            ws.rec_slot[q] = head ? -2 - slot : slot;   // heads encoded as -2 - slot
            ws.rec_key[q] = key[j];
            const bool has = tb + q < P.n;
            n_invalid += has && key[j] == ~0ull;
            n_valid += key[j] != ~0ull;
        }
        (void)lt;
        __syncwarp();
        // from here on the tile lives in shared memory (keeps registers free
        // for the model's independent dependency chains)

        for (unsigned c0 = 0; c0 < nslots; c0 += SLOT_CAP) {
            const unsigned c1 = min(nslots, c0 + SLOT_CAP);
#pragma unroll
            for (int j = 0; j < RPT; j++) {
                const int q = lane + 32 * j;
                const int hs = ws.rec_slot[q];   // heads are encoded as -2 - slot
                if (hs <= -2 && (unsigned)(-2 - hs) >= c0 && (unsigned)(-2 - hs) < c1)
                    ws.slot_key[-2 - hs - c0] = ws.rec_key[q];
            }
            __syncwarp();
            // ---- B: usage of every distinct key of the chunk, once ----
            for (unsigned g0 = c0; g0 < c1; g0 += MAX_SEG) {
                const unsigned gcnt = min((unsigned)MAX_SEG, c1 - g0);
                const bool mv = (unsigned)lane < gcnt;
                const unsigned long long mk = mv ? ws.slot_key[g0 - c0 + lane] : 0ull;
                bool mplan = false;
                if (mv) {
                    const SkelInfo &I = S.skel[(uint32_t)(mk >> 42)];
                    mplan = (long long)((mk >> 21) & 0x1fffffull) >= I.plan_tx &&
                            (long long)(mk & 0x1fffffull) >= I.plan_ty;
                }
                unsigned todo = __ballot_sync(FULL, mv && mplan);
                unsigned sweep = __ballot_sync(FULL, mv && !mplan);
                // 4 lanes per key, 8 keys per pass
                constexpr int L = 32 / MAX_SEG, G = MAX_SEG;
                const int seg = lane / L, sl = lane % L;
                // compact list of the plan keys' positions (rank -> slot lane)
                if (mv && mplan) ws.plan_pos[__popc(todo & ((1u << lane) - 1u))] = (uint8_t)lane;
                const int nplan = __popc(todo);
                __syncwarp();
                for (int p0 = 0; p0 < nplan; p0 += G) {
                    const bool act = p0 + seg < nplan;
                    const unsigned pos = act ? ws.plan_pos[p0 + seg] : 0u;
                    const unsigned long long k = __shfl_sync(FULL, mk, pos);
                    const unsigned ls = g0 - c0 + pos;
                    plan_usage(S, act, k, P.pr, ws.scratch.pl.T[seg], sl, L, &ws.res[ls],
                               ws.slot_w[ls]);
                    __syncwarp();
                }
                while (sweep) {
                    const int pos = __ffs(sweep) - 1;
                    const unsigned long long k = __shfl_sync(FULL, mk, pos);
                    slow_usage(P.gS, k, P.pr, &ws.scratch, &ws.res[g0 - c0 + pos],
                               ws.slot_w[g0 - c0 + pos], lane);
                    sweep &= sweep - 1;
                    __syncwarp();
                }
            }
            __syncwarp();
            // ---- C: per-candidate model + output / argmin (records lane + 32 j) ----
            int ls[RPT];
            uint32_t xs[RPT];
            bool inj[RPT];
            double ti[RPT], to[RPT];
            const uint32_t skx0 = ws.rec_skx[lane];
            bool same = true;
#pragma unroll
            for (int j = 0; j < RPT; j++) {
                const int q = lane + 32 * j;
                int sj = ws.rec_slot[q];
                if (sj <= -2) sj = -2 - sj;
                const uint32_t sk = ws.rec_skx[q];
                inj[j] = sj >= (int)c0 && sj < (int)c1;
                ls[j] = inj[j] ? sj - (int)c0 : 0;
                xs[j] = sk & 0xffffu;
                same = same && inj[j] && sk == skx0;
            }
            if (same) {
                model_n<RPT, true>(S, skx0 >> 16, xs, ls, ws, ti, to);
            } else {
#pragma unroll
                for (int j = 0; j < RPT; j++)
                    if (inj[j])
                        model_n<1, false>(S, ws.rec_skx[lane + 32 * j] >> 16, xs + j, ls + j, ws,
                                          ti + j, to + j);
            }
            double tt[RPT];
#pragma unroll
            for (int j = 0; j < RPT; j++) {
                const Usage &u = ws.res[ls[j]];
                // total: run-once + iters x per-iteration + transfers
                const double t_kern = __dadd_rn(to[j], __dmul_rn((double)ws.rec_it[lane + 32 * j], ti[j]));
                tt[j] = __dadd_rn(__dadd_rn(t_kern, u.th), u.td);
            }
            if (!BEST) {
#pragma unroll
                for (int j = 0; j < RPT; j++) {
                    if (!inj[j]) continue;
                    const unsigned long long i = tb + lane + 32 * j;
                    const Usage &u = ws.res[ls[j]];
                    __stcs(P.h2d + i, u.h);
                    __stcs(P.d2h + i, u.d);
                    __stcs(P.t + i, tt[j]);
                    if (P.p_iter) __stcs(P.p_iter + i, ti[j]);
                    if (P.p_once) __stcs(P.p_once + i, to[j]);
                    if (P.p_h2d) __stcs(P.p_h2d + i, u.th);
                    if (P.p_d2h) __stcs(P.p_d2h + i, u.td);
                }
            } else {
                // the lane's best of its (index-ordered) records, then one compare
                double bt = __longlong_as_double(0x7ff0000000000000LL);
                int bj = -1, bls = 0;
#pragma unroll
                for (int j = 0; j < RPT; j++)
                    if (inj[j] && tt[j] < bt) {
                        bt = tt[j];
                        bj = j;
                        bls = ls[j];
                    }
                if (bj >= 0) {
                    const unsigned long long i = P.base + tb + lane + 32 * bj;
                    if (better(bt, i, best_t, best_i)) {
                        best_t = bt;
                        best_i = i;
                        const Usage &u = ws.res[bls];
                        ws.best_h[lane] = u.h;
                        ws.best_d[lane] = u.d;
                    }
                }
            }
            __syncwarp();
        }
        // invalid records: (0, 0, NaN) outputs and counters
        if (BEST) {
            cnt_inv += n_invalid;
            cnt_val += n_valid;
        } else {
            if (n_invalid) {
#pragma unroll
                for (int j = 0; j < RPT; j++) {
                    const unsigned long long i = tb + lane + 32 * j;
                    if (i < P.n && ws.rec_slot[lane + 32 * j] == -1) {
                        __stcs(P.h2d + i, 0ull);
                        __stcs(P.d2h + i, 0ull);
                        const double nan = __longlong_as_double(0x7ff8000000000000LL);
                        __stcs(P.t + i, nan);
                        if (P.p_iter) __stcs(P.p_iter + i, nan);
                        if (P.p_once) __stcs(P.p_once + i, nan);
                        if (P.p_h2d) __stcs(P.p_h2d + i, nan);
                        if (P.p_d2h) __stcs(P.p_d2h + i, nan);
                    }
                }
            }
            const unsigned tot = __reduce_add_sync(FULL, n_invalid);
            if (lane == 0 && tot) atomicAdd(S.invalid_counter, (unsigned long long)tot);
        }
}

// One design point's data usage from its residue class's byte polynomials
// (plan.cpp; internal.h layout): per array, H2D and D2H bytes and their
// Eq. (1) transfer times added in array order (N6).  AU arrays per step with
// every coefficient load of the step issued first (independent loads instead
// of one dependent round trip per array); polynomials that vanish in every
// class (pm bit clear) are not loaded: their bytes are 0 and their transfer
// adds +0.0 to a sum that is never -0.0, i.e. nothing (exact).
template <bool BIQ, int AU>
__device__ __forceinline__ void group_usage(const unsigned long long *pp, uint32_t stride,
                                            uint32_t n_arrays, uint32_t pm, uint32_t a8,
                                            uint32_t b8, const grophecy_pcie &pc,
                                            const unsigned long long *zero, Usage &u)
{
    constexpr int NQ = BIQ ? 5 : 2;   // 16-byte coefficient pairs per polynomial
    for (uint32_t a0 = 0; a0 < n_arrays; a0 += AU) {
        ulonglong2 c[AU][2][NQ];
#pragma unroll
        for (int i = 0; i < AU; i++)
#pragma unroll
            for (int dir = 0; dir < 2; dir++) {
                const uint32_t q = 2u * (a0 + (uint32_t)i) + (uint32_t)dir;
                const bool on = a0 + (uint32_t)i < n_arrays && ((pm >> q) & 1u);
                const ulonglong2 *src =
                    reinterpret_cast<const ulonglong2 *>(on ? pp + (size_t)q * stride : zero);
#pragma unroll
                for (int m = 0; m < NQ; m++) c[i][dir][m] = __ldg(src + m);
            }
        // arrays past n_arrays read the zero polynomial: 0 bytes, no term
#pragma unroll
        for (int i = 0; i < AU; i++) {
            unsigned long long v[2];
#pragma unroll
            for (int dir = 0; dir < 2; dir++) {
                const ulonglong2 *k = c[i][dir];
                unsigned long long e = k[0].x + k[0].y * a8 + (k[1].x + k[1].y * a8) * b8;
                if (BIQ)
                    e += (unsigned long long)a8 * (a8 * (k[2].x + b8 * (k[3].x + b8 * k[4].x))) +
                         (unsigned long long)b8 * (b8 * (k[2].y + a8 * k[3].y));
                v[dir] = e;
            }
            if (v[0]) u.th = __dadd_rn(u.th, __dadd_rn(pc.h2d.alpha_s,
                                                       __dmul_rn(pc.h2d.beta_s_per_byte, __ull2double_rn(v[0]))));
            if (v[1]) u.td = __dadd_rn(u.td, __dadd_rn(pc.d2h.alpha_s,
                                                       __dmul_rn(pc.d2h.beta_s_per_byte, __ull2double_rn(v[1]))));
            u.h += v[0];
            u.d += v[1];
        }
    }
}

// group_usage over the compact table (SkelInfo::poly32_base): one 16-byte
// load {c0, c1, c2, c3} (int32, the u64 coefficients sign-extended) per
// polynomial; evaluated with wrapping 64-bit arithmetic like the u64 table
// (the same residues mod 2^64, hence the same bytes).
template <int AU>
__device__ __forceinline__ void group_usage32(const int4 *pp, uint32_t n_arrays, uint32_t pm,
                                              uint32_t a8, uint32_t b8, const grophecy_pcie &pc,
                                              const int4 *zero, Usage &u)
{
    const long long a = (long long)a8, b = (long long)b8;
    for (uint32_t a0 = 0; a0 < n_arrays; a0 += AU) {
        int4 c[AU][2];
#pragma unroll
        for (int i = 0; i < AU; i++)
#pragma unroll
            for (int dir = 0; dir < 2; dir++) {
                const uint32_t q = 2u * (a0 + (uint32_t)i) + (uint32_t)dir;
                const bool on = a0 + (uint32_t)i < n_arrays && ((pm >> q) & 1u);
                c[i][dir] = __ldg(on ? pp + q : zero);
            }
        // arrays past n_arrays read the zero polynomial: 0 bytes, no term
        // (no early exit, so every load of the step is issued up front)
#pragma unroll
        for (int i = 0; i < AU; i++) {
            unsigned long long v[2];
#pragma unroll
            for (int dir = 0; dir < 2; dir++) {
                const int4 k = c[i][dir];
                const unsigned long long t = (unsigned long long)((long long)k.w * a + (long long)k.z);
                v[dir] = (unsigned long long)((long long)k.y * a + (long long)k.x) + t * (unsigned long long)b;
            }
            if (v[0]) u.th = __dadd_rn(u.th, __dadd_rn(pc.h2d.alpha_s,
                                                       __dmul_rn(pc.h2d.beta_s_per_byte, __ull2double_rn(v[0]))));
            if (v[1]) u.td = __dadd_rn(u.td, __dadd_rn(pc.d2h.alpha_s,
                                                       __dmul_rn(pc.d2h.beta_s_per_byte, __ull2double_rn(v[1]))));
            u.h += v[0];
            u.d += v[1];
        }
    }
}

// ---- 1-D bulk copies (TMA) global -> shared with mbarrier completion ----
__device__ __forceinline__ uint32_t smem_u32(const void *p)
{
    return (uint32_t)__cvta_generic_to_shared(p);
}

__device__ __forceinline__ void mbar_init(unsigned long long *bar, uint32_t count)
{
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}

__device__ __forceinline__ void mbar_wait(unsigned long long *bar, uint32_t phase)
{
    asm volatile(
        "{\n .reg .pred p;\n"
        "W%=:\n mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
        " @!p bra W%=;\n}" ::"r"(smem_u32(bar)),
        "r"(phase)
        : "memory");
}

// Lane 0 of a warp: copy the CTILE records of the tile at tb (full, 16-byte
// aligned) into ws.rec, completing on ws.mbar.  Earlier generic-proxy reads of
// ws.rec are ordered before the async-proxy writes by the fence.
__device__ __forceinline__ void issue_copy(const Params &P, uint32_t (*rec)[CTILE],
                                           unsigned long long *mbar, unsigned long long tb,
                                           uint32_t ng)   // design points (<= 32)
{
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    const uint32_t bar = smem_u32(mbar);
    const uint32_t bytes = ng * CX * (uint32_t)sizeof(uint32_t);   // per SoA array
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar),
                 "r"(4 * bytes)
                 : "memory");
    const uint32_t *src[4] = {P.skx, P.nx, P.ny, P.iters};
#pragma unroll
    for (int a = 0; a < 4; a++)
        asm volatile(
            "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                smem_u32(rec[a])),
            "l"(src[a] + tb), "r"(bytes), "r"(bar)
            : "memory");
}
__device__ __forceinline__ void issue_tile_copy(const Params &P, CanonSmem &ws, unsigned long long tb,
                                                uint32_t ng)
{
    issue_copy(P, ws.rec, &ws.mbar, tb, ng);
}

// One canonical tile: CTILE records from tb where every group of CX
// consecutive records (lane l: records tb + CX l ...) is one design point
// (same skeleton, nx, ny, iters; xform = position in the group, the layout
// of a skeleton x transformation x size sweep) and the whole tile has one
// skeleton.  Returns false, having written nothing, if the tile is not
// canonical (the caller then runs general tiles).  Lane l:
//   A  loads its group with 16-byte loads and checks it;
//   B  computes its key's usage from the byte polynomials (keys off the plan
//      path: the warp-cooperative sweep) and the kernels' work counts;
//   C  models its CX records, XW transformations per pass over the kernels
//      (the constants of (kernel, xform) are warp-uniform: one broadcast
//      load serves 32 records), then writes outputs / keeps its argmin.
template <bool BEST>
__device__ __forceinline__ bool canon_tile(const Params &P, CanonSmem &ws, uint32_t *cw,
                                           unsigned long long tb, uint32_t ng,
                                           unsigned long long next_tb, uint32_t next_ng, int lane,
                                           double &best_t, unsigned long long &best_i,
                                           uint32_t &cnt_val)
{
    const SpaceDev &S = P.S;
    // ---- A (records staged in ws.rec by the TMA; lane l reads its group's
    //      16-byte chunks in the rotated order c = (m + l/2) mod 4, which
    //      spreads 8 consecutive lanes over all 32 banks) ----
    uint32_t acc = 0, s0, n0, m0, i0;
    {
        const uint4 *p = reinterpret_cast<const uint4 *>(ws.rec[0] + lane * CX);
        const uint32_t r = ((uint32_t)lane >> 1) & 3u;
        uint4 v[CX / 4];
#pragma unroll
        for (int m = 0; m < CX / 4; m++) v[m] = p[(m + r) & 3u];
        // record 0's skx from the first chunk read: valid groups have
        // skx[q] = s0 ^ q with (s0 & 0xffff) == 0 (transformation q at q)
        s0 = v[0].x ^ (4u * r);
        acc = s0 & 0xffffu;
#pragma unroll
        for (int m = 0; m < CX / 4; m++) {
            const uint32_t c4 = 4u * ((m + r) & 3u);
            acc |= (v[m].x ^ s0) ^ (c4 + 0u);
            acc |= (v[m].y ^ s0) ^ (c4 + 1u);
            acc |= (v[m].z ^ s0) ^ (c4 + 2u);
            acc |= (v[m].w ^ s0) ^ (c4 + 3u);
        }
    }
    auto same = [&](int arr, uint32_t &first) {
        const uint4 *p = reinterpret_cast<const uint4 *>(ws.rec[arr] + lane * CX);
        const uint32_t r = ((uint32_t)lane >> 1) & 3u;
        uint4 v[CX / 4];
#pragma unroll
        for (int m = 0; m < CX / 4; m++) v[m] = p[(m + r) & 3u];
        first = v[0].x;
#pragma unroll
        for (int m = 0; m < CX / 4; m++)
            acc |= (v[m].x ^ first) | (v[m].y ^ first) | (v[m].z ^ first) | (v[m].w ^ first);
    };
    same(1, n0);
    same(2, m0);
    same(3, i0);
    // every read of ws.rec is consumed (acc): the buffer takes the next tile
    __syncwarp();
    if (lane == 0 && next_tb != ~0ull) issue_tile_copy(P, ws, next_tb, next_ng);
    // a partial tile (the batch's last ng < 32 design points): lanes past it
    // stand in for design point 0 in the warp-wide steps and output nothing
    {
        const uint32_t s00 = __shfl_sync(FULL, s0, 0), n00 = __shfl_sync(FULL, n0, 0);
        const uint32_t m00 = __shfl_sync(FULL, m0, 0), i00 = __shfl_sync(FULL, i0, 0);
        const uint32_t a00 = __shfl_sync(FULL, acc, 0);
        if ((uint32_t)lane >= ng) {
            s0 = s00;
            n0 = n00;
            m0 = m00;
            i0 = i00;
            acc = a00;
        }
    }
    const uint32_t skel = s0 >> 16;
    const uint32_t skel_l0 = __shfl_sync(FULL, skel, 0);   // (every lane: no short-circuit)
    bool ok = acc == 0 && skel < S.n_skels && n0 - 1u < GROPHECY_MAX_DIM &&
              m0 - 1u < GROPHECY_MAX_DIM && i0 >= 1 && skel == skel_l0;
    if (ok) ok = S.skel[skel].n_xforms >= (uint32_t)CX && (S.skel[skel].flags & SKF_TABULATED);
    if (!__all_sync(FULL, ok)) return false;

    // ---- B ----
    const SkelInfo &I = S.skel[skel];   // warp-uniform from here on
    const uint32_t K = I.n_kernels, n_arrays = I.n_arrays;
    const long long nxny = (long long)((unsigned long long)n0 * m0);
    bool huge = false;
    for (uint32_t k = 0; k < K; k++) {
        const uint32_t w = w_store(aff8n(__ldg(&S.kern_work[I.k_base + k]), (int)n0, (int)m0, nxny));
        cw[k * 32 + (lane & 1) * 16 + (lane >> 1)] = w;
        huge |= w == W_HUGE;
    }
    if (__any_sync(FULL, huge)) return false;   // (nothing written yet)
    // keys off the plan path (small sizes, strided, hull): general tiles
    if (!__all_sync(FULL, n0 >= I.plan_tx && m0 >= I.plan_ty)) return false;
    {
        Usage u = {0ull, 0ull, 0.0, 0.0};
        const uint32_t stride = I.poly_stride, a8 = n0 >> 3, b8 = m0 >> 3;
        const unsigned long long *pp =
            S.poly + I.poly_base + (size_t)((n0 & 7u) * 8u + (m0 & 7u)) * (2u * n_arrays * stride);
        // skipped polynomials vanish in every class: their transfers add +0.0
        // to a sum that is never -0.0, i.e. nothing (exact)
        const uint32_t pm = I.poly_mask;
        if (I.poly32_base != POLY32_NONE)
            group_usage32<GROPHECY_AU32>(reinterpret_cast<const int4 *>(S.poly + I.poly32_base) +
                                             (size_t)((n0 & 7u) * 8u + (m0 & 7u)) * (2u * n_arrays),
                                         n_arrays, pm, a8, b8, P.pc,
                                         reinterpret_cast<const int4 *>(S.poly), u);
        else if (stride > 4) group_usage<true, 2>(pp, stride, n_arrays, pm, a8, b8, P.pc, S.poly, u);
        else group_usage<false, 4>(pp, stride, n_arrays, pm, a8, b8, P.pc, S.poly, u);
        const int q = (lane & 1) * 16 + (lane >> 1);
        ws.th[q] = u.th;
        ws.td[q] = u.td;
        ws.uh[q] = u.h;
        ws.ud[q] = u.d;
        ws.it[q] = (double)i0;
    }
    __syncwarp();
    // ---- C: lane = (transformation x, half h); groups g = 2 i + h ----
    const uint32_t X = I.n_xforms, pim = I.per_iter_mask;
    const uint32_t x = (uint32_t)lane & (CX - 1), h = (uint32_t)lane / CX;
    const KxFast *F0 = S.kx_f + I.kx_base + x;
    const uint32_t xf = __ldg(&S.xinf[I.kx_base + x]);
#pragma unroll 1
    for (int i0g = 0; i0g < 32 / 2; i0g += CG) {
        double ti[CG], to[CG];
#pragma unroll
        for (int j = 0; j < CG; j++) ti[j] = to[j] = 0.0;
        // the kernels of one sum (bit k of `mask`) in ascending k: this lane's
        // (kernel, transformation) constants, the 8 groups' work counts, the
        // saturated model, small grids from the table, the sum (N6)
        auto one_kernel = [&](uint32_t k, double (&acc)[CG]) {
            const uint32_t kxi = I.kx_base + x + k * X;
            const KxFast f = F0[(size_t)k * X];
            const uint32_t sat = f.satsh & KXF_SAT_MASK, sh = f.satsh >> KXF_SAT_BITS;
            uint32_t w[CG];
#pragma unroll
            for (int j = 0; j < CG; j += 4) {
                const uint4 v = *reinterpret_cast<const uint4 *>(&cw[k * 32 + h * 16 + i0g + j]);
                w[j] = v.x;
                w[j + 1] = v.y;
                w[j + 2] = v.z;
                w[j + 3] = v.w;
            }
            double tk[CG];
            bool gen[CG], any = false;
            uint32_t blocks[CG];
#pragma unroll
            for (int j = 0; j < CG; j++) {
                tk[j] = fast_time(f, sat, sh, w[j], S.rfh, S.rfl, gen[j], blocks[j]);
                any |= gen[j];
            }
            if (any) {
                // off the saturated path: the small-grid table (SKF_TABULATED:
                // blocks < sat <= small_stride; infeasible pairs never get
                // here); this pair's table row (32-bit element offset) once
                unsigned long long row;
                asm volatile("mad.wide.u32 %0, %1, 8, %2;"
                             : "=l"(row)
                             : "r"(kxi * S.small_stride), "l"(S.small_t));
#pragma unroll
                for (int j = 0; j < CG; j++)
                    if (gen[j]) tk[j] = __ldg(reinterpret_cast<const double *>(row) + blocks[j]);
            }
#pragma unroll
            for (int j = 0; j < CG; j++) acc[j] = __dadd_rn(acc[j], tk[j]);
        };
        // the kernels of one sum (bit k of `mask`) in ascending k: this lane's
        // (kernel, transformation) constants, the 8 groups' work counts, the
        // saturated model, small grids from the table, the sum (N6)
        auto kernel_sum = [&](uint32_t mask, double (&acc)[CG]) {
#pragma unroll 1
            for (; mask; mask &= mask - 1u) one_kernel((uint32_t)__ffs(mask) - 1u, acc);
        };
        const uint32_t kmask = K == 32 ? 0xffffffffu : (1u << K) - 1u;
        kernel_sum(pim & kmask, ti);                       // t_iter
        if (~pim & kmask) kernel_sum(~pim & kmask, to);    // t_once
        // infeasible kernels: that sum is +inf (exact, see xinf)
        const double inf = __longlong_as_double(0x7ff0000000000000LL);
        if (xf & XINF_ITER) {
#pragma unroll
            for (int j = 0; j < CG; j++) ti[j] = inf;
        }
        if (xf & XINF_ONCE) {
#pragma unroll
            for (int j = 0; j < CG; j++) to[j] = inf;
        }
        // totals: run-once + iters x per-iteration +
        // transfers.  Without run-once kernels t_once = +0.0 and
        // +0.0 + iters * t_iter = iters * t_iter exactly (both >= +0).
        const bool once = pim != (K == 32 ? 0xffffffffu : (1u << K) - 1u) || (xf & XINF_ONCE);
        double cm = __longlong_as_double(0x7ff0000000000000LL);
        int cj = -1;
        // this chunk's per-group values: consecutive in the permuted layout
        const int q0 = (int)h * 16 + i0g;
        double itv[CG], thv[CG], tdv[CG];
#pragma unroll
        for (int j = 0; j < CG; j += 2) {
            const double2 a = *reinterpret_cast<const double2 *>(&ws.it[q0 + j]);
            const double2 b = *reinterpret_cast<const double2 *>(&ws.th[q0 + j]);
            const double2 c = *reinterpret_cast<const double2 *>(&ws.td[q0 + j]);
            itv[j] = a.x; itv[j + 1] = a.y;
            thv[j] = b.x; thv[j + 1] = b.y;
            tdv[j] = c.x; tdv[j + 1] = c.y;
        }
        auto totals = [&](auto ONCE) {
#pragma unroll
            for (int j = 0; j < CG; j++) {
                const uint32_t g = 2u * (uint32_t)(i0g + j) + h;
                double tk = __dmul_rn(itv[j], ti[j]);
                if constexpr (decltype(ONCE)::value) tk = __dadd_rn(to[j], tk);
                const double tt = __dadd_rn(__dadd_rn(tk, thv[j]), tdv[j]);
                if (g >= ng) continue;   // past a partial tile
                if (BEST) {
                    // the lane's records come in increasing index order (tiles,
                    // chunks, j): strict < keeps the lowest index among ties
                    if (tt < cm) {
                        cm = tt;
                        cj = j;
                    }
                } else {
                    const unsigned long long r = tb + (unsigned long long)g * CX + x;
                    __stcs(P.h2d + r, ws.uh[q0 + j]);
                    __stcs(P.d2h + r, ws.ud[q0 + j]);
                    __stcs(P.t + r, tt);
                    if (P.p_iter) __stcs(P.p_iter + r, ti[j]);
                    if (P.p_once) __stcs(P.p_once + r, to[j]);
                    if (P.p_h2d) __stcs(P.p_h2d + r, thv[j]);
                    if (P.p_d2h) __stcs(P.p_d2h + r, tdv[j]);
                }
            }
        };
        if (once) totals(std::true_type{});
        else totals(std::false_type{});
        if (BEST && cm < best_t) {
            const uint32_t g = 2u * (uint32_t)(i0g + cj) + h;
            best_t = cm;
            best_i = P.base + tb + (unsigned long long)g * CX + x;
            ws.best_h[lane] = ws.uh[q0 + cj];
            ws.best_d[lane] = ws.ud[q0 + cj];
        }
    }
    if (BEST && (uint32_t)lane < ng) cnt_val += CX;
    __syncwarp();
    return true;
}
// Block-level epilogue of best mode: warp -> CTA -> grid argmin (last-block
// pattern; the last block also resets the ticket for reuse).
template <int NW = WARPS>   // warps per CTA
__device__ __forceinline__ void finish_best(const Params &P, const unsigned long long *best_h,
                                            const unsigned long long *best_d, int lane, int warp,
                                            double best_t, unsigned long long best_i,
                                            uint32_t cnt_inv, uint32_t cnt_val,
                                            unsigned nblocks)   // blocks taking part
{
    __shared__ Best wbest[NW];
    __shared__ bool am_last;
    // ---- argmin: warp -> CTA -> grid (last-block pattern) ----
    Best mine;
    mine.t = best_t;
    mine.i = best_i;
    mine.h = best_h[lane];
    mine.d = best_d[lane];
    mine.ninv = cnt_inv;
    mine.nval = cnt_val;
    mine = warp_best(mine);
    if (lane == 0) wbest[warp] = mine;
    __syncthreads();
    if (warp == 0) {
        Best b = lane < NW ? wbest[lane] : none_best();
        b = warp_best(b);
        if (lane == 0) {
            to_result(P.partials[blockIdx.x], b);
            __threadfence();
            const unsigned prev = atomicAdd(P.ticket, 1u);
            am_last = prev == nblocks - 1;
        }
    }
    __syncthreads();
    if (!am_last) return;
    __threadfence();
    if (warp == 0) {
        Best b = none_best();
        for (unsigned j = lane; j < nblocks; j += 32) {
            grophecy_best_result r;
            const volatile grophecy_best_result *pr = P.partials + j;
            r.t_total_s = pr->t_total_s;
            r.index = pr->index;
            r.h2d_bytes = pr->h2d_bytes;
            r.d2h_bytes = pr->d2h_bytes;
            r.n_invalid = pr->n_invalid;
            r.n_valid = pr->n_valid;
            merge(b, from_result(r));
        }
        b = warp_best(b);
        if (lane == 0) {
            if (P.map_len && b.i != ~0ull)   // striped batch: local -> global index
                b.i = P.map_base + (b.i / P.map_len) * P.map_stride + b.i % P.map_len;
            if (P.accumulate) {
                Best prev = from_result(*P.out);
                merge(prev, b);
                b = prev;
            }
            to_result(*P.out, b);
            *P.ticket = 0u;
            if (P.reset_counters) {   // pass 2 of best mode: every claim is done
                P.tile_count[0] = 0u;
                P.tile_count[CLAIM1] = 0u;
                P.tile_count[CLAIM2] = 0u;
            }
        }
    }
}

// Pass 1 of a projection (persistent): every tile of CTILE records that is
// canonical is projected here; the others (and the ragged tail) are appended
// to the space's tile list for pass 2.
template <bool BEST>
__global__ void __launch_bounds__(THREADS, GROPHECY_CMINB) canon_kernel(const Params P)
{
    extern __shared__ __align__(16) unsigned char smem_raw[];
    const int lane = threadIdx.x & 31;
    const int warp = threadIdx.x >> 5;
    unsigned char *wbase = smem_raw + (size_t)warp * P.canon_warp_bytes;
    CanonSmem &ws = *reinterpret_cast<CanonSmem *>(wbase);
    uint32_t *cw = reinterpret_cast<uint32_t *>(wbase + sizeof(CanonSmem));
    // running argmin kept lean in registers: (t, index) + counters; the
    // winner's byte counts go to shared memory (rarely updated)
    double best_t = __longlong_as_double(0x7ff0000000000000LL);
    unsigned long long best_i = ~0ull;
    uint32_t cnt_val = 0;
    ws.best_h[lane] = 0;
    ws.best_d[lane] = 0;
    const unsigned long long ntiles = (P.n + CTILE - 1) / CTILE;
    const unsigned long long wstride = (unsigned long long)gridDim.x * WARPS;
    // full tiles of 16-byte aligned records are staged in shared memory by
    // the TMA one tile ahead (the copy of the next tile overlaps phases B and
    // C of this one); the others go to the general path directly
    // design points a tile stages: 32, or the batch's last ng whole design
    // points (n - tb a multiple of 16); 0 = not for pass 1
    auto groups = [&](unsigned long long t) -> uint32_t {
        if (!P.aligned || P.pr.mem) return 0u;
        const unsigned long long tb = t * CTILE;
        if (tb + CTILE <= P.n) return (uint32_t)(CTILE / CX);
        const unsigned long long rest = P.n - tb;
        return rest % CX == 0 ? (uint32_t)(rest / CX) : 0u;
    };
    if (lane == 0) mbar_init(&ws.mbar, 1);
    __syncwarp();
    uint32_t phase = 0;
    // first tile: blockIdx.x * WARPS + warp; then each warp claims its next
    // tile from a counter (P.tile_count[CLAIM1], zeroed before the launch) one
    // tile ahead, so that the TMA copy still overlaps this tile's phases B
    // and C and the warps finish together although tile costs differ by
    // skeleton.  One warp's claims increase (argmin tie order, see totals).
    unsigned *claim = P.tile_count + CLAIM1;
    const unsigned long long t0 = (unsigned long long)blockIdx.x * WARPS + warp;
    if (lane == 0 && t0 < ntiles && groups(t0)) issue_tile_copy(P, ws, t0 * CTILE, groups(t0));
#pragma unroll 1
    for (unsigned long long tile = t0, nt; tile < ntiles; tile = nt) {
        {
            unsigned long long v = 0;
            if (lane == 0) v = (unsigned long long)atomicAdd(claim, 1u) + wstride;
            nt = __shfl_sync(FULL, v, 0);
        }
        const unsigned long long tb = tile * CTILE;
        const uint32_t ng = groups(tile), next_ng = nt < ntiles ? groups(nt) : 0u;
        const unsigned long long next_tb = next_ng ? nt * CTILE : ~0ull;
        bool done = false;
        if (ng) {   // (the memory choice, P.pr.mem, is priced by the general path only)
            mbar_wait(&ws.mbar, phase);
            phase ^= 1u;
            done = canon_tile<BEST>(P, ws, cw, tb, ng, next_tb, next_ng, lane, best_t, best_i,
                                    cnt_val);
        } else if (lane == 0 && next_tb != ~0ull) {
            issue_tile_copy(P, ws, next_tb, next_ng);   // the buffer is idle during this tile
        }
        if (!done && lane == 0) P.tile_list[atomicAdd(P.tile_count, 1u)] = (uint32_t)tile;
    }
    if (BEST) finish_best(P, ws.best_h, ws.best_d, lane, warp, best_t, best_i, 0u, cnt_val, gridDim.x);
}

// ---- Sweep tiles: pass 1 of best mode ----
// A CTA tile is WARPS canonical warp tiles of one skeleton: 32 * WARPS design
// points x CX transformations (4096 records).  Phases A/B run per warp with
// lane = design point (as canon_tile: TMA-staged records, checks, work
// counts, byte polynomials, Eq. (1) pricing) and leave each design point's
// work counts and transfer terms in CTA shared memory; after a barrier, phase
// C is CTA-wide: a warp claims a transformation x and its lanes model x for
// NCH design points each (groups 32 j + lane), so the (kernel, x) constants
// and their class (internal.h KxCls) are warp-uniform and every lane runs
// NCH independent chains of the class-specialised saturated model:
// infeasible kernels are skipped (their sum is +inf through xinf), power-of-
// two denominators and S = 0 drop their multiplications, and both divisions
// take the two-product form.  CTA tiles that are not uniform (a skeleton
// boundary, any other layout) and the batch's tail go to pass 2.
constexpr int SW_GROUPS = 32 * WARPS;                               // design points per CTA tile
constexpr unsigned long long SW_TILE = (unsigned long long)SW_GROUPS * CX;   // records per CTA tile
// chains per lane: a phase-C unit covers the tile's 256 design points (lane l,
// chain j: design point 32 j + l, i.e. chain j = warp tile j)
constexpr int NCH = WARPS;

constexpr uint32_t SW_BAD = 0xffffffffu, SW_EMPTY = 0xfffffffeu;
#ifndef GROPHECY_SMINB
#define GROPHECY_SMINB 2
#endif
#ifndef GROPHECY_XINF_SKIP
#define GROPHECY_XINF_SKIP 1
#endif
#ifndef GROPHECY_I2F_MAGIC
#define GROPHECY_I2F_MAGIC 0
#endif
#ifndef GROPHECY_DISPATCH_TREE
#define GROPHECY_DISPATCH_TREE 1   // class dispatch by uniform branches (0: switch)
#endif
#ifndef GROPHECY_FUSED
#define GROPHECY_FUSED 1
#endif
#ifndef GROPHECY_PERM
#define GROPHECY_PERM 1
#endif
// GROPHECY_PHASE_TIMING=1 (diagnostic builds only): per-warp clock64 time per
// phase of the sweep kernel, summed into g_phase_cycles and read back by
// grophecy_debug_phase_cycles (scripts/phase_timing.py)
#ifndef GROPHECY_PHASE_TIMING
#define GROPHECY_PHASE_TIMING 0
#endif
#if GROPHECY_PHASE_TIMING
__device__ unsigned long long g_phase_cycles[8];
#define PT_MARK(slot)                                                              \
    do {                                                                           \
        const long long t_ = clock64();                                            \
        if (lane == 0) atomicAdd(&g_phase_cycles[slot], (unsigned long long)(t_ - pt_last)); \
        pt_last = t_;                                                              \
    } while (0)
#else
#define PT_MARK(slot) do { } while (0)
#endif

constexpr int SW_NB = 2;   // buffers of the per-design-point phase-B results (tiles r, r + 1)
struct alignas(128) SweepSmem {
    alignas(128) uint32_t rec[4][SW_TILE];   // the CTA tile's SoA records (4 TMA bulk copies)
    unsigned long long rbar;     // completion of the record copies (phase = the tile's sequence number & 1)
    unsigned long long tbar[2];  // usage-table decision of the tile of sequence parity p (TMA or plain arrive)
    unsigned long long abar[2];  // the WARPS A/B tasks of the tile of sequence parity p are done
    unsigned long long cbar[2];  // every warp's phase C of the tile of sequence parity p is done
    // per buffer b (the tile of sequence parity b), design point g = 32 * (A/B task) + lane
    alignas(16) double2 thd[SW_NB][SW_GROUPS];   // {t_h2d, t_d2h}: one 16-byte read in the totals
    double it[SW_NB][SW_GROUPS];                 // iterations
    uint32_t smallw[SW_NB][WARPS];       // per warp tile: work slots whose grid may be unsaturated
    uint32_t wstat[SW_NB][WARPS];        // A/B result per warp tile: its skeleton, SW_BAD or SW_EMPTY
    uint32_t perm[SW_NB][CX];            // the tile's skx at each position of a design point (its first one's)
    uint32_t perm_ident[SW_NB];          // perm is the identity (units follow the cost order)
    uint32_t perm_ok[SW_NB];             // the tile's first design point is consistent
    uint4 uhdr[SW_NB][CX];               // per phase-C unit: its program header (xhdr layout) ...
    uint32_t upos[SW_NB][CX];            // ... and its position in the design points
    uint4 tinf[SW_NB];                   // the tile's skeleton: {kx_base, n_xforms, has run-once kernels, -}
    uint32_t wsk[SW_NB][WARPS];          // (TWO) per warp tile: its design points' other skeleton, or SW_BAD
    uint8_t dsk[SW_NB][SW_GROUPS];       // (TWO) per design point: 1 = the tile's second skeleton
    uint32_t ab_cnt[4];                  // A/B task claims of the tile of sequence number mod 4
    uint32_t a_done[2];                  // phase-A completions of the tile of sequence parity p
    uint32_t tile_id[4];                 // the CTA's tiles by sequence number mod 4 (claimed ahead)
    uint32_t tbl_skel;                   // skeleton whose usage table is staged (SW_BAD: none)
};
// followed by the work counts cw[b][j][lane][8] (uint32, w_store; buffer b,
// work slot j; design point g = 32 t + lane at chunk (t / 4) ^ ((lane / 4) & 1),
// so a phase-C lane reads its chains with two conflict-free 16-byte loads),
// sized by the space's largest work-slot count, then the staged usage table
// (SkelInfo::polyf_base)
__host__ __device__ constexpr uint32_t sweep_cw_offset() { return (uint32_t)((sizeof(SweepSmem) + 127) / 128 * 128); }
__host__ __device__ constexpr uint32_t sweep_tbl_offset(uint32_t wmax)
{
    return sweep_cw_offset() + (uint32_t)SW_NB * wmax * (uint32_t)SW_GROUPS * (uint32_t)sizeof(uint32_t);
}
__host__ __device__ constexpr uint32_t sweep_smem_bytes(uint32_t wmax, uint32_t tbl_bytes)
{
    return sweep_tbl_offset(wmax) + tbl_bytes;
}
__device__ __forceinline__ uint32_t cw_index(uint32_t k, uint32_t lane, uint32_t j)
{
    return k * (uint32_t)SW_GROUPS + lane * 8u + ((((j >> 2) ^ (lane >> 2)) & 1u) << 2) + (j & 3u);
}

// group_usage over the staged table (shared memory, [q][class]; SkelInfo::
// polyf_base): the non-zero H2D polynomials in array order, then the D2H
// ones, per polynomial one 16-byte load {c0, c1, c2, c3} (int32: the u64
// coefficients sign-extended), bytes = c0 + c1 a + c2 b + (c3 a) b in wrapping
// 64-bit arithmetic (the same residue mod 2^64 as the u64 table, hence the
// same bytes), priced by Eq. (1) and summed in array order per direction
// (the skipped polynomials are zero: they price and add nothing).
template <bool U32>   // every partial sum below 2^32: 32-bit wrapping evaluation (exact)
__device__ __forceinline__ void group_usage_s(const int4 *pp, uint32_t nhd, uint32_t a8, uint32_t b8,
                                              const grophecy_pcie &pc, Usage &u)
{
    const int a = (int)a8, b = (int)b8;
    const uint32_t ab = a8 * b8;
    auto run = [&](uint32_t n, const grophecy_link &lk, double &tsum, unsigned long long &bsum) {
        for (uint32_t q0 = 0; q0 < n; q0 += POLYF_AU, pp += POLYF_AU * POLY_CLASSES) {
            int4 c[POLYF_AU];
#pragma unroll
            for (int q = 0; q < (int)POLYF_AU; q++) c[q] = pp[q * POLY_CLASSES];
#pragma unroll
            for (int q = 0; q < (int)POLYF_AU; q++) {
                const int4 k = c[q];
                if (U32) {
                    const uint32_t v = (uint32_t)k.x + (uint32_t)k.y * a8 + (uint32_t)k.z * b8 + (uint32_t)k.w * ab;
                    if (v) tsum = __dadd_rn(tsum, __dadd_rn(lk.alpha_s, __dmul_rn(lk.beta_s_per_byte, __uint2double_rn(v))));
                    bsum += v;
                } else {
                    const long long s1 = (long long)k.y * a + (long long)k.x + (long long)k.z * b;
                    const unsigned long long t = (unsigned long long)((long long)k.w * a);
                    const unsigned long long v = (unsigned long long)s1 + t * (unsigned long long)(unsigned)b;
                    if (v) tsum = __dadd_rn(tsum, __dadd_rn(lk.alpha_s, __dmul_rn(lk.beta_s_per_byte, __ull2double_rn(v))));
                    bsum += v;
                }
            }
        }
    };
    run(nhd & 0xffffu, pc.h2d, u.th, u.h);
    run(nhd >> 16, pc.d2h, u.td, u.d);
}

// CTA tile copy (thread 0): the 4 SoA arrays' SW_TILE records from tb into
// sm.rec, completing on sm.rbar.  Every generic-proxy read of sm.rec by the
// CTA happened before the caller's barrier; the fence orders them before the
// async-proxy writes.
template <unsigned long long SWT>   // records per CTA tile
__device__ __forceinline__ void issue_cta_copy(const Params &P, uint32_t (*rec)[SW_TILE],
                                               unsigned long long *rbar, unsigned long long tb)
{
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    const uint32_t bar = smem_u32(rbar);
    // a full tile, or the batch's last one (a whole number of design points)
    const unsigned long long nrec = P.n - tb < SWT ? P.n - tb : SWT;
    const uint32_t bytes = (uint32_t)(nrec * sizeof(uint32_t));
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(4 * bytes)
                 : "memory");
    const uint32_t *src[4] = {P.skx, P.nx, P.ny, P.iters};
#pragma unroll
    for (int a = 0; a < 4; a++)
        asm volatile(
            "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                smem_u32(rec[a])),
            "l"(src[a] + tb), "r"(bytes), "r"(bar)
            : "memory");
}

// Phase A of one warp tile of the CTA tile staged at recs: lane l reads its
// design point's 16 records (rotated 16-byte chunks, conflict-free) and
// checks the layout of a sweep: every design point of the CTA tile holds CXT
// records of one skeleton with equal nx, ny, iters, and the transformations
// in the same order as the tile's first design point (any fixed order of
// valid transformations); warp-uniform result.  The batch's last warp tile
// may hold gw < 32 design points: lanes past it stand in for design point 0.
// A design point that differs from the tile's first in its skx: equal
// transformations record by record and one skeleton for all its records
// (which may be another than the first design point's: a tile's second
// skeleton, sweep_kernel<.., TWO>).  Out of line: rare.
template <int NCK>
__device__ __noinline__ uint32_t skx_relaxed(const uint4 *p, const uint4 *g, uint32_t r)
{
    uint32_t acc = 0, D = 0;
#pragma unroll
    for (int m = 0; m < NCK; m++) {
        const uint4 v = p[(m + r) & (uint32_t)(NCK - 1)], w = g[(m + r) & (uint32_t)(NCK - 1)];
        if (m == 0) D = (v.x ^ w.x) & 0xffff0000u;
        acc |= (v.x ^ w.x ^ D) | (v.y ^ w.y ^ D) | (v.z ^ w.z ^ D) | (v.w ^ w.w ^ D);
    }
    return acc;
}

template <int CXT, bool TWO, unsigned long long ROW>   // design-point size; two skeletons; staged length
__device__ __forceinline__ bool sweep_phase_a(const SpaceDev &S, const uint32_t (*recs)[ROW], int warp,
                                              int lane, uint32_t gw, uint32_t &s0, uint32_t &n0, uint32_t &m0,
                                              uint32_t &i0)
{
    constexpr int NCK = CXT / 4;                   // 16-byte chunks per design point and array
    constexpr uint32_t CTW = 32u * (uint32_t)CXT;   // records per warp tile
    const uint32_t *rec[4] = {recs[0] + warp * CTW, recs[1] + warp * CTW, recs[2] + warp * CTW,
                              recs[3] + warp * CTW};
    uint32_t acc;
    // rotated chunk order: the 16-byte reads of a quarter warp hit distinct banks
    const uint32_t r = NCK == 4 ? ((uint32_t)lane >> 1) & 3u : (NCK == 2 ? ((uint32_t)lane >> 2) & 1u : 0u);
    {
        const uint4 *p = reinterpret_cast<const uint4 *>(rec[0] + lane * CXT);
#if GROPHECY_PERM
        const uint4 *g = reinterpret_cast<const uint4 *>(recs[0]);   // the tile's first design point
        uint4 v[NCK], w[NCK];
#pragma unroll
        for (int m = 0; m < NCK; m++) {
            v[m] = p[(m + r) & (uint32_t)(NCK - 1)];
            w[m] = g[(m + r) & (uint32_t)(NCK - 1)];
        }
        s0 = v[0].x;
        acc = 0;
        // equal to the tile's first design point record by record (whose own
        // consistency — one skeleton, valid transformations — warp 0 checks
        // once per tile: SweepSmem::perm_ok)
#pragma unroll
        for (int m = 0; m < NCK; m++)
            acc |= (v[m].x ^ w[m].x) | (v[m].y ^ w[m].y) | (v[m].z ^ w[m].z) | (v[m].w ^ w[m].w);
        if (TWO && acc) acc = skx_relaxed<NCK>(p, g, r);   // (a second skeleton's design point)
#else
        uint4 v[NCK];
#pragma unroll
        for (int m = 0; m < NCK; m++) v[m] = p[(m + r) & (uint32_t)(NCK - 1)];
        s0 = v[0].x ^ (4u * r);
        acc = s0 & 0xffffu;
#pragma unroll
        for (int m = 0; m < NCK; m++) {
            const uint32_t c4 = 4u * ((m + r) & (uint32_t)(NCK - 1));
            acc |= (v[m].x ^ s0) ^ (c4 + 0u);
            acc |= (v[m].y ^ s0) ^ (c4 + 1u);
            acc |= (v[m].z ^ s0) ^ (c4 + 2u);
            acc |= (v[m].w ^ s0) ^ (c4 + 3u);
        }
#endif
    }
    auto same = [&](int arr, uint32_t &first) {
        const uint4 *p = reinterpret_cast<const uint4 *>(rec[arr] + lane * CXT);
        uint4 v[NCK];
#pragma unroll
        for (int m = 0; m < NCK; m++) v[m] = p[(m + r) & (uint32_t)(NCK - 1)];
        first = v[0].x;
#pragma unroll
        for (int m = 0; m < NCK; m++)
            acc |= (v[m].x ^ first) | (v[m].y ^ first) | (v[m].z ^ first) | (v[m].w ^ first);
    };
    same(1, n0);
    same(2, m0);
    same(3, i0);
    if (gw < 32u) {   // (warp-uniform: the batch's last warp tile)
        const uint32_t a0 = __shfl_sync(FULL, acc, 0), s00 = __shfl_sync(FULL, s0, 0);
        const uint32_t n00 = __shfl_sync(FULL, n0, 0), m00 = __shfl_sync(FULL, m0, 0);
        const uint32_t i00 = __shfl_sync(FULL, i0, 0);
        if ((uint32_t)lane >= gw) {
            acc = a0;
            s0 = s00;
            n0 = n00;
            m0 = m00;
            i0 = i00;
        }
    }
    // (acc == 0 in every lane: every record equals the tile's first design
    // point's in skx, so the warp tile has one skeleton)
    const uint32_t skel = s0 >> 16;
    bool ok = acc == 0 && skel < S.n_skels && n0 - 1u < GROPHECY_MAX_DIM &&
              m0 - 1u < GROPHECY_MAX_DIM && i0 >= 1;
    if (ok) ok = (S.skel[skel].flags & SKF_TABULATED) != 0;
    return __all_sync(FULL, ok);
}

// Saturated kernel times of NCH records of one (kernel, x) pair of class C
// (internal.h KxProg) from their block counts; t = cyc / freq by the
// two-product division.
template <uint32_t C>
__device__ __forceinline__ void cls_times(const double2 c01, const double2 c23, const uint32_t (&blocks)[NCH],
                                          double rfh, double rfl, double (&tk)[NCH])
{
#pragma unroll
    for (int j = 0; j < NCH; j++) {
#if GROPHECY_I2F_MAGIC
        // (2^52 + blocks) - 2^52 on the fp64 pipe: exact for blocks < 2^52
        const double bb = __dadd_rn(__hiloint2double(0x43300000, (int)blocks[j]), -0x1p52);
#else
        const double bb = __uint2double_rn(blocks[j]);
#endif
        double cyc;
        if (C == KXC_P2S0) {
            cyc = __dmul_rn(bb, c01.x);
        } else if (C == KXC_P2S) {
            cyc = __dadd_rn(__dmul_rn(bb, c01.x), __dmul_rn(bb, c01.y));
        } else {
            const double rep = __fma_rn(bb, c01.x, __dmul_rn(bb, c01.y));
            cyc = __dmul_rn(c23.x, rep);
            if (C == KXC_NS) cyc = __dadd_rn(cyc, __dmul_rn(c23.y, rep));
        }
        tk[j] = __fma_rn(cyc, rfh, __dmul_rn(cyc, rfl));
    }
}

// Transfer bytes of a design point (skeleton I, nx, ny) on the sweep path:
// phase B's evaluation read from the global copy of the tables (the staged
// one may already hold the next tile's).  Only for a lane's new running best.
__device__ __noinline__ void sweep_bytes(const unsigned long long *poly, const grophecy_pcie pc, const SkelInfo *Ip,
                                         uint32_t n0, uint32_t m0, unsigned long long *hd)
{
    const SkelInfo &I = *Ip;
    Usage u = {0ull, 0ull, 0.0, 0.0};
    const uint32_t n_arrays = I.n_arrays, stride = I.poly_stride, a8 = n0 >> 3, b8 = m0 >> 3;
    const uint32_t cls = (n0 & 7u) * 8u + (m0 & 7u), pm = I.poly_mask;
    if (I.polyf_base != POLY32_NONE) {
        const int4 *tg = reinterpret_cast<const int4 *>(poly + I.polyf_base);
        const unsigned long long bnd = (unsigned long long)I.polyf_cmax[0] +
                                       (unsigned long long)I.polyf_cmax[1] * a8 +
                                       (unsigned long long)I.polyf_cmax[2] * b8 +
                                       (unsigned long long)I.polyf_cmax[3] * ((unsigned long long)a8 * b8);
        if (bnd < (1ull << 32))
            group_usage_s<true>(tg + cls, I.polyf_nhd, a8, b8, pc, u);
        else
            group_usage_s<false>(tg + cls, I.polyf_nhd, a8, b8, pc, u);
    } else if (I.poly32_base != POLY32_NONE) {
        group_usage32<GROPHECY_AU32>(reinterpret_cast<const int4 *>(poly + I.poly32_base) +
                                         (size_t)cls * (2u * n_arrays),
                                     n_arrays, pm, a8, b8, pc, reinterpret_cast<const int4 *>(poly), u);
    } else if (stride > 4) {
        group_usage<true, 2>(poly + I.poly_base + (size_t)cls * (2u * n_arrays * stride), stride, n_arrays, pm,
                             a8, b8, pc, poly, u);
    } else {
        group_usage<false, 4>(poly + I.poly_base + (size_t)cls * (2u * n_arrays * stride), stride, n_arrays, pm,
                              a8, b8, pc, poly, u);
    }
    hd[0] = u.h;
    hd[1] = u.d;
}

// The sweep kernel works in rounds: in round r a warp runs its phase-C units
// of the CTA's tile r (phase-B results in buffer r & 1), then claims phase
// A/B tasks of tile r + 1 (one per warp tile, buffer (r + 1) & 1) from a
// shared counter, so a transformation-poor tile's idle warps prepare the next
// tile instead of waiting.  No CTA barrier: per-tile mbarriers order the
// phases (abar: tile r's A/B tasks done -> its phase C; cbar: every warp's
// phase C of tile r - 1 done -> the A/B tasks of tile r + 1 reuse its
// buffer; rbar: records staged; tbar: usage-table decision).  The last warp
// to finish phase A of a tile issues the TMA copy of the CTA's next tile
// into the (single) record buffer.
template <bool BEST, int CXT, bool TWO>   // CXT: records per design point (4, 8 or 16); TWO: a
                                          // tile may hold two skeletons
__global__ void __launch_bounds__(THREADS, GROPHECY_SMINB) sweep_kernel(const Params P)
{
    static_assert(CXT == 4 || CXT == 8 || CXT == 16, "design-point sizes of the sweep");
    constexpr unsigned long long SWT = (unsigned long long)SW_GROUPS * CXT;   // records per CTA tile
    constexpr unsigned UNITS = (unsigned)CXT * (WARPS / NCH);                // phase-C units
    constexpr unsigned CPT = (unsigned)(SWT / CTILE);                        // pass-2 chunks per CTA tile
    extern __shared__ __align__(16) unsigned char smem_raw[];
    SweepSmem &sm = *reinterpret_cast<SweepSmem *>(smem_raw);
    const uint32_t wmax = P.sweep_kmax;
    uint32_t *cw_all = reinterpret_cast<uint32_t *>(smem_raw + sweep_cw_offset());
    const int4 *tbl = reinterpret_cast<const int4 *>(smem_raw + sweep_tbl_offset(wmax));
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const SpaceDev &S = P.S;
    double best_t = __longlong_as_double(0x7ff0000000000000LL);
    unsigned long long best_i = ~0ull;
    uint32_t cnt_val = 0;
    // pass 2 may be scheduled now (it waits for this grid's completion)
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    // CTA tiles of 16-byte aligned records (the TMA's alignment): the full
    // ones, plus the batch's last partial one when the batch is a whole
    // number of design points (its missing warp tiles are empty)
    const bool sweepable = P.aligned && !P.pr.mem;
    const unsigned long long ntiles =
        sweepable ? P.n / SWT + ((P.n % SWT) && (P.n % CXT) == 0 ? 1ull : 0ull) : 0ull;
    // everything past them goes to pass 2 as warp tiles (warp-aggregated list appends)
    {
        const unsigned long long nsub = (P.n + CTILE - 1) / CTILE;
        for (unsigned long long b0 = ntiles * CPT + (unsigned long long)blockIdx.x * THREADS;
             b0 < nsub; b0 += (unsigned long long)gridDim.x * THREADS) {
            const unsigned long long sub = b0 + tid;
            const bool mine = sub < nsub;
            const unsigned bal = __ballot_sync(FULL, mine);
            unsigned base = 0;
            if (lane == 0 && bal) base = atomicAdd(P.tile_count, (unsigned)__popc(bal));
            base = __shfl_sync(FULL, base, 0);
            if (mine) P.tile_list[base + __popc(bal & ((1u << lane) - 1u))] = (uint32_t)sub;
        }
    }
    // tiles: the first is blockIdx.x, the second claimed now, tile r + 3 in
    // round r (one round before its copy is issued)
    unsigned *claim = P.tile_count + CLAIM1;
    if (tid == 0) {
        mbar_init(&sm.rbar, 1);
        mbar_init(&sm.tbar[0], 1);
        mbar_init(&sm.tbar[1], 1);
        for (int i = 0; i < 2; i++) {
            mbar_init(&sm.abar[i], WARPS);
            mbar_init(&sm.cbar[i], WARPS);
        }
        sm.tbl_skel = SW_BAD;
        sm.ab_cnt[0] = sm.ab_cnt[1] = sm.ab_cnt[2] = sm.ab_cnt[3] = 0;
        sm.a_done[0] = sm.a_done[1] = 0;
        sm.tile_id[0] = blockIdx.x;
        sm.tile_id[1] = atomicAdd(claim, 1u) + gridDim.x;
        sm.tile_id[2] = sm.tile_id[3] = 0xffffffffu;
        if (blockIdx.x < ntiles) issue_cta_copy<SWT>(P, sm.rec, &sm.rbar, (unsigned long long)blockIdx.x * SWT);
    }
    __syncthreads();
    const double rfh = S.rfh, rfl = S.rfl;
#if GROPHECY_PHASE_TIMING
    long long pt_last = clock64();
#endif
#pragma unroll 1
    for (int r = -1;; r++) {
        // tile r + 1 (stored by the first A/B task of tile r - 1, which every
        // warp has seen complete: the abar wait of its phase C of tile r - 1)
        const unsigned long long tn = sm.tile_id[(r + 1) & 3];
        // ---- C: tile r, CTA-wide; unit = transformation x ----
        if (r >= 0) {
            const uint32_t b = (uint32_t)r & 1u;
            mbar_wait(&sm.abar[b], ((uint32_t)r >> 1) & 1u);   // every A/B task of tile r
            PT_MARK(4);   // waiting for tile r's A/B tasks
            const unsigned long long tile = sm.tile_id[r & 3];
            const uint32_t ngt = (uint32_t)((P.n - tile * SWT < SWT ? P.n - tile * SWT : SWT) / CXT);
            const int gwi = (int)ngt - 32 * warp;
            const uint32_t gw = gwi <= 0 ? 0u : (gwi >= 32 ? 32u : (uint32_t)gwi);
            // uniform: every non-empty warp tile canonical, of one skeleton
            const uint32_t s_all = sm.wstat[b][0];
            bool uni;
            {   // lanes < WARPS read one warp tile's status each
                const uint32_t st = sm.wstat[b][lane & (WARPS - 1)];
                uni = __all_sync(FULL, st == s_all || st == SW_EMPTY) && s_all != SW_BAD && s_all != SW_EMPTY &&
                      sm.perm_ok[b];
            }
            // (TWO) the tile's second skeleton: the same in every warp tile that has one
            uint32_t skB = SW_BAD;
            if constexpr (TWO) {
                const uint32_t wo = sm.wsk[b][lane & (WARPS - 1)];
                if (uni && __any_sync(FULL, wo != SW_BAD)) {
                    skB = __reduce_min_sync(FULL, wo);
                    uni = skB == __reduce_max_sync(FULL, wo == SW_BAD ? 0u : wo) &&
                          __all_sync(FULL, (uint32_t)lane >= CXT ||
                                               (sm.perm[b][lane] & 0xffffu) < S.skel[skB].n_xforms);
                }
            }
            if (!uni) {
                // its pass-2 chunks (CTILE records each), one per warp
                if (lane == 0 && (unsigned)warp < CPT && (unsigned long long)warp * CTILE < (unsigned long long)ngt * CXT)
                    P.tile_list[atomicAdd(P.tile_count, 1u)] = (uint32_t)(tile * CPT + warp);
            } else {
                // the tile's skeleton (set by its first task)
                const uint4 ti4 = sm.tinf[b];
                uint32_t kx_base = ti4.x, X = ti4.y;
                bool has_once = ti4.z != 0u;
                const unsigned long long tbase = P.base + tile * SWT;
                const uint32_t *cwb = cw_all + b * wmax * (uint32_t)SW_GROUPS;
                // work slots whose grid may be unsaturated for one of the tile's
                // design points (a unit covers all of them: its chains are the
                // tile's warp tiles)
                static_assert(UNITS == (unsigned)CXT, "one chain block per unit");
                uint32_t gk = 0;
#pragma unroll
                for (int w = 0; w < WARPS; w++) gk |= sm.smallw[b][w];
                const bool mixed = TWO && skB != SW_BAD;
                // (TWO) the units of each skeleton; a design point takes part only
                // in its own skeleton's (dsk)
#pragma unroll 1
                for (uint32_t si = 0; si < (mixed ? 2u : 1u); si++) {
                if (si) {   // the second skeleton's constants (from global memory: rare)
                    const SkelInfo &IB = S.skel[skB];
                    const uint32_t km = IB.n_kernels == 32 ? 0xffffffffu : (1u << IB.n_kernels) - 1u;
                    kx_base = IB.kx_base;
                    X = IB.n_xforms;
                    has_once = (IB.per_iter_mask & km) != km;
                }
                // units in snake order over the warps (16 units: warp w takes w
                // and 15 - w; in the identity layout the costliest transformation
                // pairs with the cheapest)
#pragma unroll 1
                for (unsigned rr = 0; rr < (UNITS + WARPS - 1) / WARPS; rr++) {
                    const unsigned u = (rr & 1u) ? (rr + 1u) * WARPS - 1u - (unsigned)warp : rr * WARPS + (unsigned)warp;
                    if (u >= UNITS) continue;
                    // the unit's transformation and position (set by the tile's first task)
                    uint4 hdr = sm.uhdr[b][u % CXT];
                    uint32_t pos = sm.upos[b][u % CXT];
                    if (TWO && si) {
                        if (sm.perm_ident[b]) {
                            hdr = __ldg(&S.xhdru[kx_base + u % CXT]);
                            pos = hdr.x;
                        } else {
                            pos = u % CXT;
                            hdr = __ldg(&S.xhdr[kx_base + (sm.perm[b][pos] & 0xffffu)]);
                        }
                    }
                    const uint32_t x = hdr.x;
                    const uint32_t jb = u / CXT, xf = hdr.w & 0xffu;
#if GROPHECY_XINF_SKIP
                    // an infeasible kernel makes every total of the unit +inf (or NaN
                    // at iters = 0): none takes part in the argmin (non-finite totals
                    // never win), so the unit has nothing to compute
                    if (xf & (XINF_ITER | XINF_ONCE)) continue;
#endif
                    const KxProg *pe = S.xprog + hdr.y;
                    const uint32_t n_it = hdr.z & 0xffffu, n_all = n_it + (hdr.z >> 16);
                    double ti[NCH], to[NCH];
#pragma unroll
                    for (int j = 0; j < NCH; j++) ti[j] = to[j] = 0.0;
                    // this lane's work-count chunks (cw_index for chains jb*NCH + 4q)
                    const uint32_t *cwl = cwb + lane * (SW_GROUPS / 32);
                    uint32_t cwo[NCH / 4];
#pragma unroll
                    for (int q = 0; q < NCH / 4; q++)
                        cwo[q] = ((((jb * NCH) / 4 + (uint32_t)q) ^ ((uint32_t)lane >> 2)) & 1u) << 2;
                    static_assert(SW_GROUPS == 256, "KxProg::cwoff = slot * 256");
                    struct Ent {
                        uint4 hd, kw;
                        double2 c01, c23;
                    };
                    auto load_ent = [&](const KxProg *e) {
                        const uint4 *q = reinterpret_cast<const uint4 *>(e);
                        Ent en;
                        en.hd = __ldg(q);
                        en.kw = __ldg(q + 1);
                        en.c01 = __ldg(reinterpret_cast<const double2 *>(q + 2));
                        en.c23 = __ldg(reinterpret_cast<const double2 *>(q + 3));
                        return en;
                    };
                    auto one_kernel = [&](const Ent &en, double (&acc)[NCH]) {
                        // hd = {m, sat, cc lo, cc hi}, kw = {cwoff, sh, kbit, cls}
                        const uint32_t sh = en.kw.y;
                        const unsigned long long cc = ((unsigned long long)en.hd.w << 32) | en.hd.z;
                        uint32_t blocks[NCH];
                        const uint32_t *cwk = cwl + en.kw.x;
#pragma unroll
                        for (int q = 0; q < NCH / 4; q++) {
                            const uint4 w4 = *reinterpret_cast<const uint4 *>(cwk + cwo[q]);
                            const uint32_t w[4] = {w4.x, w4.y, w4.z, w4.w};
#pragma unroll
                            for (int t = 0; t < 4; t++)
                                blocks[4 * q + t] = (uint32_t)(((unsigned long long)w[t] * en.hd.x + cc) >> 32);
                        }
                        // the post-shift (power-of-two ipb: none) is a case of its own
                        // falling through into the class, so that no unshifted entry
                        // issues it predicated off
                        auto shift = [&] {
#pragma unroll
                            for (int j = 0; j < NCH; j++) blocks[j] >>= sh;
                        };
                        double tk[NCH];
#if GROPHECY_DISPATCH_TREE
                        // warp-uniform branches on the class bits (no indirect jump)
                        const uint32_t cl = en.kw.w;
                        if (cl & KXC_SHIFT) shift();
                        if (cl & 2u) {
                            if (cl & 1u) cls_times<KXC_NS>(en.c01, en.c23, blocks, rfh, rfl, tk);
                            else cls_times<KXC_NS0>(en.c01, en.c23, blocks, rfh, rfl, tk);
                        } else {
                            if (cl & 1u) cls_times<KXC_P2S>(en.c01, en.c23, blocks, rfh, rfl, tk);
                            else cls_times<KXC_P2S0>(en.c01, en.c23, blocks, rfh, rfl, tk);
                        }
#else
                        switch (en.kw.w) {
                        case KXC_P2S0 | KXC_SHIFT: shift(); [[fallthrough]];
                        case KXC_P2S0: cls_times<KXC_P2S0>(en.c01, en.c23, blocks, rfh, rfl, tk); break;
                        case KXC_P2S | KXC_SHIFT: shift(); [[fallthrough]];
                        case KXC_P2S: cls_times<KXC_P2S>(en.c01, en.c23, blocks, rfh, rfl, tk); break;
                        case KXC_NS0 | KXC_SHIFT: shift(); [[fallthrough]];
                        case KXC_NS0: cls_times<KXC_NS0>(en.c01, en.c23, blocks, rfh, rfl, tk); break;
                        case KXC_NS | KXC_SHIFT: shift(); [[fallthrough]];
                        default: cls_times<KXC_NS>(en.c01, en.c23, blocks, rfh, rfl, tk); break;
                        }
#endif
                        if (gk & en.kw.z) {
                            // off the saturated path: the small-grid table (SKF_TABULATED)
                            const uint32_t sat = en.hd.y & 0xffffu;
                            bool any = false;
#pragma unroll
                            for (int j = 0; j < NCH; j++) any |= blocks[j] < sat;
                            if (any) {
                                const uint32_t k = en.hd.y >> 16;   // the entry's kernel
                                const unsigned long long row =
                                    reinterpret_cast<unsigned long long>(S.small_t) +
                                    (unsigned long long)((kx_base + k * X + x) * S.small_stride) * sizeof(double);
#pragma unroll
                                for (int j = 0; j < NCH; j++)
                                    if (blocks[j] < sat)
                                        tk[j] = __ldg(reinterpret_cast<const double *>(
                                            row + (unsigned long long)blocks[j] * sizeof(double)));
                            }
                        }
#pragma unroll
                        for (int j = 0; j < NCH; j++) acc[j] = __dadd_rn(acc[j], tk[j]);
                    };
                    // sums in ascending kernel order (N6): the program lists the
                    // per-iteration kernels, then the run-once ones; infeasible
                    // kernels are not listed (their sum is +inf through xinf)
                    {
                        const KxProg *e = pe;
#pragma unroll 1
                        for (int i = (int)n_it; i > 0; i--, ++e) one_kernel(load_ent(e), ti);
#pragma unroll 1
                        for (int i = (int)(n_all - n_it); i > 0; i--, ++e) one_kernel(load_ent(e), to);
                    }
                    const double inf = __longlong_as_double(0x7ff0000000000000LL);
#if !GROPHECY_XINF_SKIP
                    if (xf & XINF_ITER) {
#pragma unroll
                        for (int j = 0; j < NCH; j++) ti[j] = inf;
                    }
                    if (xf & XINF_ONCE) {
#pragma unroll
                        for (int j = 0; j < NCH; j++) to[j] = inf;
                    }
#endif
                    // totals; without run-once kernels t_once =
                    // +0.0 and +0.0 + iters * t_iter = iters * t_iter exactly
                    const bool once = has_once || (xf & XINF_ONCE);
                    double cmin = inf;
                    int cj = -1;
                    auto totals = [&](auto ONCE, auto MIXED) {
#pragma unroll
                        for (int j = 0; j < NCH; j++) {
                            const int gj = 32 * ((int)jb * NCH + j) + lane;
                            double tk = __dmul_rn(sm.it[b][gj], ti[j]);
                            if constexpr (decltype(ONCE)::value) tk = __dadd_rn(to[j], tk);
                            const double2 thd = sm.thd[b][gj];
                            double tt = __dadd_rn(__dadd_rn(tk, thd.x), thd.y);
                            if constexpr (decltype(MIXED)::value) {
                                // the other skeleton's design point (chain j = warp tile
                                // jb*NCH + j; dsk is written for warp tiles holding the second)
                                const uint32_t d = sm.wsk[b][(int)jb * NCH + j] == SW_BAD ? 0u : sm.dsk[b][gj];
                                if (d != si) tt = __longlong_as_double(0x7ff0000000000000LL);
                            }
                            // chains in increasing record index: strict < keeps the lowest
                            // (design points past a partial tile's end have tt = +inf)
                            if (tt < cmin) {
                                cmin = tt;
                                cj = j;
                            }
                        }
                    };
                    if (TWO && mixed) {
                        if (once) totals(std::true_type{}, std::integral_constant<bool, TWO>{});
                        else totals(std::false_type{}, std::integral_constant<bool, TWO>{});
                    } else {
                        if (once) totals(std::true_type{}, std::false_type{});
                        else totals(std::false_type{}, std::false_type{});
                    }
                    if (cj >= 0) {
                        const int gj = 32 * ((int)jb * NCH + cj) + lane;
                        const unsigned long long idx = tbase + (unsigned long long)gj * CXT + pos;
                        if (better(cmin, idx, best_t, best_i)) {
                            best_t = cmin;
                            best_i = idx;
                        }
                    }
                }
                }   // skeletons
                if (lane == 0) cnt_val += gw * (uint32_t)CXT;
            }
            __syncwarp();
            if (lane == 0)
                asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&sm.cbar[b])) : "memory");
        }
        PT_MARK(5);   // phase C (model, totals, argmin)
        if (tn >= ntiles) break;
        // ---- A/B tasks of tile r + 1 (warp tile q, buffer b1), claimed until
        // none is left: every warp makes exactly one failing claim per tile, so
        // the 2 WARPS-th claim is the tile's last and resets the counter ----
        {
            const uint32_t b1 = (uint32_t)(r + 1) & 1u;
            const uint32_t ngt = (uint32_t)((P.n - tn * SWT < SWT ? P.n - tn * SWT : SWT) / CXT);
            uint32_t *cwb = cw_all + b1 * wmax * (uint32_t)SW_GROUPS;
#pragma unroll 1
            for (;;) {
                uint32_t q = 0;
                if (lane == 0) {
                    q = atomicAdd(&sm.ab_cnt[(r + 1) & 3], 1u);
                    if (q == 2u * WARPS - 1u) sm.ab_cnt[(r + 1) & 3] = 0u;
                }
                q = __shfl_sync(FULL, q, 0);
                if (q >= (uint32_t)WARPS) break;
                // the first task claims tile r + 3 (stored at its end)
                unsigned claimed = 0;
                if (q == 0 && lane == 0) claimed = atomicAdd(claim, 1u);
                mbar_wait(&sm.rbar, (uint32_t)(r + 1) & 1u);
                PT_MARK(0);   // waiting for the staged records
                const int gwi = (int)ngt - 32 * (int)q;
                const uint32_t gw = gwi <= 0 ? 0u : (gwi >= 32 ? 32u : (uint32_t)gwi);
                uint32_t s0 = 0, n0 = 0, m0 = 0, i0 = 0;
                bool ok = gw ? sweep_phase_a<CXT, TWO>(S, sm.rec, (int)q, lane, gw, s0, n0, m0, i0) : false;
                const uint32_t skel = s0 >> 16;
                // the tile's transformation order (its first design point's skx)
                uint32_t sq = 0;
                if (q == 0 && lane < CXT) sq = sm.rec[0][lane];
                // (TWO) the tile's first skeleton; at most one other among its design points
                uint32_t skA = 0, omin = SW_BAD;
                bool anyoth = false;
                if constexpr (TWO) {
                    skA = sm.rec[0][0] >> 16;
                    const bool oth = (uint32_t)lane < gw && skel != skA;
                    anyoth = __any_sync(FULL, oth);
                    if (anyoth) {
                        omin = __reduce_min_sync(FULL, oth ? skel : SW_BAD);
                        if (omin != __reduce_max_sync(FULL, oth ? skel : 0u)) ok = false;   // three: pass 2
                    }
                }
                __syncwarp();
                if (lane == 0) {
                    // every read of the record buffer by this warp is done: the
                    // tile's last one releases it to the copy of tile r + 2
                    __threadfence_block();
                    if (atomicAdd(&sm.a_done[b1], 1u) == (unsigned)WARPS - 1u) {
                        __threadfence_block();
                        sm.a_done[b1] = 0u;   // (next used by tile r + 3)
                        const unsigned long long t2 = sm.tile_id[(r + 2) & 3];
                        if (t2 < ntiles) issue_cta_copy<SWT>(P, sm.rec, &sm.rbar, t2 * SWT);
                    }
                }
                PT_MARK(1);   // phase A
                // buffer b1 was read by the phase C of tile r - 1
                if (r >= 1) mbar_wait(&sm.cbar[b1], ((uint32_t)(r - 1) >> 1) & 1u);
                if (q == 0) {
                    // warp tile 0's skeleton decides the tile's usage table: staged
                    // when it changes (every reader of the previous one finished in
                    // an earlier round)
                    if (lane == 0) {
                        const uint32_t ts = ok ? skel : SW_BAD;
                        bool staged = false;
                        if (ts != SW_BAD && ts != sm.tbl_skel && S.skel[ts].polyf_base != POLY32_NONE) {
                            const SkelInfo &I0 = S.skel[ts];
                            const uint32_t bytes =
                                ((I0.polyf_nhd & 0xffffu) + (I0.polyf_nhd >> 16)) * POLY_CLASSES * 16u;
                            sm.tbl_skel = ts;
                            if (bytes) {   // (no transfer at all: nothing to stage)
                                asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
                                const uint32_t bar = smem_u32(&sm.tbar[b1]);
                                asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar),
                                             "r"(bytes)
                                             : "memory");
                                asm volatile(
                                    "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], "
                                    "%2, [%3];" ::"r"(smem_u32(tbl)),
                                    "l"(S.poly + I0.polyf_base), "r"(bytes), "r"(bar)
                                    : "memory");
                                staged = true;
                            }
                        }
                        if (!staged)
                            asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&sm.tbar[b1]))
                                         : "memory");
                    }
                    if (lane < CXT) {
                        sm.perm[b1][lane] = sq;
                        const unsigned bad = __ballot_sync((1u << CXT) - 1u, (sq & 0xffffu) != (uint32_t)lane);
                        if (lane == 0) sm.perm_ident[b1] = bad == 0u;
                    }
                    __syncwarp();
                }
                mbar_wait(&sm.tbar[b1], ((uint32_t)(r + 1) >> 1) & 1u);
                PT_MARK(2);   // the tile's usage-table decision
                // ---- B: work counts and usage of design point g ----
                const int g = (int)q * 32 + lane;
                uint32_t wsmall = 0;
                if (ok) {
                    const SkelInfo &I = S.skel[skel];   // warp-uniform
                    const uint32_t n_arrays = I.n_arrays, nw = I.n_wslots;
                    const long long nxny = (long long)((unsigned long long)n0 * m0);
                    bool huge = false;
                    uint32_t small = 0;
                    const int4 *wf = S.wslot_work + I.w_base;
                    const uint32_t *wsat = S.wslot_sat + I.w_base;
                    if (__all_sync(FULL, (unsigned long long)I.wslot_c32 * ((unsigned long long)n0 + m0 +
                                                                             (unsigned long long)nxny) <
                                             (1ull << 31))) {
                        // every slot's count is exact in 32-bit arithmetic
                        const int nx32 = (int)n0, ny32 = (int)m0, nxny32 = (int)nxny;
                        for (uint32_t j = 0; j < nw; j++) {
                            const int4 c = __ldg(wf + j);
                            const int w = c.x + ((c.y * nx32 + c.z * ny32 + c.w * nxny32) >> 3);
                            const uint32_t ws = w <= 0 ? 0u : (uint32_t)w;   // < 2^30
                            cwb[cw_index(j, (uint32_t)lane, q)] = ws;
                            small |= (ws < __ldg(wsat + j) ? 1u : 0u) << j;
                        }
                    } else {
                        for (uint32_t j = 0; j < nw; j++) {
                            const uint32_t w = w_store(aff8n(__ldg(wf + j), (int)n0, (int)m0, nxny));
                            cwb[cw_index(j, (uint32_t)lane, q)] = w;
                            huge |= w == W_HUGE;
                            small |= (w < __ldg(wsat + j) ? 1u : 0u) << j;
                        }
                    }
                    wsmall = __reduce_or_sync(FULL, small);
                    if (q == 0) {
                        // the tile's first design point (lane 0's) is itself consistent:
                        // one skeleton, every transformation < n_xforms
                        const bool okq = TWO ? ((uint32_t)lane >= CXT ||
                                                ((sq >> 16) == skA && (sq & 0xffffu) < S.skel[skA].n_xforms))
                                             : ((uint32_t)lane >= CXT || ((sq >> 16) == skel && (sq & 0xffffu) < I.n_xforms));
                        const bool all = __all_sync(FULL, okq);
                        if (lane == 0) sm.perm_ok[b1] = all;
                        // the units' headers for phase C: in the identity layout unit u
                        // is the u-th costliest transformation (at its own position),
                        // else the transformation at position u
                        const SkelInfo &IA = TWO ? S.skel[skA] : I;   // the tile's first skeleton
                        if (all && lane == 0) {
                            const uint32_t km = IA.n_kernels == 32 ? 0xffffffffu : (1u << IA.n_kernels) - 1u;
                            sm.tinf[b1] = make_uint4(IA.kx_base, IA.n_xforms, (IA.per_iter_mask & km) != km, 0u);
                        }
                        if (all && (uint32_t)lane < CXT) {
                            uint4 h;
                            uint32_t pos;
                            if (sm.perm_ident[b1]) {
                                h = __ldg(&S.xhdru[IA.kx_base + lane]);
                                pos = h.x;
                            } else {
                                h = __ldg(&S.xhdr[IA.kx_base + (sq & 0xffffu)]);
                                pos = (uint32_t)lane;
                            }
                            sm.uhdr[b1][lane] = h;
                            sm.upos[b1][lane] = pos;
                        }
                    }
                    ok = __all_sync(FULL, !huge && n0 >= I.plan_tx && m0 >= I.plan_ty);
                    if (ok) {
                        Usage u = {0ull, 0ull, 0.0, 0.0};
                        const uint32_t stride = I.poly_stride, a8 = n0 >> 3, b8 = m0 >> 3;
                        const uint32_t cls = (n0 & 7u) * 8u + (m0 & 7u);
                        const uint32_t pm = I.poly_mask;
                        if (TWO && __any_sync(FULL, I.polyf_base != POLY32_NONE && skel != sm.tbl_skel)) {
                            // (a second skeleton in this warp tile) collectives first,
                            // then the staged table or its global copy per lane
                            const bool pf = I.polyf_base != POLY32_NONE;
                            const unsigned long long bnd =
                                (unsigned long long)I.polyf_cmax[0] + (unsigned long long)I.polyf_cmax[1] * a8 +
                                (unsigned long long)I.polyf_cmax[2] * b8 +
                                (unsigned long long)I.polyf_cmax[3] * ((unsigned long long)a8 * b8);
                            const bool u32 = __all_sync(FULL, !pf || bnd < (1ull << 32));
                            if (pf && skel == sm.tbl_skel) {
                                if (u32) group_usage_s<true>(tbl + cls, I.polyf_nhd, a8, b8, P.pc, u);
                                else group_usage_s<false>(tbl + cls, I.polyf_nhd, a8, b8, P.pc, u);
                            } else if (pf) {
                                const int4 *tg = reinterpret_cast<const int4 *>(S.poly + I.polyf_base) + cls;
                                if (u32) group_usage_s<true>(tg, I.polyf_nhd, a8, b8, P.pc, u);
                                else group_usage_s<false>(tg, I.polyf_nhd, a8, b8, P.pc, u);
                            } else if (I.poly32_base != POLY32_NONE) {
                                group_usage32<GROPHECY_AU32>(reinterpret_cast<const int4 *>(S.poly + I.poly32_base) +
                                                                 (size_t)cls * (2u * n_arrays),
                                                             n_arrays, pm, a8, b8, P.pc,
                                                             reinterpret_cast<const int4 *>(S.poly), u);
                            } else if (stride > 4) {
                                group_usage<true, 2>(S.poly + I.poly_base + (size_t)cls * (2u * n_arrays * stride),
                                                     stride, n_arrays, pm, a8, b8, P.pc, S.poly, u);
                            } else {
                                group_usage<false, 4>(S.poly + I.poly_base + (size_t)cls * (2u * n_arrays * stride),
                                                      stride, n_arrays, pm, a8, b8, P.pc, S.poly, u);
                            }
                        } else if (I.polyf_base != POLY32_NONE) {
                            // the staged table is warp tile 0's skeleton: another
                            // skeleton makes the tile non-uniform (pass 2) anyway
                            ok = skel == sm.tbl_skel;
                            if (ok) {
                                const unsigned long long bnd =
                                    (unsigned long long)I.polyf_cmax[0] + (unsigned long long)I.polyf_cmax[1] * a8 +
                                    (unsigned long long)I.polyf_cmax[2] * b8 +
                                    (unsigned long long)I.polyf_cmax[3] * ((unsigned long long)a8 * b8);
                                if (__all_sync(FULL, bnd < (1ull << 32)))
                                    group_usage_s<true>(tbl + cls, I.polyf_nhd, a8, b8, P.pc, u);
                                else
                                    group_usage_s<false>(tbl + cls, I.polyf_nhd, a8, b8, P.pc, u);
                            }
                        } else if (I.poly32_base != POLY32_NONE) {
                            group_usage32<GROPHECY_AU32>(reinterpret_cast<const int4 *>(S.poly + I.poly32_base) +
                                                             (size_t)cls * (2u * n_arrays),
                                                         n_arrays, pm, a8, b8, P.pc,
                                                         reinterpret_cast<const int4 *>(S.poly), u);
                        } else if (stride > 4) {
                            group_usage<true, 2>(S.poly + I.poly_base + (size_t)cls * (2u * n_arrays * stride),
                                                 stride, n_arrays, pm, a8, b8, P.pc, S.poly, u);
                        } else {
                            group_usage<false, 4>(S.poly + I.poly_base + (size_t)cls * (2u * n_arrays * stride),
                                                  stride, n_arrays, pm, a8, b8, P.pc, S.poly, u);
                        }
                        sm.thd[b1][g] = make_double2(u.th, u.td);
                        sm.it[b1][g] = (double)i0;
                        if (TWO && anyoth) sm.dsk[b1][g] = skel != skA;   // (read for such warp tiles only)
                    }
                } else if (q == 0 && lane == 0) {
                    sm.perm_ok[b1] = 0u;   // (warp tile 0 is not canonical: the tile is not uniform)
                }
                if (lane == 0) {
                    sm.wstat[b1][q] = gw == 0 ? SW_EMPTY : (ok ? (TWO ? skA : skel) : SW_BAD);
                    sm.smallw[b1][q] = wsmall;
                    if (TWO) sm.wsk[b1][q] = omin;
                }
                // design points past a partial tile's end: t_h2d = +inf makes their
                // totals +inf (never below the running minimum in phase C)
                if ((uint32_t)g >= ngt) sm.thd[b1][g] = make_double2(__longlong_as_double(0x7ff0000000000000LL), 0.0);
                if (q == 0 && lane == 0) sm.tile_id[(r + 3) & 3] = claimed + gridDim.x;   // tile r + 3
                __syncwarp();
                if (lane == 0)
                    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&sm.abar[b1])) : "memory");
                PT_MARK(3);   // phase B (work counts, usage)
            }
        }
    }
    // the bytes of each lane's running best (its design point's usage; the
    // record buffer is idle now: no copy is in flight after the last round)
    unsigned long long keep[2] = {0ull, 0ull};
    if (best_i != ~0ull) {
        const unsigned long long li = best_i - P.base;
        sweep_bytes(S.poly, P.pc, &S.skel[__ldg(P.skx + li) >> 16], __ldg(P.nx + li), __ldg(P.ny + li), keep);
    }
    if (!P.fused) {
        unsigned long long *bh = reinterpret_cast<unsigned long long *>(sm.rec[0]);
        bh[tid] = keep[0];
        bh[THREADS + tid] = keep[1];
        __syncwarp();
        if (BEST) finish_best(P, bh + warp * 32, bh + THREADS + warp * 32, lane, warp, best_t, best_i, 0u,
                              cnt_val, gridDim.x);
        return;
    }
    // ---- pass 2 in the same (cooperative) launch: once every CTA has
    // listed its tiles, the CTAs drain the list with the general 128-record
    // tiles (claims from a counter), each lane's running best continuing ----
    __syncthreads();
    cooperative_groups::this_grid().sync();
    WarpSmem &ws = reinterpret_cast<CtaSmem *>(smem_raw)->w[warp];
    ws.best_h[lane] = keep[0];
    ws.best_d[lane] = keep[1];
    constexpr unsigned SUBS = CTILE / WTILE;
    const unsigned units = *(volatile unsigned *)P.tile_count * SUBS;
    unsigned *next = P.tile_count + CLAIM2;
    uint32_t cnt_inv = 0;
#pragma unroll 1
    for (;;) {
        unsigned q = 0;
        if (lane == 0) q = atomicAdd(next, 1u);
        q = __shfl_sync(FULL, q, 0);
        if (q >= units) break;
        const unsigned long long t0 = (unsigned long long)P.tile_list[q / SUBS] * CTILE +
                                      (unsigned long long)(q % SUBS) * WTILE;
        if (t0 < P.n) general_tile<BEST>(P, ws, t0, lane, best_t, best_i, cnt_inv, cnt_val);
    }
    if (BEST) finish_best(P, ws.best_h, ws.best_d, lane, warp, best_t, best_i, cnt_inv, cnt_val, gridDim.x);
}

// Pass 2: the listed tiles as general 128-record tiles (any layout).
template <bool BEST>
__global__ void __launch_bounds__(THREADS, GROPHECY_MINB) general_kernel(const Params P)
{
    extern __shared__ __align__(16) unsigned char smem_raw[];
    const int lane = threadIdx.x & 31;
    const int warp = threadIdx.x >> 5;
    WarpSmem &ws = reinterpret_cast<CtaSmem *>(smem_raw)->w[warp];
    double best_t = __longlong_as_double(0x7ff0000000000000LL);
    unsigned long long best_i = ~0ull;
    uint32_t cnt_inv = 0, cnt_val = 0;
    ws.best_h[lane] = 0;
    ws.best_d[lane] = 0;
    // launched programmatically dependent on pass 1 (best mode): wait until
    // pass 1 has completed and its list / result are visible
    asm volatile("griddepcontrol.wait;" ::: "memory");
    const unsigned count = P.direct ? (unsigned)((P.n + CTILE - 1) / CTILE) : *(volatile unsigned *)P.tile_count;
    // only the blocks with listed tiles take part (none: pass 1's result and
    // outputs are final)
    // units of work: the listed tiles' 128-record sub-tiles, claimed one at a
    // time from a counter (P.tile_count[CLAIM2], zeroed with the tile count
    // before pass 1): the per-tile cost of the general sweep varies by orders of
    // magnitude, so a static split leaves warps idle at the end.  The list
    // is appended in any order (atomics across CTAs), so a warp meets its
    // records in arbitrary index order: general_tile's running best must (and
    // does) compare (t, index) lexicographically, never by t alone.
    constexpr unsigned SUBS = CTILE / WTILE;
    const unsigned units = count * SUBS;
    const unsigned nblocks = min(gridDim.x, (units + WARPS - 1) / WARPS);
    if (blockIdx.x >= nblocks) {
        if (nblocks == 0 && blockIdx.x == 0 && threadIdx.x == 0) {
            // nothing listed: pass 1 used only its tile claims; zero them here
            if (P.reset_counters) P.tile_count[CLAIM1] = 0u;
            // an empty direct batch: its (empty) result, unless merging
            if (BEST && P.direct && !P.accumulate) to_result(*P.out, none_best());
        }
        return;
    }
    unsigned *next = P.tile_count + CLAIM2;
#pragma unroll 1
    for (;;) {
        unsigned q = 0;
        if (lane == 0) q = atomicAdd(next, 1u);
        q = __shfl_sync(FULL, q, 0);
        if (q >= units) break;
        const unsigned long long t0 = (unsigned long long)(P.direct ? q / SUBS : P.tile_list[q / SUBS]) * CTILE +
                                      (unsigned long long)(q % SUBS) * WTILE;
        if (t0 < P.n) general_tile<BEST>(P, ws, t0, lane, best_t, best_i, cnt_inv, cnt_val);
    }
    if (BEST) finish_best(P, ws.best_h, ws.best_d, lane, warp, best_t, best_i, cnt_inv, cnt_val, nblocks);
}

__global__ void combine_kernel(const grophecy_best_result *in, uint32_t count,
                               grophecy_best_result *out)
{
    const int lane = threadIdx.x & 31;
    Best b = none_best();
    for (uint32_t j = lane; j < count; j += 32) merge(b, from_result(in[j]));
    b = warp_best(b);
    if (lane == 0) to_result(*out, b);
}

constexpr uint32_t SMEM_CTA_MAX = 227u * 1024u;   // opt-in shared memory per CTA (sm_100)

static void set_smem_attrs()
{
    // per device: the attributes belong to the current device's context
    static bool done_dev[64] = {};
    int dev = 0;
    cudaGetDevice(&dev);
    bool &done = done_dev[dev & 63];
    if (done) return;
    const int sm = (int)sizeof(CtaSmem), cs = (int)(WARPS * canon_warp_bytes(MAXK));
    cudaFuncSetAttribute(canon_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, cs);
    cudaFuncSetAttribute(general_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm);
    cudaFuncSetAttribute(general_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm);
    const int ss = (int)std::min<uint32_t>(
        SMEM_CTA_MAX, std::max<uint32_t>(sweep_smem_bytes(MAXK, 2u * GROPHECY_MAX_ARRAYS * POLY_CLASSES * 16u),
                                         (uint32_t)sizeof(CtaSmem)));
    cudaFuncSetAttribute(sweep_kernel<true, 4, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, ss);
    cudaFuncSetAttribute(sweep_kernel<true, 8, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, ss);
    cudaFuncSetAttribute(sweep_kernel<true, 16, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, ss);
    cudaFuncSetAttribute(sweep_kernel<true, 16, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, ss);
    done = true;
}

static int grid_for(const grophecy_space *s, unsigned long long n, int per_sm_cap, bool canon)
{
    static int occ_general = 0;
    set_smem_attrs();
    int occ = 0;
    if (canon) {
        // per space: its dynamic shared memory depends on its kernel count
        if (!s->occ_canon) {
            int o = 0;
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o, canon_kernel<false>, THREADS,
                                                          WARPS * canon_warp_bytes(s->max_kernels));
            const_cast<grophecy_space *>(s)->occ_canon = o < 1 ? 1 : o;
        }
        occ = s->occ_canon;
    } else {
        if (!occ_general) {
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ_general, general_kernel<true>, THREADS,
                                                          sizeof(CtaSmem));
            if (occ_general < 1) occ_general = 1;
        }
        occ = occ_general;
    }
    const unsigned long long want = (n + (unsigned long long)CTILE * WARPS - 1) / ((unsigned long long)CTILE * WARPS);
    unsigned long long cap = (unsigned long long)s->grid_best * (unsigned long long)std::min(occ, per_sm_cap);
    if (cap > s->max_partials - 1) cap = s->max_partials - 1;   // last slot = result
    return (int)std::max<unsigned long long>(1ull, std::min(want, cap));
}

// The sweep kernel for the space's design-point size.
using SweepFn = void (*)(Params);
static SweepFn sweep_fn(const grophecy_space *s, bool two)
{
    if (two && s->sweep_cx == 16) return sweep_kernel<true, 16, true>;   // (design points of 16 only)
    return s->sweep_cx == 4 ? sweep_kernel<true, 4, false>
                            : (s->sweep_cx == 8 ? sweep_kernel<true, 8, false> : sweep_kernel<true, 16, false>);
}

// Two-skeleton sweep tiles pay a little on every tile and save the general
// path on the tiles that straddle a skeleton boundary: worth it when a batch
// has few tiles per skeleton (the boundary tiles are a visible share of the
// work or of the latency).
static bool sweep_two(const grophecy_space *s, unsigned long long n)
{
    if (s->sweep_two_env >= 0) return s->sweep_two_env != 0;   // test hook
    const unsigned long long tiles = n / ((unsigned long long)SW_GROUPS * s->sweep_cx) + 1;
    return s->dev.n_skels > 1 && tiles < 128ull * s->dev.n_skels;
}

// Dynamic shared memory of the (fused) sweep launch: its own layout, or the
// general tiles' one after the grid barrier, whichever is larger.
static uint32_t sweep_launch_smem(const grophecy_space *s)
{
    return std::max<uint32_t>(sweep_smem_bytes(s->max_wslots, s->usage_tbl_bytes), (uint32_t)sizeof(CtaSmem));
}

// Persistent grid of the sweep kernel: every SM full (occupancy per space:
// its dynamic shared memory depends on the largest kernel count), at most one
// CTA per CTA tile (at least one: it lists the tail for pass 2).
static int sweep_grid(const grophecy_space *s, unsigned long long n)
{
    set_smem_attrs();
    if (!s->occ_sweep) {
        int o = 0;
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o, sweep_fn(s, false), THREADS, sweep_launch_smem(s));
        const_cast<grophecy_space *>(s)->occ_sweep = o < 1 ? 1 : o;
    }
    const unsigned long long swt = (unsigned long long)SW_GROUPS * s->sweep_cx;   // records per CTA tile
    const unsigned long long want = std::max<unsigned long long>(1ull, (n + swt - 1) / swt);
    unsigned long long cap = (unsigned long long)s->grid_best * (unsigned long long)s->occ_sweep;
    if (cap > s->max_partials - 1) cap = s->max_partials - 1;   // last slot = result
    // test hook: a small grid makes every CTA run many tiles in sequence
    if (s->sweep_grid_env) cap = std::min<unsigned long long>(cap, s->sweep_grid_env);
    return (int)std::min(want, cap);
}

// One projection = per chunk of at most GROPHECY_TILE_CAP tiles: reset the
// tile list, pass 1 (canonical tiles), pass 2 (the listed tiles).  Best mode
// accumulates the chunks into P.out.
template <bool BEST>
static int launch_passes(const grophecy_space *s, Params P, cudaStream_t st)
{
    const unsigned long long cap = (unsigned long long)GROPHECY_TILE_CAP * CTILE;
    const unsigned long long n = P.n;
    // canonical groups sit at global indices that are multiples of their
    // size (CX = 16 for the eval kernel, the space's sweep_cx for best mode);
    // a batch starting inside a group (e.g. a shard boundary) projects its
    // head on its own so the tiles of the rest stay aligned
    const unsigned long long gcx = BEST ? s->sweep_cx : (unsigned long long)CX;
    const unsigned long long head = (gcx - P.base % gcx) % gcx;
    unsigned long long off = 0;
    do {
        Params Q = P;
        Q.n = off == 0 && head ? std::min(head, n) : std::min(cap, n - off);
        Q.skx += off; Q.nx += off; Q.ny += off; Q.iters += off;
        Q.base += off;
        {
            const uintptr_t m = (uintptr_t)Q.skx | (uintptr_t)Q.nx | (uintptr_t)Q.ny | (uintptr_t)Q.iters;
            Q.aligned = (m & 15u) == 0;   // this chunk's records (vector loads, TMA)
        }
        if (!BEST) {
            Q.h2d += off; Q.d2h += off; Q.t += off;
            if (Q.p_iter) Q.p_iter += off;
            if (Q.p_once) Q.p_once += off;
            if (Q.p_h2d) Q.p_h2d += off;
            if (Q.p_d2h) Q.p_d2h += off;
        } else if (off) {
            Q.accumulate = 1;
        }
        // count + claim counters: zero after space creation and after every
        // best projection (its pass 2 resets them); eval leaves them dirty
        grophecy_space *sm_ = const_cast<grophecy_space *>(s);
        cudaError_t e = cudaSuccess;
        if (!BEST || !sm_->counters_clean) {
            e = cudaMemsetAsync(Q.tile_count, 0, (std::max(CLAIM1, CLAIM2) + 1) * sizeof(unsigned int), st);
            if (e != cudaSuccess) return cuda_fail(e, "cudaMemsetAsync(tile count)");
        }
        const int grid = grid_for(s, Q.n, 32, false);
        Q.canon_warp_bytes = canon_warp_bytes(s->max_kernels);
        Q.reset_counters = 0;   // (pass 2 only, below: pass 1's list must survive pass 1)
        // batches the sweep takes nothing of (unaligned, the memory choice) and
        // batches smaller than one tile (pass 2 alone is quicker) go to pass 2 whole
        Q.direct = BEST && !(Q.aligned && !Q.pr.mem && Q.n >= (unsigned long long)SW_GROUPS * s->sweep_cx &&
                             sweep_launch_smem(s) <= SMEM_CTA_MAX);
        int launches = 1;
        Q.fused = 0;
        if (BEST && !Q.direct && GROPHECY_FUSED) {
            // passes 1 and 2 in one cooperative launch: CTA sweep tiles
            // (canonical layouts, one skeleton per tile), a grid barrier, then
            // the listed tiles on the general path
            Q.sweep_kmax = s->max_wslots;
            Q.fused = 1;
            Q.reset_counters = 1;
            cudaLaunchConfig_t cfg = {};
            cfg.blockDim = dim3(THREADS);
            cfg.stream = st;
            cudaLaunchAttribute attr[1];
            attr[0].id = cudaLaunchAttributeCooperative;
            attr[0].val.cooperative = 1;
            cfg.attrs = attr;
            cfg.numAttrs = 1;
            cfg.gridDim = dim3(sweep_grid(s, Q.n));
            cfg.dynamicSmemBytes = sweep_launch_smem(s);
            e = cudaLaunchKernelEx(&cfg, sweep_fn(s, sweep_two(s, Q.n)), Q);
            if (e != cudaSuccess) return cuda_fail(e, "projection (best) sweep launch");
            sm_->counters_clean = true;
            count_launch(1);
            off += Q.n;
            continue;
        } else if (BEST && !Q.direct) {
            // pass 1 alone (pass 2 launched below, programmatically dependent)
            const int grid_s = sweep_grid(s, Q.n);
            Q.sweep_kmax = s->max_wslots;
            sweep_fn(s, sweep_two(s, Q.n))<<<grid_s, THREADS, sweep_launch_smem(s), st>>>(Q);
            launches++;
        } else if (!BEST) {
            const int grid_c = grid_for(s, Q.n, 32, true);
            canon_kernel<false><<<grid_c, THREADS, WARPS * Q.canon_warp_bytes, st>>>(Q);
            launches++;
        }
        if (!(BEST && Q.direct)) Q.accumulate = BEST ? 1 : 0;   // pass 2 merges into pass 1's result
        if (BEST) {
            Q.reset_counters = 1;
            // programmatic dependent launch: pass 2's launch overlaps pass 1
            cudaLaunchConfig_t cfg = {};
            cfg.gridDim = dim3(grid);
            cfg.blockDim = dim3(THREADS);
            cfg.dynamicSmemBytes = sizeof(CtaSmem);
            cfg.stream = st;
            cudaLaunchAttribute attr[1];
            attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
            attr[0].val.programmaticStreamSerializationAllowed = Q.direct ? 0 : 1;
            cfg.attrs = attr;
            cfg.numAttrs = 1;
            e = cudaLaunchKernelEx(&cfg, general_kernel<true>, Q);
            if (e != cudaSuccess) return cuda_fail(e, "projection (best) pass 2 launch");
            sm_->counters_clean = true;
        } else {
            general_kernel<BEST><<<grid, THREADS, sizeof(CtaSmem), st>>>(Q);
            sm_->counters_clean = false;
        }
        count_launch(launches);
        e = cudaGetLastError();
        if (e != cudaSuccess) return cuda_fail(e, BEST ? "projection (best) launch" : "projection (eval) launch");
        off += Q.n;
    } while (off < n);
    return GROPHECY_OK;
}

static int check_batch(const grophecy_space *s, const grophecy_pcie *pc, const grophecy_batch *b)
{
    if (!s || !pc || !b) {
        set_error("null argument");
        return GROPHECY_EINVAL;
    }
    if (b->n && (!b->skx || !b->nx || !b->ny || !b->iters)) {
        set_error("null record array");
        return GROPHECY_EINVAL;
    }
    if (b->stripe_len && b->stripe_stride < b->stripe_len) {
        set_error("stripe_stride < stripe_len");
        return GROPHECY_EINVAL;
    }
    return GROPHECY_OK;
}

static Params make_params(const grophecy_space *s, const grophecy_pcie *pc, const grophecy_batch *b)
{
    Params P;
    P.S = s->dev;
    P.gS = s->dev_copy;
    P.pc = *pc;
    P.pr.pc = *pc;
    P.pr.mem = 0;
    memset(&P.pr.mm, 0, sizeof P.pr.mm);
    P.skx = b->skx;
    P.nx = b->nx;
    P.ny = b->ny;
    P.iters = b->iters;
    P.n = b->n;
    P.base = b->index_base;
    P.map_len = b->stripe_len;
    P.map_stride = b->stripe_stride;
    P.map_base = b->index_base;
    if (b->stripe_len) P.base = 0;   // batch-local indices (launch_best adds the local offset)
    P.h2d = nullptr;
    P.d2h = nullptr;
    P.t = nullptr;
    P.p_iter = P.p_once = P.p_h2d = P.p_d2h = nullptr;
    P.partials = s->partials;
    P.ticket = s->ticket;
    P.out = nullptr;
    P.accumulate = 0;
    P.tile_list = s->tile_list;
    P.tile_count = s->tile_count;
    P.canon_warp_bytes = canon_warp_bytes(s->max_kernels);
    const uintptr_t m = (uintptr_t)b->skx | (uintptr_t)b->nx | (uintptr_t)b->ny | (uintptr_t)b->iters;
    P.aligned = (m & 15u) == 0;
    return P;
}

int launch_best(grophecy_space *s, const grophecy_pcie *pc, const grophecy_batch *b,
                grophecy_best_result *dout, int accumulate, cudaStream_t st, uint64_t local_off)
{
    DeviceGuard guard(s->device);
    Params P = make_params(s, pc, b);
    if (P.map_len) P.base = local_off;
    P.out = dout;
    P.accumulate = accumulate;
    return launch_passes<true>(s, P, st);
}

}  // namespace grophecy

using namespace grophecy;

extern "C" {

int grophecy_eval_parts(const grophecy_space *s, const grophecy_pcie *pc, const grophecy_batch *b,
                        uint64_t *h2d, uint64_t *d2h, double *t, const grophecy_parts *parts,
                        void *stream)
{
    int rc = check_batch(s, pc, b);
    if (rc) return rc;
    if (b->n == 0) return GROPHECY_OK;
    if (!h2d || !d2h || !t) {
        set_error("null output array");
        return GROPHECY_EINVAL;
    }
    Params P = make_params(s, pc, b);
    P.h2d = (unsigned long long *)h2d;
    P.d2h = (unsigned long long *)d2h;
    P.t = t;
    DeviceGuard guard(s->device);
    if (parts) {
        P.p_iter = parts->t_iter_s;
        P.p_once = parts->t_once_s;
        P.p_h2d = parts->t_h2d_s;
        P.p_d2h = parts->t_d2h_s;
    }
    return launch_passes<false>(s, P, (cudaStream_t)stream);
}

int grophecy_eval(const grophecy_space *s, const grophecy_pcie *pc, const grophecy_batch *b,
                  uint64_t *h2d, uint64_t *d2h, double *t, void *stream)
{
    return grophecy_eval_parts(s, pc, b, h2d, d2h, t, nullptr, stream);
}

static int status_of(const grophecy_best_result &r);

// NEXT-4 (reading 17): the projection with every array's pinned /
// pageable choice; the general path prices it (mem_terms).
static int mem_params(const grophecy_space *s, const grophecy_memory_model *m,
                      const grophecy_batch *b, Params &P)
{
    if (!m) {
        set_error("null memory model");
        return GROPHECY_EINVAL;
    }
    int rc = check_batch(s, &m->pinned, b);
    if (rc) return rc;
    P = make_params(s, &m->pinned, b);
    P.pr.mm = *m;
    P.pr.mem = 1;
    return GROPHECY_OK;
}

int grophecy_eval_mem(const grophecy_space *s, const grophecy_memory_model *m,
                      const grophecy_batch *b, uint64_t *h2d, uint64_t *d2h, double *t,
                      const grophecy_parts *parts, void *stream)
{
    Params P;
    int rc = mem_params(s, m, b, P);
    if (rc) return rc;
    if (b->n == 0) return GROPHECY_OK;
    if (!h2d || !d2h || !t) {
        set_error("null output array");
        return GROPHECY_EINVAL;
    }
    DeviceGuard guard(s->device);
    P.h2d = (unsigned long long *)h2d;
    P.d2h = (unsigned long long *)d2h;
    P.t = t;
    if (parts) {
        P.p_iter = parts->t_iter_s;
        P.p_once = parts->t_once_s;
        P.p_h2d = parts->t_h2d_s;
        P.p_d2h = parts->t_d2h_s;
    }
    return launch_passes<false>(s, P, (cudaStream_t)stream);
}

int grophecy_best_mem(grophecy_space *s, const grophecy_memory_model *m, const grophecy_batch *b,
                      grophecy_best_result *host_out, void *stream)
{
    Params P;
    int rc = mem_params(s, m, b, P);
    if (rc) return rc;
    if (!host_out) {
        set_error("null host_out");
        return GROPHECY_EINVAL;
    }
    DeviceGuard guard(s->device);
    cudaStream_t st = (cudaStream_t)stream;
    grophecy_best_result *dres = s->partials + (s->max_partials - 1);
    P.out = dres;
    P.accumulate = 0;
    rc = launch_passes<true>(s, P, st);
    if (rc) return rc;
    cudaError_t e = cudaMemcpyAsync(host_out, dres, sizeof *host_out, cudaMemcpyDeviceToHost, st);
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    if (e != cudaSuccess) return cuda_fail(e, "grophecy_best_mem");
    return status_of(*host_out);
}

int grophecy_best_async(grophecy_space *s, const grophecy_pcie *pc, const grophecy_batch *b,
                        grophecy_best_result *dout, int accumulate, void *stream)
{
    int rc = check_batch(s, pc, b);
    if (rc) return rc;
    if (!dout) {
        set_error("null device_out");
        return GROPHECY_EINVAL;
    }
    return launch_best(s, pc, b, dout, accumulate, (cudaStream_t)stream);
}

static int status_of(const grophecy_best_result &r)
{
    if (r.index == ~0ull) {
        set_error("no valid candidate with finite projected time");
        return GROPHECY_ENOFEASIBLE;
    }
    if (r.n_invalid) {
        set_error("batch contains invalid records");
        return GROPHECY_EBADCAND;
    }
    return GROPHECY_OK;
}

int grophecy_best(grophecy_space *s, const grophecy_pcie *pc, const grophecy_batch *b,
                  grophecy_best_result *host_out, void *stream)
{
    int rc = check_batch(s, pc, b);
    if (rc) return rc;
    if (!host_out) {
        set_error("null host_out");
        return GROPHECY_EINVAL;
    }
    cudaStream_t st = (cudaStream_t)stream;
    // the result slot lives in the space's scratch, after the partials
    DeviceGuard guard(s->device);
    grophecy_best_result *dres = s->partials + (s->max_partials - 1);
    rc = launch_best(s, pc, b, dres, 0, st);
    if (rc) return rc;
    cudaError_t e = cudaMemcpyAsync(host_out, dres, sizeof *host_out, cudaMemcpyDeviceToHost, st);
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    if (e != cudaSuccess) return cuda_fail(e, "grophecy_best");
    return status_of(*host_out);
}

// Diagnostic builds (GROPHECY_PHASE_TIMING=1): copy out and reset the sweep
// kernel's per-phase cycle sums (warp-cycles); ENOTSUP-like EINVAL otherwise.
int grophecy_debug_phase_cycles(uint64_t *out8)
{
#if GROPHECY_PHASE_TIMING
    if (!out8) return GROPHECY_EINVAL;
    cudaError_t e = cudaMemcpyFromSymbol(out8, g_phase_cycles, 8 * sizeof(uint64_t));
    if (e == cudaSuccess) {
        static const unsigned long long zero[8] = {};
        e = cudaMemcpyToSymbol(g_phase_cycles, zero, sizeof zero);
    }
    return e == cudaSuccess ? GROPHECY_OK : cuda_fail(e, "phase cycles");
#else
    (void)out8;
    set_error("built without GROPHECY_PHASE_TIMING");
    return GROPHECY_EINVAL;
#endif
}

int grophecy_best_combine(const grophecy_best_result *din, uint32_t count,
                          grophecy_best_result *dout, void *stream)
{
    if (!dout || (count && !din)) {
        set_error("null argument");
        return GROPHECY_EINVAL;
    }
    combine_kernel<<<1, 32, 0, (cudaStream_t)stream>>>(din, count, dout);
    count_launch();
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e, "combine_kernel launch");
    return GROPHECY_OK;
}

// End-to-end path with host records: chunked H2D copies on a copy stream,
// double-buffered, overlapped with the fused kernel on the caller's stream;
// one accumulating result slot; one D2H of 48 bytes at the end.
int grophecy_best_host(grophecy_space *s, const grophecy_pcie *pc, const grophecy_batch *hb,
                       grophecy_best_result *host_out, void *stream)
{
    if (!s || !pc || !hb || !host_out || (hb->n && (!hb->skx || !hb->nx || !hb->ny || !hb->iters))) {
        set_error("null argument");
        return GROPHECY_EINVAL;
    }
    if (hb->stripe_len && hb->stripe_stride < hb->stripe_len) {
        set_error("stripe_stride < stripe_len");
        return GROPHECY_EINVAL;
    }
    const uint32_t *skx = hb->skx, *nx = hb->nx, *ny = hb->ny, *iters = hb->iters;
    const uint64_t n = hb->n;
    cudaStream_t st = (cudaStream_t)stream;
    cudaError_t e;
    DeviceGuard guard(s->device);
    const uint64_t CHUNK = 1ull << 23;   // records per chunk (128 MiB of records)
    const size_t need = (size_t)CHUNK * 16;
    if (!s->copy_stream) {
        if ((e = cudaStreamCreateWithFlags(&s->copy_stream, cudaStreamNonBlocking)) != cudaSuccess)
            return cuda_fail(e, "cudaStreamCreate");
        for (int i = 0; i < 2; i++) {
            cudaEventCreateWithFlags(&s->ev_copied[i], cudaEventDisableTiming);
            cudaEventCreateWithFlags(&s->ev_done[i], cudaEventDisableTiming);
        }
    }
    if (s->stage_bytes < need) {
        for (int i = 0; i < 2; i++) {
            if (s->stage[i]) cudaFree(s->stage[i]);
            s->stage[i] = nullptr;
            if ((e = cudaMalloc(&s->stage[i], need)) != cudaSuccess) return cuda_fail(e, "cudaMalloc(stage)");
        }
        s->stage_bytes = need;
    }
    grophecy_best_result *dres = s->partials + (s->max_partials - 1);
    grophecy_best_result init;
    grophecy_best_combine_host(nullptr, 0, &init);
    if ((e = cudaMemcpyAsync(dres, &init, sizeof init, cudaMemcpyHostToDevice, st)) != cudaSuccess)
        return cuda_fail(e, "init result");
    // copies of chunk c may start once the kernel of chunk c-2 finished
    cudaEventRecord(s->ev_done[0], st);
    cudaEventRecord(s->ev_done[1], st);
    for (uint64_t off = 0, c = 0; off < n; off += CHUNK, c++) {
        const uint64_t m = std::min<uint64_t>(CHUNK, n - off);
        const int slot = (int)(c & 1);
        uint32_t *buf = (uint32_t *)s->stage[slot];
        cudaStreamWaitEvent(s->copy_stream, s->ev_done[slot], 0);
        const uint32_t *src[4] = {skx, nx, ny, iters};
        for (int f = 0; f < 4; f++) {
            e = cudaMemcpyAsync(buf + (size_t)f * CHUNK, src[f] + off, m * 4, cudaMemcpyHostToDevice,
                                s->copy_stream);
            if (e != cudaSuccess) return cuda_fail(e, "H2D chunk");
        }
        cudaEventRecord(s->ev_copied[slot], s->copy_stream);
        cudaStreamWaitEvent(st, s->ev_copied[slot], 0);
        // the chunk is records [off, off + m) of the host batch: same index
        // map, local offset off
        grophecy_batch b = {buf, buf + CHUNK, buf + 2 * CHUNK, buf + 3 * CHUNK, m,
                            hb->index_base, hb->stripe_len, hb->stripe_stride};
        if (!hb->stripe_len) b.index_base = hb->index_base + off;
        int rc = launch_best(s, pc, &b, dres, 1, st, hb->stripe_len ? off : 0);
        if (rc) return rc;
        cudaEventRecord(s->ev_done[slot], st);
    }
    e = cudaMemcpyAsync(host_out, dres, sizeof *host_out, cudaMemcpyDeviceToHost, st);
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    if (e != cudaSuccess) return cuda_fail(e, "grophecy_best_host");
    return status_of(*host_out);
}

}  // extern "C"
