#include <cstdlib>
// Host side of the C ABI: PCIe fit, design-space validation, per-(kernel,
// transformation) constant precompute and device upload.
//
// Compiled with -ffp-contract=off: every double expression below is evaluated
// exactly as written (DESIGN.md §3 N1) so that the constants the GPU consumes
// are bitwise the values the definition produces.
#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <cmath>
#include <cstdio>
#include <climits>
#include <cstring>
#include <string>
#include <vector>

#include "grophecy.h"
#include "internal.h"

namespace grophecy {

static thread_local std::string g_err;
static std::atomic<uint64_t> g_launches{0};

void set_error(const std::string &msg) { g_err = msg; }

int cuda_fail(cudaError_t e, const char *what)
{
    set_error(std::string(what) + ": " + cudaGetErrorString(e));
    return GROPHECY_ECUDA;
}

void count_launch(uint64_t n) { g_launches.fetch_add(n, std::memory_order_relaxed); }

static int fail(int code, const std::string &msg)
{
    set_error(msg);
    return code;
}

static double dmin(double a, double b) { return a < b ? a : b; }

static bool fin_nonneg(double v) { return std::isfinite(v) && v >= 0.0; }

static bool coef_ok(const grophecy_affine8 &a)
{
    const int32_t L = 1 << 15;
    return a.c1 >= -L && a.c1 <= L && a.c2 >= -L && a.c2 <= L && a.c3 >= -L && a.c3 <= L;
}

// lcm(l, step) with step 0 / 1 = dense
static uint64_t lcm_step(uint64_t l, uint32_t step)
{
    const uint64_t s = step > 1 ? step : 1;
    uint64_t a = l, b = s;
    while (b) { const uint64_t t = a % b; a = b; b = t; }
    return l / a * s;
}

static int validate(const grophecy_skeleton_desc *skels, uint32_t n_skels,
                    const grophecy_gpu_model *g)
{
    if (!skels || !g) return fail(GROPHECY_EINVAL, "null skeleton array or gpu model");
    if (n_skels < 1) return fail(GROPHECY_EINVAL, "n_skels must be >= 1");
    if (n_skels > GROPHECY_MAX_SKELS) return fail(GROPHECY_ELIMIT, "too many skeletons");
    if (g->n_sm < 1 || g->warp_size < 1 || g->max_threads_per_block < 1 ||
        g->max_blocks_per_sm < 1 || g->max_threads_per_sm < 1 || g->regs_per_sm < 1 ||
        g->smem_per_sm < 1)
        return fail(GROPHECY_EINVAL, "gpu model integers must be >= 1");
    const double gd[] = {g->freq_hz, g->mem_bw_Bps, g->mem_ld_cycles, g->dep_del_coal,
                         g->dep_del_uncoal, g->issue_cycles};
    for (double v : gd)
        if (!std::isfinite(v) || !(v > 0.0))
            return fail(GROPHECY_EINVAL, "gpu model doubles must be finite and > 0");
    for (uint32_t s = 0; s < n_skels; s++) {
        const grophecy_skeleton_desc &S = skels[s];
        char where[64];
        snprintf(where, sizeof where, "skeleton %u: ", s);
        if (S.n_kernels < 1 || S.n_xforms < 1)
            return fail(GROPHECY_EINVAL, std::string(where) + "needs >= 1 kernel and transformation");
        if (S.n_kernels > GROPHECY_MAX_KERNELS) return fail(GROPHECY_ELIMIT, std::string(where) + "too many kernels");
        if (S.n_arrays > GROPHECY_MAX_ARRAYS) return fail(GROPHECY_ELIMIT, std::string(where) + "too many arrays");
        if (S.n_regions > GROPHECY_MAX_REGIONS) return fail(GROPHECY_ELIMIT, std::string(where) + "too many regions");
        if (S.n_xforms > GROPHECY_MAX_XFORMS) return fail(GROPHECY_ELIMIT, std::string(where) + "too many transformations");
        if (!S.kernels || !S.kx || (S.n_arrays && !S.arrays) || (S.n_regions && !S.regions))
            return fail(GROPHECY_EINVAL, std::string(where) + "null table");
        for (uint32_t k = 0; k < S.n_kernels; k++)
            if (!coef_ok(S.kernels[k].work_items))
                return fail(GROPHECY_ELIMIT, std::string(where) + "work coefficient out of range");
        for (uint32_t a = 0; a < S.n_arrays; a++) {
            if (!coef_ok(S.arrays[a].rows) || !coef_ok(S.arrays[a].cols) ||
                !coef_ok(S.arrays[a].planes))
                return fail(GROPHECY_ELIMIT, std::string(where) + "extent coefficient out of range");
            if (S.arrays[a].elem_bytes < 1)
                return fail(GROPHECY_EINVAL, std::string(where) + "elem_bytes must be >= 1");
        }
        std::vector<uint32_t> per_array(S.n_arrays, 0);
        for (uint32_t j = 0; j < S.n_regions; j++) {
            const grophecy_region_desc &r = S.regions[j];
            if (r.kernel >= S.n_kernels || r.array >= S.n_arrays)
                return fail(GROPHECY_EINVAL, std::string(where) + "region kernel/array index out of range");
            if (r.mode < 1 || r.mode > 3)
                return fail(GROPHECY_EINVAL, std::string(where) + "region mode must be R, W or R|W");
            if (r.r_step > GROPHECY_MAX_STEP || r.c_step > GROPHECY_MAX_STEP)
                return fail(GROPHECY_ELIMIT, std::string(where) + "region step > 64");
            if (!coef_ok(r.r0) || !coef_ok(r.r1) || !coef_ok(r.c0) || !coef_ok(r.c1) ||
                !coef_ok(r.p0) || !coef_ok(r.p1))
                return fail(GROPHECY_ELIMIT, std::string(where) + "region coefficient out of range");
            if (++per_array[r.array] > GROPHECY_MAX_REGIONS_PER_ARRAY)
                return fail(GROPHECY_ELIMIT, std::string(where) + "more than 32 regions on one array");
        }
        if (S.flags & ~(uint32_t)GROPHECY_SKEL_HULL)
            return fail(GROPHECY_EINVAL, std::string(where) + "unknown skeleton flags");
        if (S.reserved) return fail(GROPHECY_EINVAL, std::string(where) + "reserved must be 0");
        for (uint32_t a = 0; a < S.n_arrays; a++) {
            uint64_t lr = 1, lc = 1;
            for (uint32_t j = 0; j < S.n_regions; j++) {
                const grophecy_region_desc &r = S.regions[j];
                if (r.array != a || (r.flags & GROPHECY_REGION_WHOLE)) continue;
                lr = lcm_step(lr, r.r_step);
                lc = lcm_step(lc, r.c_step);
            }
            if (lr > GROPHECY_MAX_STEP_LCM || lc > GROPHECY_MAX_STEP_LCM)
                return fail(GROPHECY_ELIMIT, std::string(where) + "lcm of an array's steps > 64");
        }
        for (uint64_t i = 0; i < (uint64_t)S.n_xforms * S.n_kernels; i++) {
            const grophecy_kx_desc &c = S.kx[i];
            if (c.tpb < 1 || c.ipt < 1 || c.tpb > 65536u || c.ipt > 65536u ||
                (uint64_t)c.tpb * c.ipt > 0xffffffffull)
                return fail(GROPHECY_ELIMIT, std::string(where) + "tpb/ipt out of range");
            if (!fin_nonneg(c.total_insts) || !fin_nonneg(c.coal_insts) ||
                !fin_nonneg(c.uncoal_insts) || !fin_nonneg(c.synch_insts) ||
                !std::isfinite(c.uncoal_per_mw) || !std::isfinite(c.load_bytes_per_warp))
                return fail(GROPHECY_EINVAL, std::string(where) + "instruction counts must be finite and >= 0");
            if (c.total_insts < c.coal_insts + c.uncoal_insts)
                return fail(GROPHECY_EINVAL, std::string(where) + "total_insts < coal + uncoal");
            if (!(c.uncoal_per_mw >= 1.0) || !(c.load_bytes_per_warp > 0.0))
                return fail(GROPHECY_EINVAL, std::string(where) + "uncoal_per_mw must be >= 1, load_bytes_per_warp > 0");
        }
    }
    return GROPHECY_OK;
}

// Per-(kernel, transformation) constants — DESIGN.md §3 N5 part A, plus the
// saturated-grid reduction of part B.  Same operation order as the definition.
static void precompute(const grophecy_kx_desc &c, const grophecy_gpu_model &g, KxES &es,
                       KxD &dd_, KxI &ii, KxJ &jj, KxG &gg)
{
    uint64_t occ;
    if (c.tpb > g.max_threads_per_block) {
        occ = 0;
    } else {
        occ = std::min<uint64_t>(g.max_blocks_per_sm, g.max_threads_per_sm / c.tpb);
        if (c.regs_per_thread > 0)
            occ = std::min<uint64_t>(occ, g.regs_per_sm / ((uint64_t)c.regs_per_thread * c.tpb));
        if (c.smem_per_block > 0) occ = std::min<uint64_t>(occ, g.smem_per_sm / c.smem_per_block);
    }
    uint64_t wpb = c.tpb / g.warp_size + (c.tpb % g.warp_size != 0);
    uint64_t ipb = (uint64_t)c.tpb * c.ipt;
    double mem = c.coal_insts + c.uncoal_insts;
    double comp = g.issue_cycles * c.total_insts;

    std::memset(&gg, 0, sizeof gg);
    gg.comp = comp;
    gg.synch = c.synch_insts;
    jj.ipb = (uint32_t)ipb;
    jj.occ = (uint32_t)occ;
    jj.wpb = (uint32_t)wpb;
    jj.flags = (occ == 0 ? KXF_INFEASIBLE : 0u) | (mem == 0.0 ? KXF_NOMEM : 0u);
    ii.magic = ipb == 1 ? 0 : (~0ull) / ipb + 1;   // ceil(2^64 / ipb)
    if (mem != 0.0) {
        double mlu = g.mem_ld_cycles + (c.uncoal_per_mw - 1.0) * g.dep_del_uncoal;
        double mlc = g.mem_ld_cycles;
        double wu = c.uncoal_insts / mem;
        double wc = c.coal_insts / mem;
        double ml = mlu * wu + mlc * wc;
        double dd = (g.dep_del_uncoal * c.uncoal_per_mw) * wu + g.dep_del_coal * wc;
        double mwp0 = ml / dd;
        double bwpw = g.freq_hz * c.load_bytes_per_warp / ml;
        double bwr = g.mem_bw_Bps / bwpw;
        double memc = mlu * c.uncoal_insts + mlc * c.coal_insts;
        double cwpf = (memc + comp) / comp;
        double cpm = comp / mem;
        gg.mwp0 = mwp0; gg.bwr = bwr; gg.memc = memc; gg.cwpf = cwpf; gg.cpm = cpm;
        gg.ml = ml; gg.dd = dd;
    }
    if (occ == 0) {
        es = {0.0, 0.0};
        dd_ = {1.0, 1.0};
        ii.sat_blocks = ~0ull;
        return;
    }
    // Saturated grid: blocks >= n_sm and ceil(blocks / n_sm) >= occ.
    uint64_t nsm = g.n_sm;
    ii.sat_blocks = std::max<uint64_t>(nsm, (occ - 1) * nsm + 1);
    double N = (double)(occ * wpb);
    double D = (double)(occ * nsm);
    dd_.D = D;
    dd_.rD = 1.0 / D;
    if (mem == 0.0) {
        es.E = comp * N;
        es.S = 0.0;
        return;
    }
    double mpk = gg.bwr / (double)nsm;
    double mwp = dmin(dmin(gg.mwp0, mpk), N);
    double cwp = dmin(gg.cwpf, N);
    if (mwp == N && cwp == N)
        es.E = gg.memc + comp + gg.cpm * (mwp - 1.0);
    else if (cwp >= mwp || comp > gg.memc)
        es.E = gg.memc * N / mwp + gg.cpm * (mwp - 1.0);
    else
        es.E = gg.ml + comp * N;
    es.S = gg.dd * (mwp - 1.0) * c.synch_insts * (double)occ;
}

// The two-product division x / v = RN(x * hi + RN(x * lo)), hi = RN(1/v),
// lo = RN(1/v - hi) (the residual 1 - v * hi is exact by FMA), is bitwise the
// IEEE quotient for every double x (normal operands) when the odd part of v's
// significand is below 2^50: x / v then lies at least ulp / (2 * odd) from
// every rounding midpoint while the unevaluated sum errs by at most
// ulp * 2^-52.  div2_ok checks the condition.
static bool div2_ok(double v)
{
    if (!(v > 0.0) || !std::isfinite(v)) return false;
    int e = 0;
    uint64_t M = (uint64_t)std::ldexp(std::frexp(v, &e), 53);   // exact 53-bit significand
    while (!(M & 1u)) M >>= 1;
    return M < (1ull << 50);
}
static void split_recip(double v, double &hi, double &lo)
{
    hi = 1.0 / v;
    lo = std::fma(-v, hi, 1.0) / v;
}
// Saturated constants usable by the fast path: zero or normal and far from
// overflow, so every product of the two-product divisions stays normal.
static bool fast_const_ok(double c) { return c == 0.0 || (c >= 0x1p-900 && c <= 0x1p+900); }

// Kernel time on a grid of `blocks` < sat_blocks blocks: the general branch of
// DESIGN.md §3 N5 step by step, in the definition's operation order (the same
// order as the device's kernel_time and the oracle).  Tabulated at space
// creation: on such grids the time depends on (kernel, xform, blocks) only.
static double small_grid_time(const KxJ &J, const KxG &G, uint64_t nsm, double freq,
                              uint64_t blocks)
{
    if (blocks == 0) return 0.0;
    const uint64_t asm_ = std::min<uint64_t>(nsm, blocks);
    uint64_t abps = blocks / asm_ + (blocks % asm_ != 0);
    if ((uint64_t)J.occ < abps) abps = J.occ;
    const double N = (double)(abps * (uint64_t)J.wpb);
    const double rep = (double)blocks / (double)(abps * asm_);
    double cyc;
    if (J.flags & KXF_NOMEM) {
        cyc = G.comp * N * rep;
    } else {
        const double mpk = G.bwr / (double)asm_;
        const double mwp = dmin(dmin(G.mwp0, mpk), N);
        const double cwp = dmin(G.cwpf, N);
        const double cpm_term = G.cpm * (mwp - 1.0);
        if (mwp == N && cwp == N)
            cyc = (G.memc + G.comp + cpm_term) * rep;
        else if (cwp >= mwp || G.comp > G.memc)
            cyc = (G.memc * N / mwp + cpm_term) * rep;
        else
            cyc = (G.ml + G.comp * N) * rep;
        const double sync = G.dd * (mwp - 1.0) * G.synch * (double)abps * rep;
        cyc = cyc + sync;
    }
    return cyc / freq;
}

}  // namespace grophecy

using namespace grophecy;

extern "C" {

int grophecy_abi_version(void) { return GROPHECY_ABI_VERSION; }

const char *grophecy_last_error(void) { return g_err.c_str(); }

uint64_t grophecy_launch_count(void) { return g_launches.load(); }

int grophecy_fit_pcie(double t_small_s, double t_large_s, uint64_t large_bytes,
                      grophecy_link *out)
{
    if (!out) return fail(GROPHECY_EINVAL, "out is NULL");
    if (!std::isfinite(t_small_s) || !std::isfinite(t_large_s) || t_small_s < 0.0 ||
        !(t_large_s > 0.0) || large_bytes == 0)
        return fail(GROPHECY_EINVAL, "need finite t_small >= 0, t_large > 0, large_bytes > 0");
    out->alpha_s = t_small_s;
    out->beta_s_per_byte = t_large_s / (double)large_bytes;
    return GROPHECY_OK;
}

double grophecy_pcie_time(const grophecy_link *link, uint64_t bytes)
{
    if (!link || bytes == 0) return 0.0;
    return link->alpha_s + link->beta_s_per_byte * (double)bytes;
}

double grophecy_speedup(double t_cpu_s, double t_gpu_s) { return t_cpu_s / t_gpu_s; }

double grophecy_error_magnitude(double predicted, double measured)
{
    return std::fabs(predicted - measured) / measured;
}

double grophecy_mean(const double *values, uint64_t n)
{
    if (!values || n == 0) return NAN;
    double s = 0.0;
    for (uint64_t i = 0; i < n; i++) s += values[i];
    return s / (double)n;
}

int grophecy_space_validate(const grophecy_skeleton_desc *skels, uint32_t n_skels,
                            const grophecy_gpu_model *gpu)
{
    return validate(skels, n_skels, gpu);
}

static size_t align_up(size_t v, size_t a) { return (v + a - 1) / a * a; }

int grophecy_space_create(const grophecy_skeleton_desc *skels, uint32_t n_skels,
                          const grophecy_gpu_model *gpu, int device, grophecy_space **out)
{
    if (!out) return fail(GROPHECY_EINVAL, "out is NULL");
    *out = nullptr;
    int rc = validate(skels, n_skels, gpu);
    if (rc) return rc;

    // ---- host tables ----
    std::vector<SkelInfo> info(n_skels);
    std::vector<int4> kwork;
    std::vector<uint32_t> kflags;
    std::vector<ArrayDev> arrays;
    std::vector<RegionDev> regions;
    std::vector<KxES> kes;
    std::vector<KxD> kd;
    std::vector<KxI> ki;
    std::vector<KxJ> kj;
    std::vector<KxG> kg;
    std::vector<KxFast> kf;
    std::vector<KxProg> kprog;    // sweep-kernel programs (all skeletons)
    std::vector<uint4> xhdr;      // per (skeleton, xform) at kx_base + x: program header
    std::vector<uint32_t> xord;   // per (skeleton, unit) at kx_base + u: xforms by descending cost
    std::vector<uint4> xhdru;     // the headers in that order
    std::vector<uint32_t> kwsat;  // per (skeleton, kernel): work count saturating every xform
    std::vector<int4> wslot_work;     // per (skeleton, work slot): the distinct work functions
    std::vector<uint32_t> wslot_sat;  // per (skeleton, work slot): max kwsat of its kernels
    std::vector<uint32_t> xinf;   // per (skeleton, xform) at kx_base + x: XINF_* bits
    // the fast path divides by freq with the two-product method: without it
    // (a frequency whose odd significand is >= 2^50) every pair takes the
    // general path's step-by-step definition
    const bool freq_ok = div2_ok(gpu->freq_hz);
    // poly[0..9]: an all-zero polynomial (the device reads it instead of the
    // polynomials that vanish in every class: unconditional loads)
    std::vector<unsigned long long> poly(POLY_ZERO_WORDS, 0ull);
    auto a4 = [](const grophecy_affine8 &a) { return make_int4(a.c0, a.c1, a.c2, a.c3); };
    for (uint32_t s = 0; s < n_skels; s++) {
        const grophecy_skeleton_desc &S = skels[s];
        SkelInfo &I = info[s];
        std::memset(&I, 0, sizeof I);
        I.n_kernels = S.n_kernels;
        I.n_arrays = S.n_arrays;
        I.n_xforms = S.n_xforms;
        I.n_regions = S.n_regions;
        I.k_base = (uint32_t)kwork.size();
        I.a_base = (uint32_t)arrays.size();
        I.kx_base = (uint32_t)kes.size();
        I.flags = S.flags & GROPHECY_SKEL_HULL;
        for (uint32_t j = 0; j < S.n_regions; j++)
            if (!(S.regions[j].flags & GROPHECY_REGION_WHOLE) &&
                (S.regions[j].r_step > 1 || S.regions[j].c_step > 1))
                I.flags |= SKF_STRIDED;
        if (skeleton_rank3(S)) I.flags |= SKF_RANK3;
        SkelPlanHost plan;
        if (compile_plan(S, plan)) {
            I.plan_tx = plan.tx;
            I.plan_ty = plan.ty;
            // keep every skeleton's table 16-byte aligned (2 coefficients)
            if (poly.size() & 1) poly.push_back(0);
            I.poly_base = (uint32_t)poly.size();
            I.poly_stride = plan.poly_stride;
            poly.insert(poly.end(), plan.poly.begin(), plan.poly.end());
            // polynomials that vanish in every size class price no transfer
            // (Eq. (1) is applied only to non-zero bytes) and are skipped
            I.poly_mask = 0;
            const size_t np = 2 * (size_t)S.n_arrays, st = plan.poly_stride;
            for (size_t c = 0; c < POLY_CLASSES; c++)
                for (size_t q = 0; q < np; q++)
                    for (size_t m = 0; m < st; m++)
                        if (plan.poly[(c * np + q) * st + m]) I.poly_mask |= 1u << q;
            // compact int32 copy (bilinear tables whose coefficients, read as
            // two's-complement int64, all fit int32): half the bytes per load
            I.poly32_base = POLY32_NONE;
            bool fits = st == 4;
            for (size_t i = 0; fits && i < plan.poly.size(); i++) {
                const int64_t v = (int64_t)plan.poly[i];
                fits = v >= INT32_MIN && v <= INT32_MAX;
            }
            if (fits) {
                I.poly32_base = (uint32_t)poly.size();   // even: 16-byte aligned
                for (size_t i = 0; i < plan.poly.size(); i += 4) {
                    uint64_t w[2];
                    const uint32_t c[4] = {(uint32_t)plan.poly[i], (uint32_t)plan.poly[i + 1],
                                           (uint32_t)plan.poly[i + 2], (uint32_t)plan.poly[i + 3]};
                    std::memcpy(w, c, sizeof w);
                    poly.push_back(w[0]);
                    poly.push_back(w[1]);
                }
            }
        } else {
            I.plan_tx = I.plan_ty = 0xffffffffu;   // never applicable
            I.poly_base = I.poly_stride = 0;
            I.poly_mask = 0;
            I.poly32_base = POLY32_NONE;
        }
        // the sweep kernel's copy of the bilinear int32 table, laid out
        // polynomial-major ([q][class]: lanes of different size classes read
        // different shared-memory banks): the H2D polynomials that are not
        // zero in every class, in array order, then the D2H ones, each list
        // padded with zero polynomials to a multiple of POLYF_AU (zero
        // polynomials price nothing: Eq. (1) is applied to non-zero bytes only)
        I.polyf_base = POLY32_NONE;
        I.polyf_nhd = 0;
        for (int m = 0; m < 4; m++) I.polyf_cmax[m] = 0xffffffffu;
        if (I.poly32_base != POLY32_NONE) {
            const size_t np = 2 * (size_t)S.n_arrays;
            std::vector<size_t> lists[2];
            for (size_t q = 0; q < np; q++)
                if ((I.poly_mask >> q) & 1u) lists[q & 1].push_back(q);
            size_t nl[2];
            for (int d = 0; d < 2; d++) nl[d] = (lists[d].size() + POLYF_AU - 1) / POLYF_AU * POLYF_AU;
            I.polyf_nhd = (uint32_t)nl[0] | (uint32_t)nl[1] << 16;
            for (int m = 0; m < 4; m++) {
                uint64_t mx = 0;
                for (int d = 0; d < 2; d++)
                    for (size_t q : lists[d])
                        for (size_t c = 0; c < POLY_CLASSES; c++) {
                            const int64_t v = (int32_t)(uint32_t)plan.poly[(c * np + q) * 4 + m];
                            mx = std::max<uint64_t>(mx, (uint64_t)(v < 0 ? -v : v));
                        }
                I.polyf_cmax[m] = (uint32_t)std::min<uint64_t>(mx, 0xffffffffull);
            }
            I.polyf_base = (uint32_t)poly.size();   // even: 16-byte aligned
            for (int d = 0; d < 2; d++)
                for (size_t i = 0; i < nl[d]; i++)
                    for (size_t c = 0; c < POLY_CLASSES; c++) {
                        uint32_t w4[4] = {0u, 0u, 0u, 0u};
                        if (i < lists[d].size())
                            for (int m = 0; m < 4; m++) w4[m] = (uint32_t)plan.poly[(c * np + lists[d][i]) * 4 + m];
                        uint64_t w[2];
                        std::memcpy(w, w4, sizeof w);
                        poly.push_back(w[0]);
                        poly.push_back(w[1]);
                    }
        }
        I.per_iter_mask = 0;
        for (uint32_t k = 0; k < S.n_kernels; k++)
            if (S.kernels[k].flags & GROPHECY_KERNEL_PER_ITER) I.per_iter_mask |= 1u << k;
        for (uint32_t k = 0; k < S.n_kernels; k++) {
            kwork.push_back(a4(S.kernels[k].work_items));
            kflags.push_back(S.kernels[k].flags);
        }
        // work slots: kernels with the same work function share one count
        // per design point in the sweep kernel
        std::vector<uint32_t> kslot(S.n_kernels);
        I.w_base = (uint32_t)wslot_work.size();
        I.n_wslots = 0;
        {
            uint64_t cm = 0;
            bool c0ok = true;
            for (uint32_t k = 0; k < S.n_kernels; k++) {
                const int4 w = a4(S.kernels[k].work_items);
                uint32_t j = 0;
                while (j < I.n_wslots) {
                    const int4 &v = wslot_work[I.w_base + j];
                    if (v.x == w.x && v.y == w.y && v.z == w.z && v.w == w.w) break;
                    j++;
                }
                if (j == I.n_wslots) {
                    wslot_work.push_back(w);
                    wslot_sat.push_back(0u);
                    I.n_wslots++;
                    const int64_t c[3] = {w.y, w.z, w.w};
                    for (int m = 0; m < 3; m++) cm = std::max<uint64_t>(cm, (uint64_t)(c[m] < 0 ? -c[m] : c[m]));
                    c0ok = c0ok && w.x > -(1 << 29) && w.x < (1 << 29);
                }
                kslot[k] = j;
            }
            I.wslot_c32 = c0ok ? (uint32_t)std::min<uint64_t>(cm, 0xffffffffull) : 0xffffffffu;
        }
        for (uint32_t a = 0; a < S.n_arrays; a++) {
            ArrayDev A;
            A.rows = a4(S.arrays[a].rows);
            A.cols = a4(S.arrays[a].cols);
            A.elem_bytes = S.arrays[a].elem_bytes;
            A.liveout = (S.arrays[a].flags & GROPHECY_ARRAY_LIVEOUT) ? 1u : 0u;
            A.r_base = (uint32_t)regions.size();
            A.lr = A.lc = 1;
            A.planes = a4(S.arrays[a].planes);
            A.rank3 = !affine_is(S.arrays[a].planes, 1);
            A.pad1 = 0;
            // regions of this array, stably sorted by kernel (order within a
            // kernel is irrelevant: usage does not depend on region order)
            std::vector<const grophecy_region_desc *> rs;
            for (uint32_t j = 0; j < S.n_regions; j++)
                if (S.regions[j].array == a) rs.push_back(&S.regions[j]);
            std::stable_sort(rs.begin(), rs.end(), [](const grophecy_region_desc *x,
                                                      const grophecy_region_desc *y) {
                return x->kernel < y->kernel;
            });
            A.r_count = (uint32_t)rs.size();
            for (size_t j = 0; j < rs.size(); j++) {
                RegionDev R;
                R.r0 = a4(rs[j]->r0); R.r1 = a4(rs[j]->r1);
                R.c0 = a4(rs[j]->c0); R.c1 = a4(rs[j]->c1);
                R.whole = (rs[j]->flags & GROPHECY_REGION_WHOLE) ? 1u : 0u;
                // an irregular write may write any element: whole read + write
                R.mode = (R.whole && (rs[j]->mode & GROPHECY_W)) ? (rs[j]->mode | GROPHECY_R)
                                                                  : rs[j]->mode;
                R.rs = (!R.whole && rs[j]->r_step > 1) ? rs[j]->r_step : 1u;
                R.cs = (!R.whole && rs[j]->c_step > 1) ? rs[j]->c_step : 1u;
                R.pad0 = R.pad1 = 0;
                R.p0 = a4(rs[j]->p0);
                R.p1 = a4(rs[j]->p1);
                if (!R.whole && !(affine_is(rs[j]->p0, 0) && affine_is(rs[j]->p1, 1))) A.rank3 = 1;
                A.lr = (uint32_t)lcm_step(A.lr, R.rs);
                A.lc = (uint32_t)lcm_step(A.lc, R.cs);
                R.kernel = rs[j]->kernel;
                uint32_t upto = 0;
                for (size_t q = 0; q < rs.size(); q++)
                    if (rs[q]->kernel <= rs[j]->kernel) upto |= 1u << q;
                R.upto = upto;
                regions.push_back(R);
            }
            arrays.push_back(A);
        }
        const size_t kx0 = kf.size();   // this skeleton's kx_base
        kwsat.resize(kwork.size(), 0u);
        std::vector<double> xcost(S.n_xforms, 0.0);
        xinf.resize(kx0 + (size_t)S.n_kernels * S.n_xforms, 0u);
        xhdr.resize(kx0 + (size_t)S.n_kernels * S.n_xforms, make_uint4(0u, 0u, 0u, 0u));
        xord.resize(kx0 + (size_t)S.n_kernels * S.n_xforms, 0u);
        xhdru.resize(kx0 + (size_t)S.n_kernels * S.n_xforms, make_uint4(0u, 0u, 0u, 0u));
        std::vector<KxProg> pair_prog((size_t)S.n_kernels * S.n_xforms);
        for (uint32_t k = 0; k < S.n_kernels; k++)
            for (uint32_t x = 0; x < S.n_xforms; x++) {
                KxES es; KxD d; KxI i; KxJ j; KxG g;
                precompute(S.kx[(size_t)x * S.n_kernels + k], *gpu, es, d, i, j, g);
                if (S.kernels[k].flags & GROPHECY_KERNEL_PER_ITER) j.flags |= KXF_PER_ITER;
                kes.push_back(es); kd.push_back(d); ki.push_back(i); kj.push_back(j);
                kg.push_back(g);
                KxFast f;
                // blocks = hi32(w m + cc) >> sh = ceil(w / ipb) for w < 2^30
                // (internal.h); pairs off the fast path: blocks = 0 < sat
                const uint32_t dv = j.ipb;
                uint32_t sh = 0;
                if (dv == 1) {
                    f.m = 0xffffffffu;
                    f.cc = 0xffffffffull;
                } else if (dv <= (1u << 30)) {
                    uint32_t l = 0;
                    while ((1ull << l) < dv) l++;
                    const uint64_t m = ((1ull << (31 + l)) + dv - 1) / dv;
                    f.m = (uint32_t)m;
                    f.cc = (uint64_t)(dv - 1) * m;
                    sh = l - 1;
                } else {
                    f.m = 0;
                    f.cc = 0;
                }
                uint32_t sat;
                if (j.flags & KXF_INFEASIBLE) {
                    // occupancy 0: t_k = +inf for every size (N5).  The fast
                    // path yields a finite 0 here (sat = 0, never the general
                    // branch) and the record's sum is set to +inf from xinf
                    // (+inf + finite = +inf in any order: exact)
                    f.E = 0.0; f.S = 0.0; f.rDh = 1.0; f.rDl = 0.0; sat = 0;
                    xinf[kx0 + x] |= (S.kernels[k].flags & GROPHECY_KERNEL_PER_ITER) ? XINF_ITER : XINF_ONCE;
                } else if (dv > (1u << 30) || i.sat_blocks >= KXF_SAT_MASK || !freq_ok ||
                           !div2_ok(d.D) || !fast_const_ok(es.E) || !fast_const_ok(es.S)) {
                    f.E = 0.0; f.S = 0.0; f.rDh = 1.0; f.rDl = 0.0; sat = KXF_SAT_MASK;
                    f.m = 0;
                    f.cc = 0;
                } else {
                    f.E = es.E; f.S = es.S;
                    split_recip(d.D, f.rDh, f.rDl);
                    sat = (uint32_t)i.sat_blocks;
                }
                f.satsh = sat | sh << KXF_SAT_BITS;
                kf.push_back(f);
                // the sweep kernel's program entry (internal.h KxProg)
                KxProg c;
                std::memset(&c, 0, sizeof c);
                uint32_t pcls = KXC_NONE;
                {
                    // power-of-two ipb: no post-shift (m = 2^(32 - l))
                    uint32_t psh = sh, pm = f.m;
                    uint64_t pcc = f.cc;
                    if (dv >= 2 && dv <= (1u << 30) && (dv & (dv - 1)) == 0) {
                        uint32_t l = 0;
                        while ((1u << l) < dv) l++;
                        pm = 1u << (32 - l);
                        pcc = (uint64_t)(dv - 1) * pm;
                        psh = 0;
                    }
                    c.m = pm;
                    c.cc = pcc;
                    c.sat = (sat & 0xffffu) | k << 16;   // (the sweep reads it for tabulated pairs only)
                    c.sh = psh;
                    c.cwoff = kslot[k] * 256u;   // = slot * SW_GROUPS (project.cu)
                    c.kbit = 1u << kslot[k];
                }
                if (!(j.flags & KXF_INFEASIBLE) && sat != KXF_SAT_MASK && sat <= KXP_SAT_MAX) {
                    const bool p2 = f.rDl == 0.0, s0 = f.S == 0.0;
                    // blocks < sat <=> w <= (sat - 1) * ipb
                    const uint64_t ws = (uint64_t)(sat - 1) * dv + 1;
                    uint32_t &kw = kwsat[I.k_base + k];
                    kw = (uint32_t)std::max<uint64_t>(kw, std::min<uint64_t>(ws, 1ull << 30));
                    xcost[x] += 5.0 + (p2 ? (s0 ? 4.0 : 6.0) : (s0 ? 6.0 : 8.0));
                    if (p2) {
                        c.c[0] = f.E * f.rDh;   // exact: rDh = 2^-k, E normal (fast_const_ok)
                        c.c[1] = f.S * f.rDh;
                        pcls = s0 ? KXC_P2S0 : KXC_P2S;
                    } else {
                        c.c[0] = f.rDh;
                        c.c[1] = f.rDl;
                        c.c[2] = f.E;
                        c.c[3] = f.S;
                        pcls = s0 ? KXC_NS0 : KXC_NS;
                    }
                }
                // KXC_SHIFT: the class's program post-shifts the block counts
                c.cls = pcls | (pcls != KXC_NONE && c.sh ? KXC_SHIFT : 0u);
                pair_prog[(size_t)x * S.n_kernels + k] = c;
            }
        for (uint32_t k = 0; k < S.n_kernels; k++)
            wslot_sat[I.w_base + kslot[k]] = std::max(wslot_sat[I.w_base + kslot[k]], kwsat[I.k_base + k]);
        // per transformation: its program header (at kx_base + x) and program
        // (feasible saturated-capable kernels, per-iteration ones then run-once
        // ones, each in ascending kernel order: N6); the header carries an
        // estimated cost for the phase-C claim order (longest first)
        for (uint32_t x = 0; x < S.n_xforms; x++) {
            if (xinf[kx0 + x]) xcost[x] = 0.0;   // the sweep skips the unit (no finite total)
            const uint32_t first = (uint32_t)kprog.size();
            uint32_t n_it = 0, n_on = 0;
            for (int pass = 0; pass < 2; pass++)
                for (uint32_t k = 0; k < S.n_kernels; k++) {
                    const bool per = (S.kernels[k].flags & GROPHECY_KERNEL_PER_ITER) != 0;
                    const KxProg &e = pair_prog[(size_t)x * S.n_kernels + k];
                    if (per != (pass == 0) || e.cls == KXC_NONE) continue;
                    kprog.push_back(e);
                    (pass == 0 ? n_it : n_on)++;
                }
            const uint32_t cost = (uint32_t)std::min(xcost[x], 16777215.0);
            xhdr[kx0 + x] = make_uint4(x, first, n_it | n_on << 16, xinf[kx0 + x] | cost << 8);
        }
        // phase-C claim order of the transformations (longest first: the CTA's
        // warps finish together)
        {
            std::vector<uint32_t> ord(S.n_xforms);
            for (uint32_t x = 0; x < S.n_xforms; x++) ord[x] = x;
            std::stable_sort(ord.begin(), ord.end(),
                             [&](uint32_t a, uint32_t b) { return xcost[a] > xcost[b]; });
            for (uint32_t u = 0; u < S.n_xforms; u++) {
                xord[kx0 + u] = ord[u];
                xhdru[kx0 + u] = xhdr[kx0 + ord[u]];
            }
        }
    }

    // ---- small-grid table: t(kernel, xform, blocks) for blocks < sat32 ----
    uint32_t max_sat = 0;
    for (const KxFast &f : kf)
        if (kxf_sat(f) != KXF_SAT_MASK) max_sat = std::max(max_sat, kxf_sat(f));
    const uint32_t small_stride = std::min<uint32_t>(max_sat, SMALL_GRID_MAX);
    std::vector<double> small((size_t)kf.size() * small_stride, 0.0);
    for (size_t q = 0; q < kf.size(); q++)
        if (kxf_sat(kf[q]) <= small_stride)
            for (uint32_t b = 0; b < kxf_sat(kf[q]); b++)
                small[q * small_stride + b] = small_grid_time(kj[q], kg[q], gpu->n_sm, gpu->freq_hz, b);

    // the canonical kernel indexes the table with 32-bit element offsets
    const bool small_idx32 = (uint64_t)kf.size() * small_stride < (1ull << 32);
    for (uint32_t s = 0; s < n_skels; s++) {
        bool tab = small_idx32;
        const uint32_t nkx = skels[s].n_kernels * skels[s].n_xforms;
        for (uint32_t q = info[s].kx_base; q < info[s].kx_base + nkx; q++)
            tab = tab && kxf_sat(kf[q]) <= small_stride;
        if (tab) info[s].flags |= SKF_TABULATED;
    }

    // ---- one device blob ----
    struct Part { const void *src; size_t bytes; size_t off; };
    std::vector<Part> parts = {
        {info.data(), info.size() * sizeof(SkelInfo), 0},
        {kwork.data(), kwork.size() * sizeof(int4), 0},
        {kflags.data(), kflags.size() * sizeof(uint32_t), 0},
        {arrays.data(), arrays.size() * sizeof(ArrayDev), 0},
        {regions.data(), regions.size() * sizeof(RegionDev), 0},
        {kes.data(), kes.size() * sizeof(KxES), 0},
        {kd.data(), kd.size() * sizeof(KxD), 0},
        {ki.data(), ki.size() * sizeof(KxI), 0},
        {kj.data(), kj.size() * sizeof(KxJ), 0},
        {kg.data(), kg.size() * sizeof(KxG), 0},
        {poly.data(), poly.size() * sizeof(unsigned long long), 0},
        {kf.data(), kf.size() * sizeof(KxFast), 0},
        {small.data(), small.size() * sizeof(double), 0},
        {xinf.data(), xinf.size() * sizeof(uint32_t), 0},
        {kprog.data(), kprog.size() * sizeof(KxProg), 0},
        {xhdr.data(), xhdr.size() * sizeof(uint4), 0},
        {kwsat.data(), kwsat.size() * sizeof(uint32_t), 0},
        {xord.data(), xord.size() * sizeof(uint32_t), 0},
        {xhdru.data(), xhdru.size() * sizeof(uint4), 0},
        {wslot_work.data(), wslot_work.size() * sizeof(int4), 0},
        {wslot_sat.data(), wslot_sat.size() * sizeof(uint32_t), 0},
    };
    size_t total = 0;
    for (auto &p : parts) {
        p.off = total;
        total = align_up(total + p.bytes, 256);
    }
    std::vector<unsigned char> host(total, 0);
    for (auto &p : parts)
        if (p.bytes) std::memcpy(host.data() + p.off, p.src, p.bytes);

    int prev = 0;
    cudaError_t e = cudaGetDevice(&prev);
    if (e != cudaSuccess) return cuda_fail(e, "cudaGetDevice");
    if ((e = cudaSetDevice(device)) != cudaSuccess) return cuda_fail(e, "cudaSetDevice");

    grophecy_space *sp = new grophecy_space();
    std::memset(sp, 0, sizeof *sp);
    sp->device = device;
    auto bail = [&](cudaError_t err, const char *what) {
        if (sp->blob) cudaFree(sp->blob);
        delete sp;
        cudaSetDevice(prev);
        return cuda_fail(err, what);
    };
    int nsm = 0;
    if ((e = cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, device)) != cudaSuccess)
        return bail(e, "cudaDeviceGetAttribute");
    sp->max_partials = (uint32_t)nsm * 32u;
    size_t scratch_off = align_up(total, 256);
    size_t part_bytes = sizeof(grophecy_best_result) * sp->max_partials;
    const size_t list_bytes = (size_t)GROPHECY_TILE_CAP * sizeof(uint32_t);
    size_t blob = scratch_off + align_up(part_bytes, 256) + 256 + align_up(sizeof(SpaceDev), 256) +
                  list_bytes;
    if ((e = cudaMalloc(&sp->blob, blob)) != cudaSuccess) return bail(e, "cudaMalloc(space)");
    sp->blob_bytes = blob;
    if ((e = cudaMemcpy(sp->blob, host.data(), total, cudaMemcpyHostToDevice)) != cudaSuccess)
        return bail(e, "cudaMemcpy(space)");
    unsigned char *base = (unsigned char *)sp->blob;
    sp->partials = (grophecy_best_result *)(base + scratch_off);
    unsigned char *ctr = base + scratch_off + align_up(part_bytes, 256);
    sp->ticket = (unsigned int *)ctr;
    sp->invalid_counter = (unsigned long long *)(ctr + 64);
    sp->tile_count = (unsigned int *)(ctr + 128);   // + the tile-claim counters (project.cu CLAIM1/2)
    sp->tile_list = (uint32_t *)(ctr + 256 + align_up(sizeof(SpaceDev), 256));
    if ((e = cudaMemset(ctr, 0, 256)) != cudaSuccess) return bail(e, "cudaMemset(space)");

    SpaceDev &D = sp->dev;
    D.skel = (const SkelInfo *)(base + parts[0].off);
    D.kern_work = (const int4 *)(base + parts[1].off);
    D.kern_flags = (const uint32_t *)(base + parts[2].off);
    D.arrays = (const ArrayDev *)(base + parts[3].off);
    D.regions = (const RegionDev *)(base + parts[4].off);
    D.kx_es = (const KxES *)(base + parts[5].off);
    D.kx_d = (const KxD *)(base + parts[6].off);
    D.kx_i = (const KxI *)(base + parts[7].off);
    D.kx_j = (const KxJ *)(base + parts[8].off);
    D.kx_g = (const KxG *)(base + parts[9].off);
    D.poly = (const unsigned long long *)(base + parts[10].off);
    D.kx_f = (const KxFast *)(base + parts[11].off);
    D.small_t = (const double *)(base + parts[12].off);
    D.xinf = (const uint32_t *)(base + parts[13].off);
    D.xprog = (const KxProg *)(base + parts[14].off);
    D.xhdr = (const uint4 *)(base + parts[15].off);
    D.wslot_work = (const int4 *)(base + parts[19].off);
    D.wslot_sat = (const uint32_t *)(base + parts[20].off);
    D.xord = (const uint32_t *)(base + parts[17].off);
    D.xhdru = (const uint4 *)(base + parts[18].off);
    D.small_stride = small_stride;
    D.n_skels = n_skels;
    D.n_sm = gpu->n_sm;
    D.freq = gpu->freq_hz;
    D.rfreq = 1.0 / gpu->freq_hz;
    split_recip(gpu->freq_hz, D.rfh, D.rfl);
    D.invalid_counter = sp->invalid_counter;
    sp->dev_copy = (SpaceDev *)(ctr + 256);
    if ((e = cudaMemcpy(sp->dev_copy, &D, sizeof D, cudaMemcpyHostToDevice)) != cudaSuccess)
        return bail(e, "cudaMemcpy(space header)");
    sp->grid_best = nsm;
    sp->usage_tbl_bytes = 0;
    for (uint32_t q = 0; q < n_skels; q++)
        if (info[q].polyf_base != POLY32_NONE)
            sp->usage_tbl_bytes = std::max<uint32_t>(
                sp->usage_tbl_bytes,
                ((info[q].polyf_nhd & 0xffffu) + (info[q].polyf_nhd >> 16)) * POLY_CLASSES * 16u);
    // the sweep's design points: records of one (skeleton, nx, ny, iters) for
    // every transformation, so their size is the skeletons' common n_xforms
    // test hooks (read once per space, not per launch)
    sp->sweep_two_env = -1;
    if (const char *e = getenv("GROPHECY_SWEEP_TWO")) sp->sweep_two_env = atoi(e) != 0;
    sp->sweep_grid_env = 0;
    if (const char *e = getenv("GROPHECY_SWEEP_GRID")) sp->sweep_grid_env = (uint32_t)std::max(0, atoi(e));
    sp->sweep_cx = 16;
    {
        bool same = true;
        for (uint32_t q = 1; q < n_skels; q++) same = same && skels[q].n_xforms == skels[0].n_xforms;
        const uint32_t x = skels[0].n_xforms;
        if (same && (x == 4 || x == 8)) sp->sweep_cx = x;
    }
    sp->max_kernels = 1;
    sp->max_wslots = 1;
    for (uint32_t q = 0; q < n_skels; q++) {
        sp->max_kernels = std::max(sp->max_kernels, skels[q].n_kernels);
        sp->max_wslots = std::max(sp->max_wslots, info[q].n_wslots);
    }
    sp->occ_canon = 0;
    sp->grid_eval = nsm;
    cudaSetDevice(prev);
    *out = sp;
    return GROPHECY_OK;
}

void grophecy_space_destroy(grophecy_space *sp)
{
    if (!sp) return;
    int prev = 0;
    cudaGetDevice(&prev);
    cudaSetDevice(sp->device);
    if (sp->copy_stream) {
        cudaStreamSynchronize(sp->copy_stream);
        cudaStreamDestroy(sp->copy_stream);
        for (int i = 0; i < 2; i++) {
            cudaEventDestroy(sp->ev_copied[i]);
            cudaEventDestroy(sp->ev_done[i]);
        }
    }
    for (int i = 0; i < 2; i++)
        if (sp->stage[i]) cudaFree(sp->stage[i]);
    if (sp->gscratch) cudaFree(sp->gscratch);
    if (sp->mscratch) cudaFree(sp->mscratch);
    if (sp->blob) cudaFree(sp->blob);
    cudaSetDevice(prev);
    delete sp;
}

int grophecy_invalid_count(grophecy_space *sp, uint64_t *count, void *stream)
{
    if (!sp || !count) return fail(GROPHECY_EINVAL, "null argument");
    cudaStream_t st = (cudaStream_t)stream;
    unsigned long long v = 0;
    cudaError_t e = cudaMemcpyAsync(&v, sp->invalid_counter, sizeof v, cudaMemcpyDeviceToHost, st);
    if (e == cudaSuccess) e = cudaMemsetAsync(sp->invalid_counter, 0, sizeof v, st);
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    if (e != cudaSuccess) return cuda_fail(e, "grophecy_invalid_count");
    *count = v;
    return GROPHECY_OK;
}

// (t, index) lexicographic min-loc with counter sums; "none" = index UINT64_MAX.
int grophecy_best_combine_host(const grophecy_best_result *in, uint32_t count,
                               grophecy_best_result *out)
{
    if (!out || (count && !in)) return fail(GROPHECY_EINVAL, "null argument");
    grophecy_best_result b;
    b.t_total_s = INFINITY;
    b.index = ~0ull;
    b.h2d_bytes = b.d2h_bytes = 0;
    b.n_invalid = b.n_valid = 0;
    for (uint32_t i = 0; i < count; i++) {
        const grophecy_best_result &r = in[i];
        b.n_invalid += r.n_invalid;
        b.n_valid += r.n_valid;
        if (r.index == ~0ull) continue;
        if (b.index == ~0ull || r.t_total_s < b.t_total_s ||
            (r.t_total_s == b.t_total_s && r.index < b.index)) {
            b.t_total_s = r.t_total_s;
            b.index = r.index;
            b.h2d_bytes = r.h2d_bytes;
            b.d2h_bytes = r.d2h_bytes;
        }
    }
    *out = b;
    return GROPHECY_OK;
}

// One group split across two consecutive batches (NEXT-1 cross-shard fix-up).
int grophecy_group_merge_host(const grophecy_group_result *a, const grophecy_group_result *b,
                              grophecy_group_result *out)
{
    if (!a || !b || !out) return fail(GROPHECY_EINVAL, "null argument");
    if (a->first + a->count != b->first)
        return fail(GROPHECY_EINVAL, "group_merge: b does not follow a");
    grophecy_group_result m = *a;
    m.count = a->count + b->count;
    // "none" has index UINT64_MAX and t = +inf, so it never wins
    if (b->best_index != ~0ull &&
        (a->best_index == ~0ull || b->best_t_s < a->best_t_s ||
         (b->best_t_s == a->best_t_s && b->best_index < a->best_index))) {
        m.best_t_s = b->best_t_s;
        m.best_index = b->best_index;
        m.h2d_bytes = b->h2d_bytes;
        m.d2h_bytes = b->d2h_bytes;
    }
    *out = m;
    return GROPHECY_OK;
}

}  // extern "C"
