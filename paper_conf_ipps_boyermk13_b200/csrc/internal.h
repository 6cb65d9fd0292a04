// Internal layout of a grophecy_space (host + device).  Product code only.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <string>
#include <vector>

#include "grophecy.h"

namespace grophecy {

// Per (skeleton, kernel, transformation) constants, precomputed on the host in
// the exact operation order of DESIGN.md §3 N5.  Stored struct-of-arrays by
// field pair (index kxi = skel.kx_base + k * n_xforms + x) so the 16 lanes of
// a candidate group read 16 consecutive 16-byte entries.
//
// "Saturated" grid: blocks >= sat_blocks  <=>  #Active_SMs == n_sm and
// active blocks/SM == occ; then N, MWP, CWP and the H&K case are constants
// and cyc = E*rep + S*rep with rep = blocks / D (D = occ * n_sm).
struct __align__(16) KxES { double E, S; };         // case expression, synch factor
struct __align__(16) KxD  { double D, rD; };        // rep denominator and RN(1/D)
struct __align__(16) KxI  { uint64_t magic; uint64_t sat_blocks; };  // ceil(2^64/ipb) (0 if ipb==1)
struct __align__(16) KxJ  { uint32_t ipb, occ, wpb, flags; };        // flags: KXF_*
enum : uint32_t { KXF_INFEASIBLE = 1u, KXF_NOMEM = 2u, KXF_PER_ITER = 4u };
enum : uint32_t { XINF_ITER = 1u, XINF_ONCE = 2u };

// Packed fast-path record (48 B, one address per (kernel, transformation)).
// Work counts are stored as w in [0, 2^30) (else W_HUGE: the general path).
// blocks = ceil(w / ipb) = hi32(w * m + cc) >> sh: for ipb = d >= 2,
// l = ceil(log2 d), m = ceil(2^(31 + l) / d) < 2^32, cc = (d - 1) m, sh = l - 1
// (Granlund-Montgomery: floor(n m / 2^(31 + l)) = floor(n / d) for every
// n = w + d - 1 < 2^31); d = 1: m = cc = 2^32 - 1, sh = 0.  satsh = sat |
// sh << KXF_SAT_BITS; the saturated formula holds iff blocks >= sat.
// Pairs the fast path cannot take (ipb > 2^30, sat >= KXF_SAT_MASK): m = cc =
// 0 (blocks = 0) and sat = KXF_SAT_MASK, i.e. always the general path.
// Infeasible (occupancy 0): E = S = 0, sat = 0 (a finite 0 from the fast
// path, replaced by +inf through SpaceDev::xinf).
constexpr uint32_t KXF_SAT_BITS = 27, KXF_SAT_MASK = (1u << KXF_SAT_BITS) - 1u;
// rep = RN(blocks / D) = RN(blocks * rDh + RN(blocks * rDl)) with rDh = RN(1/D),
// rDl = RN(1/D - rDh) (one DMUL + one DFMA, exact for integer blocks and
// integer D < 2^50: DESIGN.md §5 "two-product division"); t = cyc / freq the
// same way with SpaceDev::rfh / rfl.
struct __align__(16) KxFast {
    uint32_t m, satsh;        // first: the chain starts with blocks
    uint64_t cc;
    double rDl, rDh, E, S;
};
inline uint32_t kxf_sat(const KxFast &f) { return f.satsh & KXF_SAT_MASK; }

// Class-specialised saturated constants (sweep kernel).  With
// b = blocks (an integer), rep = RN(b / D) and cyc = RN(RN(E rep) + RN(S rep)):
//   P2S0  D a power of two, S = 0:  cyc = RN(b E')            c = {E' = E / D}
//   P2S   D a power of two:         cyc = RN(RN(b E') + RN(b S'))   c = {E', S'}
//   NS0   S = 0:                    cyc = RN(E rep)          c = {rDh, rDl, E}
//   NS    otherwise:                the full form            c = {rDh, rDl, E, S}
// (b / D = b 2^-k is exact when D = 2^k, and E 2^-k, S 2^-k are exact scalings,
// so RN(E rep) = RN(b E'); S = 0 makes RN(S rep) = +0.0, which adds nothing.)
// m / satsh / cc as in KxFast.
// A transformation's program (sweep kernel): its feasible kernels' entries in
// summation order (per-iteration kernels, then run-once ones, each ascending;
// infeasible kernels are left out: their sum is +inf through xinf).
enum : uint32_t { KXC_P2S0 = 0u, KXC_P2S = 1u, KXC_NS0 = 2u, KXC_NS = 3u, KXC_SHIFT = 4u, KXC_NONE = 8u };
// blocks = hi32(w m + cc) >> sh (as KxFast; a power-of-two ipb = 2^l uses
// m = 2^(32 - l), cc = (ipb - 1) m, sh = 0); the kernel's work slot j
// (SkelInfo::n_wslots) as its work-count offset cwoff = j * 256 (sweep shared
// memory) and its bit kbit = 1 << j; sat = sat_blocks | k << 16 (kernel k:
// the small-grid table's row), sat_blocks <= SMALL_GRID_MAX (the sweep path
// requires tabulated pairs).  Fields unpacked: 64 bytes, four 16-byte loads.
struct __align__(16) KxProg {
    uint32_t m, sat;
    uint64_t cc;
    uint32_t cwoff, sh, kbit, cls;
    double c[4];
};
constexpr uint32_t KXP_SAT_MAX = 0x7ffu;

// General-grid constants (small grids / huge W), read only off the fast path.
struct KxG {
    double comp, mwp0, bwr, memc, cwpf, cpm, ml, dd, synch, pad;
};

struct SkelInfo {
    uint32_t n_kernels, n_arrays, n_xforms, n_regions;
    uint32_t k_base;   // into kern_work / kern_flags
    uint32_t a_base;   // into arrays
    uint32_t kx_base;  // into kx tables
    uint32_t flags;    // GROPHECY_SKEL_* (HULL) | SKF_*
    // usage plan (plan.cpp): valid for nx >= plan_tx and ny >= plan_ty; its
    // byte polynomials at poly[poly_base + ...] (SkelPlanHost layout)
    uint32_t plan_tx, plan_ty, poly_base, poly_stride;
    uint32_t per_iter_mask;   // bit k = kernel k per-iteration
    uint32_t poly_mask;       // bit 2a + dir: byte polynomial not zero in every size class
    // compact copy of a bilinear table whose coefficients all fit int32:
    // poly[poly32_base + 2 * (c * n_polys + p)] holds int4 {c0, c1, c2, c3}
    // (sign-extended they are the u64 coefficients); POLY32_NONE if absent
    uint32_t poly32_base;
    // the sweep kernel's table: poly[polyf_base + 2 * (q * 64 + c)] holds
    // int4 {c0, c1, c2, c3} of list entry q in size class c; the entries are
    // the H2D polynomials not zero in every class (array order), padded with
    // zero ones to a multiple of POLYF_AU, then the D2H ones likewise;
    // polyf_nhd = (padded H2D count) | (padded D2H count) << 16.
    // POLY32_NONE if absent (staged whole into shared memory)
    uint32_t polyf_base;
    uint32_t polyf_nhd;
    // bound of |coefficient m| over the sweep table's polynomials (saturated
    // at 2^32 - 1): when cmax0 + cmax1 a + cmax2 b + cmax3 a b < 2^32 every
    // partial sum of a polynomial is below 2^32, so its 32-bit wrapping
    // evaluation is the exact byte count
    uint32_t polyf_cmax[4];
    // sweep kernel: the distinct work-count functions of the kernels ("work
    // slots", first-use order) at wslot_work[w_base + j], j < n_wslots; a
    // program entry reads its kernel's slot.  wslot_c32: max |c1|, |c2|, |c3|
    // over the slots (0xffffffff when some |c0| >= 2^29): when
    // wslot_c32 * (nx + ny + nx ny) < 2^31 every slot's count is exact in
    // 32-bit arithmetic
    uint32_t w_base, n_wslots, wslot_c32, pad_w;
};
constexpr uint32_t POLYF_AU = 4;   // arrays per step of the fp64 usage evaluation

struct ArrayDev {
    int4 rows, cols;
    uint32_t elem_bytes, liveout, r_base, r_count;   // regions [r_base, r_base+r_count)
    uint32_t lr, lc;    // lcm of the regions' row / column steps (1 = dense array)
    uint32_t rank3;     // planes != 1 or a region's plane range != [0, 1) (N4r)
    uint32_t pad1;
    int4 planes;
};
enum : uint32_t {
    SKF_STRIDED = 1u << 16,     // some region has a step > 1
    SKF_TABULATED = 1u << 17,   // every (kernel, xform) off the saturated path is in the
                                // small-grid table or infeasible (canonical kernel eligible)
    SKF_RANK3 = 1u << 18,       // some array is rank-3 (no usage plan: general sweep)
};

constexpr uint32_t PLAN_MAX_EXPR = 128;   // < 256: programs pack u8 indices

// Host-side result of compiling one skeleton's usage plan.
struct SkelPlanHost {
    bool ok = false;
    uint32_t tx = 0, ty = 0;
    std::vector<int4> exprs;
    std::vector<uint32_t> prog;           // band programs (see plan.cpp)
    std::vector<uint32_t> h_off, d_off;   // per array, into prog
    // Byte polynomials (plan.cpp, "residue-class polynomials"): for size class
    // c = (nx mod 8) * 8 + (ny mod 8) and polynomial p = 2 * array + dir,
    // poly[(c * n_polys + p) * poly_stride + m] = coefficient of monomial m in
    // (a, b) = (nx div 8, ny div 8), monomials {1, a, b, ab, a^2, b^2, a^2 b,
    // a b^2, a^2 b^2}; stride 4 when every skeleton term is bilinear, else 10
    // (9 + pad).  Coefficients are mod 2^64 (wrapping); elem_bytes and the
    // live-out flag are folded in, so P(a, b) = transfer bytes of the array.
    std::vector<uint64_t> poly;
    uint32_t poly_stride = 0;
};
constexpr uint32_t POLY_CLASSES = 64;
constexpr uint32_t POLY_ZERO_WORDS = 10;   // SpaceDev::poly[0..9] = 0 (one zero polynomial)
constexpr uint32_t POLY32_NONE = 0xffffffffu;
constexpr uint32_t SMALL_GRID_MAX = 1024;   // tabulated small grids per (kernel, xform)
#define GROPHECY_TILE_CAP (1u << 21)        // tiles of 512 records per projection pass

// P(a, b) of one byte polynomial (host and device share the formula; device
// copy in project.cu).  a, b < 2^18.
inline uint64_t poly_eval_host(const uint64_t *c, uint32_t stride, uint64_t a, uint64_t b)
{
    uint64_t v = c[0] + c[1] * a + (c[2] + c[3] * a) * b;
    if (stride > 4) v += a * (a * (c[4] + b * (c[6] + b * c[8]))) + b * (b * (c[5] + a * c[7]));
    return v;
}

// Regions are stored grouped by array and sorted by kernel within an array,
// so "first writer" = lowest set bit of a mask and upto = mask of regions of
// the same array whose kernel <= this region's kernel.
// mode is the effective mode: an irregular (WHOLE) write is a may-write and
// carries R as well (reading 10).  rs / cs: steps (1 = dense).
struct RegionDev {
    int4 r0, r1, c0, c1;
    uint32_t mode, whole, upto, kernel;
    uint32_t rs, cs, pad0, pad1;
    int4 p0, p1;        // plane range (rank-3 arrays)
};

struct SpaceDev {
    const SkelInfo *skel;
    const int4 *kern_work;
    const uint32_t *kern_flags;
    const ArrayDev *arrays;
    const RegionDev *regions;
    const KxES *kx_es;
    const KxD *kx_d;
    const KxI *kx_i;
    const KxJ *kx_j;
    const KxG *kx_g;
    const KxFast *kx_f;
    // sweep kernel: per (skeleton, xform x) at kx_base + x the program
    // header {x, first entry, n_iter | n_once << 16, xinf bits | cost << 8}
    // (cost: estimated work, for the phase-C claim order); the programs
    const uint4 *xhdr;
    const KxProg *xprog;
    const uint32_t *xord;       // per (skeleton, unit u) at kx_base + u: xforms by descending cost
    const uint4 *xhdru;         // xhdr in that order (one load per unit in the identity layout)
    const unsigned long long *poly;   // usage byte polynomials (all skeletons)
    // small-grid kernel times: small_t[kxi * small_stride + blocks] for
    // blocks < sat32 when sat32 <= small_stride (space.cpp small_grid_time)
    const double *small_t;
    // per (skeleton, xform), at kx_base + x: some per-iteration (XINF_ITER) /
    // run-once (XINF_ONCE) kernel is infeasible, so that sum is +inf
    const uint32_t *xinf;
    // sweep kernel: per (skeleton, work slot) at w_base + j, the slot's work
    // function and the smallest work count w for which the grid of every
    // (kernel of the slot, transformation) is saturated (blocks >= sat)
    const int4 *wslot_work;
    const uint32_t *wslot_sat;
    uint32_t small_stride;
    uint32_t n_skels;
    uint32_t n_sm;
    double freq, rfreq;
    // 1/freq as an unevaluated sum rfh + rfl (fast path: t = RN(cyc * rfh +
    // RN(cyc * rfl)) = RN(cyc / freq) when freq's odd significand < 2^50)
    double rfh, rfl;
    unsigned long long *invalid_counter;
};

}  // namespace grophecy

struct grophecy_space {
    int device;
    grophecy::SpaceDev dev;
    grophecy::SpaceDev *dev_copy;        // the same struct in device memory (rare paths)
    void *blob;                          // one device allocation for all tables
    size_t blob_bytes;
    grophecy_best_result *partials;      // best-mode per-block partials
    uint32_t *tile_list;                 // pass 1 -> pass 2 tile list (GROPHECY_TILE_CAP)
    unsigned int *tile_count;
    unsigned int *ticket;                // best-mode last-block counter
    unsigned long long *invalid_counter;
    uint32_t max_partials;
    int grid_best, grid_eval;            // persistent grid sizes
    uint32_t max_kernels;                // largest kernel count of the space's skeletons
    uint32_t max_wslots;                 // largest work-slot count (SkelInfo::n_wslots)
    int sweep_two_env;                   // test hooks read at creation: GROPHECY_SWEEP_TWO (-1: unset)
    uint32_t sweep_grid_env;             // ... and GROPHECY_SWEEP_GRID (0: unset)
    uint32_t sweep_cx;                   // sweep kernel's design-point size (4, 8 or 16: the
                                         // skeletons' common n_xforms, else 16)
    int occ_canon;                       // pass-1 CTAs per SM (0 = not yet queried)
    int occ_sweep;                       // sweep-kernel CTAs per SM (0 = not yet queried)
    uint32_t usage_tbl_bytes;            // largest padded usage table (sweep shared memory)
    bool counters_clean;                 // tile counters known zero (after a best projection)
    // group_best scratch (grown on demand)
    void *gscratch;
    size_t gscratch_bytes;
    // best_allreduce: gathered results + the combined one (grown on demand)
    void *mscratch;
    size_t mscratch_bytes;
    // e2e host path staging
    void *stage[2];
    size_t stage_bytes;
    cudaStream_t copy_stream;
    cudaEvent_t ev_copied[2], ev_done[2];
};

namespace grophecy {
// The affine value is the constant v (c1 = c2 = c3 = 0).
inline bool affine_is(const grophecy_affine8 &a, int32_t v)
{
    return a.c0 == v && a.c1 == 0 && a.c2 == 0 && a.c3 == 0;
}
// Some array of the skeleton is rank-3 (N4r): planes != 1, or a
// (non-whole) region's plane range is not [0, 1).
inline bool skeleton_rank3(const grophecy_skeleton_desc &S)
{
    for (uint32_t a = 0; a < S.n_arrays; a++)
        if (!affine_is(S.arrays[a].planes, 1)) return true;
    for (uint32_t j = 0; j < S.n_regions; j++)
        if (!(S.regions[j].flags & GROPHECY_REGION_WHOLE) &&
            !(affine_is(S.regions[j].p0, 0) && affine_is(S.regions[j].p1, 1)))
            return true;
    return false;
}
// Makes the space's device current for one ABI call (and restores the
// caller's): launches, streams and the per-device kernel attributes match.
struct DeviceGuard {
    int prev = -1;
    explicit DeviceGuard(int device)
    {
        if (cudaGetDevice(&prev) == cudaSuccess && prev != device) cudaSetDevice(device);
        else prev = -1;
    }
    ~DeviceGuard()
    {
        if (prev >= 0) cudaSetDevice(prev);
    }
};
bool compile_plan(const grophecy_skeleton_desc &S, SkelPlanHost &out);
void set_error(const std::string &msg);
int cuda_fail(cudaError_t e, const char *what);
void count_launch(uint64_t n = 1);
// local_off: for a striped batch, the batch-local index of its record 0
// (chunked host batches)
int launch_best(grophecy_space *s, const grophecy_pcie *pcie, const grophecy_batch *b,
                grophecy_best_result *dout, int accumulate, cudaStream_t st, uint64_t local_off = 0);
}  // namespace grophecy
