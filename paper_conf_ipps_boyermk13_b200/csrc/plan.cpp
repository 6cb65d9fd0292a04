// Usage plans: the data-usage analysis of one skeleton "compiled" at space
// creation into closed-form band programs valid on a size domain.
//
// For one array the H2D / D2H element counts are areas of unions of cells of
// the grid cut by the region bounds (§III-B; DESIGN.md §3
// N4).  The bounds are size-affine expressions v = c0 + floor(L(nx, ny) / 8).
// On a domain D = [tx, 2^20] x [ty, 2^20] where every pairwise order between
// the bounds (and 0 and the array extent) is FIXED, the cell structure, the
// clamping and the first-reader / first-writer of every cell are the same for
// all sizes in D, so
//     count = sum_bands (row[e] - row[s]) * sum_runs (col[e'] - col[s'])
// with row/col values the (unclamped-by-construction) bound expressions.
// Equal values at some sizes only produce zero-height slabs, so a fixed
// non-strict order suffices.
//
// u <= v on D is proven exactly: floor(a) - floor(b) >= (a - b) - 7/8 for
// a, b in Z/8, so  8(v0 - u0) - 7 + (Lv - Lu)(nx, ny) >= 0  on D  implies
// v - u >= 0 on D; the left side is bilinear in (nx, ny), hence its minimum
// over the box D is at a corner.
//
// Keys outside the domain (or skeletons without a plan: strided sections,
// the approximate hull mode) take the general cooperative paths on the device.
#include <algorithm>
#include <cstdint>
#include <vector>

#include "grophecy.h"
#include "internal.h"

namespace grophecy {

namespace {

struct Ex {
    int64_t c0, c1, c2, c3;
    bool operator==(const Ex &o) const { return c0 == o.c0 && c1 == o.c1 && c2 == o.c2 && c3 == o.c3; }
};

Ex ex_of(const grophecy_affine8 &a) { return {a.c0, a.c1, a.c2, a.c3}; }
const Ex ZERO = {0, 0, 0, 0};

struct Dom {
    int64_t x0, x1, y0, y1;
};

bool nonneg_on(int64_t a, int64_t b, int64_t c, int64_t d, const Dom &D)
{
    const int64_t xs[2] = {D.x0, D.x1}, ys[2] = {D.y0, D.y1};
    for (int64_t x : xs)
        for (int64_t y : ys)
            if (a + b * x + c * y + d * x * y < 0) return false;
    return true;
}

// proven u <= v at every size of D
bool le(const Ex &u, const Ex &v, const Dom &D)
{
    if (u == v) return true;
    return nonneg_on(8 * (v.c0 - u.c0) - 7, v.c1 - u.c1, v.c2 - u.c2, v.c3 - u.c3, D);
}

enum Ord { LT, GT, EQ, UNK };

Ord order(const Ex &u, const Ex &v, const Dom &D)
{
    if (u == v) return EQ;
    const bool a = le(u, v, D), b = le(v, u, D);
    if (a && b) return EQ;   // cannot happen for distinct coefficients (slack), kept for safety
    if (a) return LT;
    if (b) return GT;
    return UNK;
}

// clamp(x, 0, E) resolved symbolically on D; false if the branch varies.
bool clamp_sym(const Ex &x, const Ex &E, const Dom &D, Ex &out)
{
    if (le(x, ZERO, D)) { out = ZERO; return true; }
    if (le(E, x, D)) { out = E; return true; }
    if (le(ZERO, x, D) && le(x, E, D)) { out = x; return true; }
    return false;
}

// Sort expression list into classes of a fixed order on D.  pos[i] = class of
// vals[i]; reps = one representative per class, ascending.
bool classify(const std::vector<Ex> &vals, const Dom &D, std::vector<int> &pos, std::vector<Ex> &reps)
{
    const size_t m = vals.size();
    std::vector<int> idx(m);
    for (size_t i = 0; i < m; i++) idx[i] = (int)i;
    for (size_t i = 0; i < m; i++)
        for (size_t j = i + 1; j < m; j++)
            if (order(vals[i], vals[j], D) == UNK) return false;
    std::stable_sort(idx.begin(), idx.end(), [&](int a, int b) { return order(vals[a], vals[b], D) == LT; });
    pos.assign(m, 0);
    reps.clear();
    for (size_t k = 0; k < m; k++) {
        const int i = idx[k];
        if (k == 0 || order(vals[idx[k - 1]], vals[i], D) != EQ) reps.push_back(vals[i]);
        pos[i] = (int)reps.size() - 1;
    }
    return true;
}

struct ArrayProg {
    std::vector<Ex> rowv, colv;                 // class representatives
    std::vector<std::vector<uint8_t>> hcell, dcell;   // [row slab][col slab]
};

// Compile one array on domain D.  regs: the array's regions (any order).
bool compile_array(const grophecy_array_desc &A, const std::vector<const grophecy_region_desc *> &regs,
                   const Dom &D, ArrayProg &P)
{
    P = ArrayProg();
    Ex Er = ex_of(A.rows), Ec = ex_of(A.cols);
    // extents R = max(0, rows), C = max(0, cols)
    Ex R, C;
    if (le(Er, ZERO, D)) R = ZERO;
    else if (le(ZERO, Er, D)) R = Er;
    else return false;
    if (le(Ec, ZERO, D)) C = ZERO;
    else if (le(ZERO, Ec, D)) C = Ec;
    else return false;
    if (R == ZERO || C == ZERO) return true;    // empty array: no cells

    struct Box { Ex r0, r1, c0, c1; uint32_t kernel, mode; };
    std::vector<Box> boxes;
    for (const grophecy_region_desc *g : regs) {
        Box b;
        b.kernel = g->kernel;
        b.mode = g->mode;
        if (g->flags & GROPHECY_REGION_WHOLE) {
            if (g->mode & GROPHECY_W) b.mode |= GROPHECY_R;   // may-write (reading 10)
            b.r0 = ZERO; b.r1 = R; b.c0 = ZERO; b.c1 = C;
        } else {
            if (!clamp_sym(ex_of(g->r0), R, D, b.r0) || !clamp_sym(ex_of(g->r1), R, D, b.r1) ||
                !clamp_sym(ex_of(g->c0), C, D, b.c0) || !clamp_sym(ex_of(g->c1), C, D, b.c1))
                return false;
        }
        // always empty on D?
        if (le(b.r1, b.r0, D) || le(b.c1, b.c0, D)) continue;
        if (!le(b.r0, b.r1, D) || !le(b.c0, b.c1, D)) return false;
        boxes.push_back(b);
    }
    std::vector<Ex> rv = {ZERO, R}, cv = {ZERO, C};
    for (const Box &b : boxes) {
        rv.push_back(b.r0); rv.push_back(b.r1);
        cv.push_back(b.c0); cv.push_back(b.c1);
    }
    std::vector<int> rp, cp;
    if (!classify(rv, D, rp, P.rowv) || !classify(cv, D, cp, P.colv)) return false;
    const int nr = (int)P.rowv.size() - 1, nc = (int)P.colv.size() - 1;
    if (nr <= 0 || nc <= 0) return true;
    P.hcell.assign(nr, std::vector<uint8_t>(nc, 0));
    P.dcell.assign(nr, std::vector<uint8_t>(nc, 0));
    const uint32_t INF = 0xffffffffu;
    for (int i = 0; i < nr; i++)
        for (int j = 0; j < nc; j++) {
            uint32_t fr = INF, fw = INF;
            for (size_t q = 0; q < boxes.size(); q++) {
                const int r0 = rp[2 + 2 * q], r1 = rp[3 + 2 * q];
                const int c0 = cp[2 + 2 * q], c1 = cp[3 + 2 * q];
                if (r0 <= i && i + 1 <= r1 && c0 <= j && j + 1 <= c1) {
                    if ((boxes[q].mode & GROPHECY_R) && boxes[q].kernel < fr) fr = boxes[q].kernel;
                    if ((boxes[q].mode & GROPHECY_W) && boxes[q].kernel < fw) fw = boxes[q].kernel;
                }
            }
            P.hcell[i][j] = fr != INF && fr <= fw;
            P.dcell[i][j] = fw != INF;
        }
    return true;
}

// Emit the program of one cell matrix as u32 words: [n_terms] then one word
// per (band, run) term packing four expression indices (u8 each):
//   rs | re << 8 | cs << 16 | ce << 24,
//   count = sum_terms (val[re] - val[rs]) * (val[ce] - val[cs]).
// Bands merge consecutive row slabs with identical column patterns; runs are
// maximal column runs of a band.
template <class F>
void emit(const std::vector<std::vector<uint8_t>> &cell, const std::vector<Ex> &rowv,
          const std::vector<Ex> &colv, F idx, std::vector<uint32_t> &out)
{
    const size_t at = out.size();
    out.push_back(0);
    uint32_t nt = 0;
    const int nr = (int)cell.size();
    int i = 0;
    while (i < nr) {
        bool any = false;
        for (uint8_t v : cell[i]) any |= v != 0;
        if (!any) { i++; continue; }
        int e = i + 1;
        while (e < nr && cell[e] == cell[i]) e++;
        const int nc = (int)cell[i].size();
        for (int j = 0; j < nc;) {
            if (!cell[i][j]) { j++; continue; }
            int k = j + 1;
            while (k < nc && cell[i][k]) k++;
            out.push_back((uint32_t)idx(rowv[i]) | ((uint32_t)idx(rowv[e]) << 8) |
                          ((uint32_t)idx(colv[j]) << 16) | ((uint32_t)idx(colv[k]) << 24));
            nt++;
            j = k;
        }
        i = e;
    }
    out[at] = nt;
}

// Residue-class polynomials.  With nx = 8a + r, ny = 8b + s (0 <= r, s < 8):
//   c1 nx + c2 ny + c3 nx ny = 8 (c1 a + c2 b + c3 (8ab + s a + r b)) + (c1 r + c2 s + c3 r s)
// so every bound v = c0 + floor(L / 8) is EXACTLY bilinear in (a, b) on the
// class (r, s):  v = k0 + k1 a + k2 b + k3 ab with
//   k0 = c0 + floor((c1 r + c2 s + c3 r s) / 8), k1 = c1 + c3 s, k2 = c2 + c3 r, k3 = 8 c3.
// A program term (row e - row s)(col e - col s) is a product of two such forms,
// so each count = sum of terms is a polynomial of degree <= 2 in a and in b,
// exact in wrapping 64-bit arithmetic (the true count fits).  Evaluating the 9
// coefficients replaces evaluating every bound and every term per key.
using u64 = uint64_t;
struct Bil {
    u64 k[4];
};

Bil bil_of(const Ex &e, int64_t r, int64_t s)
{
    Bil v;
    const int64_t rem = e.c1 * r + e.c2 * s + e.c3 * r * s;
    v.k[0] = (u64)(e.c0 + (rem >> 3));   // arithmetic shift: floor
    v.k[1] = (u64)(e.c1 + e.c3 * s);
    v.k[2] = (u64)(e.c2 + e.c3 * r);
    v.k[3] = (u64)(8 * e.c3);
    return v;
}

void compile_polys(const grophecy_skeleton_desc &S, const std::vector<Ex> &table, SkelPlanHost &out)
{
    const uint32_t np = 2 * S.n_arrays;
    std::vector<u64> full((size_t)POLY_CLASSES * np * 9, 0);
    bool biq = false;
    for (uint32_t c = 0; c < POLY_CLASSES; c++) {
        const int64_t r = c >> 3, s = c & 7;
        std::vector<Bil> v(table.size());
        for (size_t e = 0; e < table.size(); e++) v[e] = bil_of(table[e], r, s);
        for (uint32_t a = 0; a < S.n_arrays; a++)
            for (uint32_t dir = 0; dir < 2; dir++) {
                u64 *m = &full[((size_t)c * np + 2 * a + dir) * 9];
                const uint32_t *p = out.prog.data() + (dir ? out.d_off[a] : out.h_off[a]);
                for (uint32_t t = 0; t < p[0]; t++) {
                    const uint32_t w = p[1 + t];
                    const Bil &rs = v[w & 0xff], &re = v[(w >> 8) & 0xff];
                    const Bil &cs = v[(w >> 16) & 0xff], &ce = v[w >> 24];
                    u64 D[4], C[4];
                    for (int i = 0; i < 4; i++) {
                        D[i] = re.k[i] - rs.k[i];
                        C[i] = ce.k[i] - cs.k[i];
                    }
                    m[0] += D[0] * C[0];
                    m[1] += D[0] * C[1] + D[1] * C[0];
                    m[2] += D[0] * C[2] + D[2] * C[0];
                    m[3] += D[0] * C[3] + D[3] * C[0] + D[1] * C[2] + D[2] * C[1];
                    m[4] += D[1] * C[1];
                    m[5] += D[2] * C[2];
                    m[6] += D[1] * C[3] + D[3] * C[1];
                    m[7] += D[2] * C[3] + D[3] * C[2];
                    m[8] += D[3] * C[3];
                }
                const bool live = dir == 0 || (S.arrays[a].flags & GROPHECY_ARRAY_LIVEOUT);
                const u64 eb = live ? S.arrays[a].elem_bytes : 0;
                for (int i = 0; i < 9; i++) {
                    m[i] *= eb;
                    if (i >= 4 && m[i]) biq = true;
                }
            }
    }
    out.poly_stride = biq ? 10 : 4;
    out.poly.assign((size_t)POLY_CLASSES * np * out.poly_stride, 0);
    for (size_t q = 0; q < (size_t)POLY_CLASSES * np; q++)
        for (uint32_t i = 0; i < (biq ? 9u : 4u); i++) out.poly[q * out.poly_stride + i] = full[q * 9 + i];
}

}  // namespace

bool compile_plan(const grophecy_skeleton_desc &S, SkelPlanHost &out)
{
    out = SkelPlanHost();
    // the approximate (hull) mode, strided sections and rank-3 arrays take
    // the general path
    if (S.flags & GROPHECY_SKEL_HULL) return false;
    if (skeleton_rank3(S)) return false;
    for (uint32_t j = 0; j < S.n_regions; j++)
        if (!(S.regions[j].flags & GROPHECY_REGION_WHOLE) &&
            (S.regions[j].r_step > 1 || S.regions[j].c_step > 1))
            return false;
    std::vector<std::vector<const grophecy_region_desc *>> regs(S.n_arrays);
    for (uint32_t j = 0; j < S.n_regions; j++) regs[S.regions[j].array].push_back(&S.regions[j]);

    auto try_dom = [&](int64_t tx, int64_t ty, std::vector<ArrayProg> &progs) {
        const Dom D = {tx, (int64_t)GROPHECY_MAX_DIM, ty, (int64_t)GROPHECY_MAX_DIM};
        progs.assign(S.n_arrays, ArrayProg());
        for (uint32_t a = 0; a < S.n_arrays; a++)
            if (!compile_array(S.arrays[a], regs[a], D, progs[a])) return false;
        return true;
    };
    // smallest domain corner (tx, ty) over powers of two, minimising log tx + log ty
    int best_l = -1, best_tx = 0, best_ty = 0;
    std::vector<ArrayProg> progs;
    for (int ly = 0; ly <= 20; ly++) {
        int lo = 0, hi = 21;   // find minimal lx in [0, 20] that works (21 = none)
        while (lo < hi) {
            const int mid = (lo + hi) / 2;
            if (try_dom(1ll << mid, 1ll << ly, progs)) hi = mid;
            else lo = mid + 1;
        }
        if (lo <= 20 && (best_l < 0 || lo + ly < best_l)) {
            best_l = lo + ly;
            best_tx = lo;
            best_ty = ly;
        }
        if (best_l >= 0 && ly >= best_l) break;
    }
    if (best_l < 0) return false;
    if (!try_dom(1ll << best_tx, 1ll << best_ty, progs)) return false;

    // table: kernel work expressions first (entry k = kernel k, read by the
    // model), then the usage expressions
    std::vector<Ex> table;
    for (uint32_t k = 0; k < S.n_kernels; k++) table.push_back(ex_of(S.kernels[k].work_items));
    auto idx = [&](const Ex &e) -> uint16_t {
        for (size_t i = 0; i < table.size(); i++)
            if (table[i] == e) return (uint16_t)i;
        table.push_back(e);
        return (uint16_t)(table.size() - 1);
    };
    for (uint32_t a = 0; a < S.n_arrays; a++) {
        out.h_off.push_back((uint32_t)out.prog.size());
        emit(progs[a].hcell, progs[a].rowv, progs[a].colv, idx, out.prog);
        out.d_off.push_back((uint32_t)out.prog.size());
        emit(progs[a].dcell, progs[a].rowv, progs[a].colv, idx, out.prog);
    }
    if (table.size() > PLAN_MAX_EXPR) return false;
    for (const Ex &e : table)
        out.exprs.push_back(make_int4((int)e.c0, (int)e.c1, (int)e.c2, (int)e.c3));
    compile_polys(S, table, out);
    out.tx = 1u << best_tx;
    out.ty = 1u << best_ty;
    out.ok = true;
    return true;
}

}  // namespace grophecy

// ---- host evaluation of a plan (diagnostic entry point, mirrors the device) ----
namespace {
int64_t aff8_host(const int4 &c, int64_t nx, int64_t ny)
{
    const int64_t num = (int64_t)c.y * nx + (int64_t)c.z * ny + (int64_t)c.w * nx * ny;
    return (int64_t)c.x + (num >> 3);
}
}  // namespace

using namespace grophecy;

extern "C" int grophecy_plan_usage_host(const grophecy_skeleton_desc *skel, int64_t nx, int64_t ny,
                                        uint64_t *h2d_per_array, uint64_t *d2h_per_array,
                                        uint32_t *plan_tx, uint32_t *plan_ty)
{
    if (!skel || !h2d_per_array || !d2h_per_array) {
        set_error("null argument");
        return GROPHECY_EINVAL;
    }
    SkelPlanHost P;
    if (!compile_plan(*skel, P)) {
        if (plan_tx) *plan_tx = 0xffffffffu;
        if (plan_ty) *plan_ty = 0xffffffffu;
        set_error("skeleton has no usage plan");
        return GROPHECY_ELIMIT;
    }
    if (plan_tx) *plan_tx = P.tx;
    if (plan_ty) *plan_ty = P.ty;
    if (nx < (int64_t)P.tx || ny < (int64_t)P.ty) {
        set_error("size outside the plan's domain");
        return GROPHECY_ELIMIT;
    }
    // the device evaluates the residue-class byte polynomials; the band
    // programs they were derived from are evaluated alongside as a check
    std::vector<int64_t> val(P.exprs.size());
    for (size_t e = 0; e < P.exprs.size(); e++) val[e] = aff8_host(P.exprs[e], nx, ny);
    const uint32_t np = 2 * skel->n_arrays;
    const uint32_t cls = (uint32_t)((nx & 7) * 8 + (ny & 7));
    for (uint32_t a = 0; a < skel->n_arrays; a++) {
        for (int which = 0; which < 2; which++) {
            const uint32_t *p = P.prog.data() + (which ? P.d_off[a] : P.h_off[a]);
            const uint32_t nt = *p++;
            uint64_t cnt = 0;
            for (uint32_t t = 0; t < nt; t++, p++) {
                const uint32_t w = *p;
                cnt += (uint64_t)((val[(w >> 8) & 0xff] - val[w & 0xff]) *
                                  (val[w >> 24] - val[(w >> 16) & 0xff]));
            }
            const uint64_t eb = skel->arrays[a].elem_bytes;
            const bool live = which == 0 || (skel->arrays[a].flags & GROPHECY_ARRAY_LIVEOUT);
            const uint64_t bytes = live ? cnt * eb : 0;
            const uint64_t pb = poly_eval_host(
                P.poly.data() + ((size_t)cls * np + 2 * a + which) * P.poly_stride, P.poly_stride,
                (uint64_t)(nx >> 3), (uint64_t)(ny >> 3));
            if (pb != bytes) {
                set_error("usage polynomial disagrees with its band program");
                return GROPHECY_EINTERNAL;
            }
            if (which == 0) h2d_per_array[a] = pb;
            else d2h_per_array[a] = pb;
        }
    }
    return GROPHECY_OK;
}

// Diagnostic: size of the compiled plan of `skel` (expressions, program words,
// bands and runs summed over arrays, max bands of one array).
extern "C" int grophecy_plan_stats(const grophecy_skeleton_desc *skel, uint32_t *stats)
{
    if (!skel || !stats) return GROPHECY_EINVAL;
    SkelPlanHost P;
    if (!compile_plan(*skel, P)) return GROPHECY_ELIMIT;
    uint32_t bands = 0, runs = 0, maxb = 0, maxw = 0;
    for (uint32_t a = 0; a < skel->n_arrays; a++)
        for (int which = 0; which < 2; which++) {
            const uint32_t nt = P.prog[which ? P.d_off[a] : P.h_off[a]];
            runs += nt;
            bands += nt;
            if (nt > maxb) maxb = nt;
            if (nt + 1 > maxw) maxw = nt + 1;
        }
    stats[0] = (uint32_t)P.exprs.size();
    stats[1] = (uint32_t)P.prog.size();
    stats[2] = bands;
    stats[3] = runs;
    stats[4] = maxb;
    stats[5] = maxw;
    stats[6] = P.poly_stride;
    // distinct residue classes among the 64 byte-polynomial sets
    const size_t blk = 2 * (size_t)skel->n_arrays * P.poly_stride;
    uint32_t distinct = 0;
    for (size_t c = 0; c < POLY_CLASSES; c++) {
        bool seen = false;
        for (size_t e = 0; e < c && !seen; e++)
            seen = std::equal(P.poly.begin() + c * blk, P.poly.begin() + (c + 1) * blk,
                              P.poly.begin() + e * blk);
        distinct += !seen;
    }
    stats[7] = distinct;
    stats[8] = (uint32_t)(P.poly.size() * sizeof(uint64_t));
    return GROPHECY_OK;
}
