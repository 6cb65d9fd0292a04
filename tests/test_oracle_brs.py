"""Oracle pins for the full-BRS row:
* strided sections [l:u:s] ([5]) in the exact cell method against
  the literal per-element bitmap, and hand-counted cases;
* irregular ("may") writes (reading 10) by hand;
* the Havlak-Kennedy approximate UNION mode (N4h): hand-computed
  unions / containment, the proven bound hull >= exact, equality on the
  paper's whole-array workloads (Table I skeletons) and on one-read /
  one-write arrays."""
import numpy as np
import pytest

from synth import skeletons as S
from tests.tiny import DUMMY_KX, random_tiny_skeleton, rng


def _sk(arrays, regions, K=2, hull=False):
    s = {"name": "t", "arrays": arrays,
         "kernels": [{"name": f"k{k}", "work": (0, 0, 0, 8), "per_iter": True} for k in range(K)],
         "regions": regions, "kx": [[DUMMY_KX] * K]}
    if hull:
        s["hull"] = True
    return s


def _arr(rows, cols, eb=1, liveout=True):
    return {"name": "a", "rows": (rows, 0, 0, 0), "cols": (cols, 0, 0, 0), "elem_bytes": eb,
            "liveout": liveout}


def _reg(k, mode, r0, r1, c0, c1, rs=1, cs=1, whole=False, a=0):
    return {"kernel": k, "array": a, "mode": mode, "whole": whole, "r0": (r0, 0, 0, 0),
            "r1": (r1, 0, 0, 0), "c0": (c0, 0, 0, 0), "c1": (c1, 0, 0, 0), "r_step": rs,
            "c_step": cs}


def _u(O, sk, nx=1, ny=1, bitmap=False):
    h, d = O.usage(sk, nx, ny, bitmap=bitmap)
    return [int(v) for v in h], [int(v) for v in d]


def test_strided_hand_counts(O):
    # 1 x 10 row, read columns 0,2,4,6,8 then write columns 1,4,7 (stride 3 from 1)
    sk = _sk([_arr(1, 10)], [_reg(0, "R", 0, 1, 0, 10, cs=2), _reg(1, "W", 0, 1, 1, 10, cs=3)])
    assert _u(O, sk) == ([5], [3])
    # the lattice is anchored at the unclamped lower bound: [-1:10:2] covers 1,3,5,7,9
    sk = _sk([_arr(1, 10)], [_reg(0, "R", 0, 1, -1, 10, cs=2)])
    assert _u(O, sk) == ([5], [0])
    # written (stride 2 from 0) before read (dense): only odd columns go H2D
    sk = _sk([_arr(1, 10)], [_reg(0, "W", 0, 1, 0, 10, cs=2), _reg(1, "R", 0, 1, 0, 10)])
    assert _u(O, sk) == ([5], [5])
    # 2-D: 6 x 6, rows 0,3 x cols 0,2,4 read, rows 1..5 step 2 written
    sk = _sk([_arr(6, 6, eb=4)], [_reg(0, "R", 0, 6, 0, 6, rs=3, cs=2),
                                 _reg(0, "W", 1, 6, 0, 6, rs=2)])
    assert _u(O, sk) == ([2 * 3 * 4], [3 * 6 * 4])


def test_maywrite_hand_counts(O):
    W = dict(whole=True)
    # an irregular write alone: every element may be written -> the original
    # data must be on the GPU (H2D) and everything comes back (D2H)
    sk = _sk([_arr(4, 4)], [_reg(0, "W", 0, 0, 0, 0, **W)])
    assert _u(O, sk) == ([16], [16])
    # after a full regular write, nothing needs to go H2D
    sk = _sk([_arr(4, 4)], [_reg(0, "W", 0, 4, 0, 4), _reg(1, "W", 0, 0, 0, 0, **W)])
    assert _u(O, sk) == ([0], [16])
    # partially written first: only the rest goes H2D
    sk = _sk([_arr(4, 4)], [_reg(0, "W", 0, 2, 0, 4), _reg(1, "W", 0, 0, 0, 0, **W)])
    assert _u(O, sk) == ([8], [16])
    # temporaries: nothing back
    sk = _sk([_arr(4, 4, liveout=False)], [_reg(0, "W", 0, 0, 0, 0, **W)])
    assert _u(O, sk) == ([16], [0])
    # irregular read-modify-write equals the may-write
    sk = _sk([_arr(4, 4)], [_reg(0, "RW", 0, 0, 0, 0, **W)])
    assert _u(O, sk) == ([16], [16])


@pytest.mark.parametrize("seed", range(6))
def test_strided_cells_equal_bitmap(O, seed):
    r = rng(4000 + seed)
    for _ in range(300):
        sk, nx, ny = random_tiny_skeleton(r, strided=True, maywrite=True)
        assert _u(O, sk, nx, ny) == _u(O, sk, nx, ny, bitmap=True), (sk, nx, ny)


def test_hull_hand_cases(O):
    # HK union of [0:8:2] and [1:9:2] is [0:9:1]: 10 elements (exact: 10 as well)
    sk = _sk([_arr(1, 10)], [_reg(0, "R", 0, 1, 0, 9, cs=2), _reg(0, "R", 0, 1, 1, 10, cs=2)],
             hull=True)
    assert _u(O, sk) == ([10], [0])
    # [0:4:4] u [6:6:2] (singleton): gcd(4, 0, 6) = 2 -> [0:6:2] = 4 elements
    sk = _sk([_arr(1, 10)], [_reg(0, "R", 0, 1, 0, 5, cs=4), _reg(0, "R", 0, 1, 6, 7, cs=2)],
             hull=True)
    assert _u(O, sk) == ([4], [0])
    exact = dict(sk, hull=False)
    assert _u(O, exact) == ([3], [0])
    # writes [0,2) and [8,10) then a read of [4,6): not inside ONE earlier
    # write section -> kept (2 elements); written data = hull [0:9] = 10
    regs = [_reg(0, "W", 0, 1, 0, 2), _reg(0, "W", 0, 1, 8, 10), _reg(1, "R", 0, 1, 4, 6)]
    assert _u(O, _sk([_arr(1, 10)], regs, hull=True)) == ([2], [10])
    assert _u(O, _sk([_arr(1, 10)], regs)) == ([2], [4])
    # a read inside one earlier write section is "previously written"
    regs = [_reg(0, "W", 0, 1, 0, 10), _reg(1, "R", 0, 1, 3, 7)]
    assert _u(O, _sk([_arr(1, 10)], regs, hull=True)) == ([0], [10])
    # ...but not one of the same kernel (reads see the pre-kernel state)
    regs = [_reg(0, "W", 0, 1, 0, 10), _reg(0, "R", 0, 1, 3, 7)]
    assert _u(O, _sk([_arr(1, 10)], regs, hull=True)) == ([4], [10])
    # a strided write does not contain a dense read of its range
    regs = [_reg(0, "W", 0, 1, 0, 10, cs=2), _reg(1, "R", 0, 1, 0, 10, cs=4)]
    assert _u(O, _sk([_arr(1, 10)], regs, hull=True)) == ([0], [5])
    regs = [_reg(0, "W", 0, 1, 0, 10, cs=2), _reg(1, "R", 0, 1, 1, 10, cs=4)]
    assert _u(O, _sk([_arr(1, 10)], regs, hull=True)) == ([3], [5])


@pytest.mark.parametrize("seed", range(4))
def test_hull_is_an_upper_bound_of_exact(O, seed):
    """Proven in DESIGN.md N4h: a read section is dropped only if one earlier
    write contains it, so every element read before written is in the read
    hull; the write hull contains every written element."""
    r = rng(5000 + seed)
    for _ in range(400):
        sk, nx, ny = random_tiny_skeleton(r, strided=bool(seed % 2), maywrite=True)
        he, de = _u(O, sk, nx, ny)
        hh, dh = _u(O, dict(sk, hull=True), nx, ny)
        assert all(a <= b for a, b in zip(he, hh)) and all(a <= b for a, b in zip(de, dh))


def test_hull_equals_exact_single_sections(O):
    """One read section and one write section per array, the read in an
    earlier or equal kernel: the hull is the section itself in both modes."""
    r = rng(77)
    n = 0
    for _ in range(2000):
        sk, nx, ny = random_tiny_skeleton(r, strided=True, max_regions=6)
        ok = True
        for a in range(len(sk["arrays"])):
            rd = [g for g in sk["regions"] if g["array"] == a and "R" in g["mode"]]
            wr = [g for g in sk["regions"] if g["array"] == a and "W" in g["mode"]]
            if len(rd) > 1 or len(wr) > 1 or (rd and wr and rd[0]["kernel"] > wr[0]["kernel"]):
                ok = False
        if not ok:
            continue
        n += 1
        assert _u(O, sk, nx, ny) == _u(O, dict(sk, hull=True), nx, ny), sk
    assert n > 100


@pytest.mark.parametrize("make", [S.s1_hotspot, S.s2_hotspot_pp2, S.s3_srad, S.s4_cfd,
                                  S.s5_vecadd, S.s6_stassuij])
def test_hull_equals_exact_on_table1_workloads(O, make):
    """The paper's applications access whole arrays (Table I): the
    approximate mode reproduces the exact sizes."""
    sk = make()
    for n in (64, 512, 1024, 4096):
        nx, ny = (n, 1) if sk["name"] in ("cfd", "vecadd") else (n, n)
        if sk["name"] == "stassuij":
            nx, ny = 2048, 132
        assert _u(O, sk, nx, ny) == _u(O, dict(sk, hull=True), nx, ny)
