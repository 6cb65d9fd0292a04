"""Rank-3 arrays (SURVEY §8(f) NEXT-3 "rank-3 arrays"; N4r): the
oracle's cell method with plane slabs against the literal per-element
definition, closed-form 3-D stencil counts, the reduction to 2-D, and the
hull bound.  Arrays are [planes][rows][cols]; a region's planes are [p0, p1)."""
import pytest

from tests.tiny import random_tiny_skeleton, rng


def _u(O, sk, nx=8, ny=8, bitmap=False):
    h, d = O.usage(sk, nx, ny, bitmap=bitmap)
    return [int(v) for v in h], [int(v) for v in d]


def _arr(P, R, C, eb=4, liveout=True):
    return {"name": "a", "rows": (R, 0, 0, 0), "cols": (C, 0, 0, 0), "planes": (P, 0, 0, 0),
            "elem_bytes": eb, "liveout": liveout}


def _reg(k, mode, p0, p1, r0, r1, c0, c1, whole=False, a=0):
    return {"kernel": k, "array": a, "mode": mode, "whole": whole,
            "p0": (p0, 0, 0, 0), "p1": (p1, 0, 0, 0), "r0": (r0, 0, 0, 0), "r1": (r1, 0, 0, 0),
            "c0": (c0, 0, 0, 0), "c1": (c1, 0, 0, 0)}


def _sk(arrays, regions, K=2, hull=False):
    from tests.tiny import DUMMY_KX
    s = {"name": "r3", "arrays": arrays,
         "kernels": [{"name": f"k{k}", "work": (64, 0, 0, 0), "per_iter": True} for k in range(K)],
         "regions": regions, "kx": [[DUMMY_KX] * K]}
    if hull:
        s["hull"] = True
    return s


def test_stencil_7point_closed_form(O):
    """out[1:P-1][1:R-1][1:C-1] = f(in[...]): H2D = P R C (in), D2H = (P-2)(R-2)(C-2)."""
    P, R, C = 5, 6, 7
    sk = _sk([_arr(P, R, C), _arr(P, R, C)],
             [_reg(0, "R", 0, P, 0, R, 0, C, a=0), _reg(0, "W", 1, P - 1, 1, R - 1, 1, C - 1, a=1)])
    assert _u(O, sk) == ([4 * P * R * C, 0], [0, 4 * (P - 2) * (R - 2) * (C - 2)])


def test_plane_ranges_first_reader_writer(O):
    """Kernel 0 writes planes [0, 2), kernel 1 reads planes [1, 4): only planes
    2 and 3 are read before written; all written planes come back."""
    sk = _sk([_arr(4, 2, 3)], [_reg(0, "W", 0, 2, 0, 2, 0, 3), _reg(1, "R", 1, 4, 0, 2, 0, 3)])
    assert _u(O, sk) == ([4 * 2 * 2 * 3], [4 * 2 * 2 * 3])
    # a whole (irregular) read covers every plane
    sk = _sk([_arr(4, 2, 3)], [_reg(0, "R", 0, 0, 0, 0, 0, 0, whole=True)], K=1)
    assert _u(O, sk) == ([4 * 4 * 2 * 3], [0])
    # empty and clamped plane ranges
    sk = _sk([_arr(4, 2, 3)], [_reg(0, "R", 3, 3, 0, 2, 0, 3), _reg(0, "R", -5, 1, 0, 2, 0, 3),
                               _reg(1, "W", 3, 99, 0, 1, 0, 1)])
    assert _u(O, sk) == ([4 * 1 * 2 * 3], [4 * 1])


def test_single_plane_equals_2d(O):
    r = rng(9100)
    for _ in range(200):
        sk, nx, ny = random_tiny_skeleton(r, strided=True, maywrite=True)
        sk3 = dict(sk, arrays=[dict(a, planes=(1, 0, 0, 0)) for a in sk["arrays"]],
                   regions=[dict(g, p0=(0, 0, 0, 0), p1=(1, 0, 0, 0)) for g in sk["regions"]])
        assert _u(O, sk, nx, ny) == _u(O, sk3, nx, ny)


@pytest.mark.parametrize("seed", range(4))
def test_rank3_cells_equal_bitmap(O, seed):
    r = rng(9200 + seed)
    for _ in range(250):
        sk, nx, ny = random_tiny_skeleton(r, strided=seed % 2 == 1, maywrite=True, rank3=True)
        assert _u(O, sk, nx, ny) == _u(O, sk, nx, ny, bitmap=True), (sk, nx, ny)


def test_rank3_hull_bounds_exact(O):
    r = rng(9300)
    for _ in range(300):
        sk, nx, ny = random_tiny_skeleton(r, maywrite=True, rank3=True)
        eh, ed = _u(O, sk, nx, ny)
        hh, hd = _u(O, dict(sk, hull=True), nx, ny)
        assert all(a <= b for a, b in zip(eh, hh)) and all(a <= b for a, b in zip(ed, hd))
