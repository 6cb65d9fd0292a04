"""The seeded input generators (no method arithmetic here)."""
import numpy as np

from synth import records as R
from synth import skeletons as S
from synth.splitmix import Stream, counter, mix64


def test_splitmix64_reference_vector():
    # Vigna's splitmix64.c with seed 0: first output 0xE220A8397B1DCDAF
    st = Stream(0)
    assert st.next() == 0xE220A8397B1DCDAF
    assert counter(0, 0) == 0xE220A8397B1DCDAF
    v = counter(0, np.arange(4, dtype=np.uint64))
    assert int(v[0]) == 0xE220A8397B1DCDAF
    assert [int(x) for x in v[1:]] == [counter(0, k) for k in (1, 2, 3)]


def test_records_closed_form_any_slice():
    c = R.config("c4")
    full = R.gen_records(c, 10**9 - 5000, 10**9)
    part = R.gen_records(c, 10**9 - 1234, 10**9 - 17)
    for k in full:
        assert np.array_equal(full[k][5000 - 1234:5000 - 17], part[k])


def test_group_structure():
    c = R.with_n(R.config("c3"), 4096)
    rec = R.gen_records(c)
    x = rec["skx"] & 0xFFFF
    assert np.array_equal(x, np.arange(4096) % 16)
    for f in ("nx", "ny", "iters"):
        g = rec[f].reshape(-1, 16)
        assert (g == g[:, :1]).all()
    assert (rec["nx"] >= 256).all() and (rec["nx"] <= 8192).all()
    assert (rec["iters"] >= 1).all() and (rec["iters"] <= 1024).all()


def test_c4_size_rules():
    c = R.config("c4")
    G = c["n"] // 16
    names = [s["name"] for s in c["skeletons"]]
    for sidx, name in enumerate(names):
        g0 = -(-sidx * G // 16)
        rec = R.gen_records(c, g0 * 16, g0 * 16 + 64)
        assert ((rec["skx"] >> 16) == sidx).all()
        if name in ("cfd", "vecadd"):
            assert (rec["ny"] == 1).all() and (rec["nx"] >= 1024).all()
        elif name == "stassuij":
            assert (rec["nx"] == 2048).all() and (rec["ny"] == 132).all()
        else:
            assert np.array_equal(rec["nx"], rec["ny"])


def test_random_skeletons_respect_limits():
    for s in S.random_skeletons(0x5EED0003, 64):
        assert 4 <= len(s["kernels"]) <= 16 and len(s["arrays"]) == 8
        assert len(s["regions"]) <= 256
        for a in range(8):
            assert sum(1 for r in s["regions"] if r["array"] == a) <= 32
        for row in s["kx"]:
            for c in row:
                assert c["total"] >= c["coal"] + c["uncoal"]
        assert all(not r["whole"] or r["mode"] == "R" for r in s["regions"])
