"""The two-product division the fast path uses: for a divisor
v whose odd significand is below 2^50, x / v == RN(x * hi + RN(x * lo)) with
hi = RN(1/v), lo = RN((1 - v * hi) / v).  The proof is in DESIGN.md; this test
checks it empirically against the IEEE division of the C compiler (gcc,
-ffp-contract=off, explicit fma()) on random inputs of the kinds the path
uses: integer block counts over integer denominators occ * n_sm, and arbitrary
cycle counts over GPU clock frequencies.
Test infrastructure only: a standalone C snippet, nothing from the product.
"""
import ctypes as C
import os
import subprocess
import tempfile

import pytest

SRC = r"""
#include <math.h>
#include <stdint.h>
static uint64_t s;
static uint64_t nx(void) { uint64_t z = (s += 0x9E3779B97F4A7C15ull);
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull; z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31); }
static double q2(double x, double hi, double lo) { return fma(x, hi, x * lo); }
/* kind 0: integer x in [1, 2^30), integer v in [1, 2^20); kind 1: x = random
   double in [2^-20, 2^60), v = given divisor.  Returns the mismatch count. */
long long run(int kind, double v_fixed, long long n, uint64_t seed) {
  s = seed; long long bad = 0;
  for (long long i = 0; i < n; i++) {
    double v, x;
    if (kind == 0) { v = (double)(1 + nx() % ((1u << 20) - 1)); x = (double)(1 + nx() % ((1u << 30) - 1)); }
    else { v = v_fixed; x = ldexp(1.0 + (double)(nx() >> 11) * 0x1p-53, (int)(nx() % 80) - 20); }
    double hi = 1.0 / v, lo = fma(-v, hi, 1.0) / v;
    if (q2(x, hi, lo) != x / v) bad++;
  }
  return bad;
}
"""


@pytest.fixture(scope="module")
def lib():
    d = tempfile.mkdtemp()
    c, so = os.path.join(d, "d.c"), os.path.join(d, "d.so")
    open(c, "w").write(SRC)
    subprocess.check_call(["gcc", "-O2", "-ffp-contract=off", "-fno-fast-math", "-fPIC",
                           "-shared", "-o", so, c, "-lm"])
    L = C.CDLL(so)
    L.run.argtypes = [C.c_int, C.c_double, C.c_longlong, C.c_uint64]
    L.run.restype = C.c_longlong
    return L


def test_integer_over_integer(lib):
    assert lib.run(0, 0.0, 20_000_000, 1) == 0


@pytest.mark.parametrize("freq", [1.35e9, 1.965e9, 1.4e9, 7e8, 2.1e9 + 1, 1e6])
def test_any_double_over_clock(lib, freq):
    assert lib.run(1, freq, 5_000_000, 2) == 0

