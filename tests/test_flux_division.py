"""Pins the arithmetic claim the CUDA flux interpolation (M5, mdn_device.cuh `flux_interp`) rests on.

The oracle evaluates (x - kappa_i) / (kappa_{i+1} - kappa_i) with an IEEE division (P:116 reading
#19).  The kernel instead uses a stored y = RN(1/b) and two FMAs (Markstein's correction):
q = RN(a y), r = fma(-q, b, a), q' = fma(r, y, q), which is RN(a/b) whenever 0 <= a < b and no
over/underflow occurs.  This test checks the claim against IEEE division in C on random,
flux-table-shaped and adversarial operands (all-ones / all-zeros significands, a just below b).
"""
import os
import subprocess
import tempfile

import pytest

SRC = r"""
#include <math.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
static uint64_t s = 0x9E3779B97F4A7C15ull;
static uint64_t xr(void) { s ^= s << 13; s ^= s >> 7; s ^= s << 17; return s; }
static double u01(void) { return (double)(xr() >> 11) * (1.0 / 9007199254740992.0); }
static double bits(uint64_t b) { double d; memcpy(&d, &b, 8); return d; }
int main(int argc, char** argv) {
  long n = atol(argv[1]), bad = 0;
  for (long t = 0; t < n; ++t) {
    double b;
    switch (t % 4) {
      case 0: b = ldexp(1.0 + u01(), (int)(xr() % 40) - 30); break;
      case 1: {  /* significand near all-ones or all-zeros */
        uint64_t m = (xr() & 1) ? 0xFFFFFFFFFFFFFull - (xr() % 64) : (xr() % 64);
        b = bits(((uint64_t)(1011 + xr() % 20) << 52) | m);
        break;
      }
      case 2: {  /* knot spacings of a cumulative-flux table, as the kernel forms them */
        double k1 = 1.5 + 14.0 * u01();
        double k2 = k1 + ldexp(0.5 + u01(), -(int)(xr() % 24) - 1);
        b = k2 - k1;
        break;
      }
      default: b = ldexp(1.0 + u01(), (int)(xr() % 10) - 12);
    }
    double a = u01() * b;
    if (xr() % 8 == 0) a = (1.0 - ldexp(u01(), -(int)(xr() % 52))) * b;
    if (xr() % 16 == 0) a = nextafter(b, 0.0);
    if (xr() % 32 == 0) a = 0.0;
    if (!(a < b)) a = nextafter(b, 0.0);
    volatile double y = 1.0 / b;
    volatile double q = a * y;
    double r = fma(-q, b, a);
    double q2 = fma(r, y, q);
    volatile double ex = a / b;
    if (q2 != ex) {
      if (bad < 5) printf("mismatch a=%a b=%a got=%a ieee=%a\n", a, b, q2, ex);
      ++bad;
    }
  }
  printf("n=%ld bad=%ld\n", n, bad);
  return bad != 0;
}
"""


def test_markstein_quotient_equals_ieee_division():
    with tempfile.TemporaryDirectory() as d:
        c = os.path.join(d, "t.c")
        exe = os.path.join(d, "t")
        open(c, "w").write(SRC)
        try:
            subprocess.run(["gcc", "-O2", "-ffp-contract=off", "-o", exe, c, "-lm"], check=True,
                           capture_output=True, text=True)
        except (OSError, subprocess.CalledProcessError) as e:  # pragma: no cover
            pytest.skip(f"no C compiler: {e}")
        r = subprocess.run([exe, "20000000"], capture_output=True, text=True, timeout=600)
        assert r.returncode == 0, r.stdout + r.stderr
        assert "bad=0" in r.stdout
