"""Pin for the device's Eq. 2 division (R5''').

The CUDA path computes each quotient of Eq. 2 (sqrt(V)/(kT), OV/T, (OV/T)/k)
as q = a*rb, then two FMA corrections q += (a - b q) rb, from rb = RN(1/b)
precomputed on the host (split_device.cuh div_rcp_rn).  The oracle divides
with IEEE '/'.  Markstein's theorem says the second correction is the
correctly rounded quotient once the first has made q faithful; this test
checks the claim independently of both implementations: the same five
operations in C (fma from libm, -ffp-contract=off) against C's '/' over the
operand ranges Eq. 2 produces and random doubles.
"""
import os
import shutil
import subprocess
import tempfile

import pytest

SRC = r"""
#include <math.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
static uint64_t s = 0x9E3779B97F4A7C15ull;
static uint64_t rnd(void) { s ^= s << 13; s ^= s >> 7; s ^= s << 17; return s; }
static double div_rcp(double a, double b, double rb) {
    double q = a * rb;
    double r = fma(-b, q, a);
    q = fma(r, rb, q);
    r = fma(-b, q, a);
    return fma(r, rb, q);
}
static long bad = 0, n = 0;
static void chk(double a, double b) {
    ++n;
    if (div_rcp(a, b, 1.0 / b) != a / b) { if (bad < 5) printf("MISMATCH %a / %a\n", a, b); ++bad; }
}
int main(int argc, char** argv) {
    long N = atol(argv[1]);
    /* structured: every k in [1, 1024] against chain totals T and block-count products k*T */
    for (uint64_t k = 1; k <= 1024; ++k)
        for (int i = 0; i < 200; ++i) {
            uint64_t T = (rnd() >> 32) | 1;                   /* T < 2^32 */
            uint64_t OV = rnd() >> (32 + rnd() % 32);         /* OV < 2^32 */
            uint64_t V = rnd() >> (1 + rnd() % 63);           /* V < 2^63 */
            double y = (double)OV / (double)T;
            chk((double)OV, (double)T);
            chk(y, (double)k);
            chk(sqrt((double)(int64_t)V), (double)k * (double)T);
        }
    /* random operands */
    for (long i = 0; i < N; ++i) {
        double a = ldexp((double)(rnd() >> 11), -(int)(rnd() % 64));
        double b = ldexp((double)((rnd() >> 11) | 1), -(int)(rnd() % 40));
        chk(a, b);
    }
    chk(0.0, 3.0);
    chk(1.0, 3.0);
    chk(2.0, 2.0);
    printf("checked %ld mismatches %ld\n", n, bad);
    return bad != 0;
}
"""


@pytest.mark.skipif(shutil.which("gcc") is None, reason="gcc not available")
def test_reciprocal_two_fma_division_is_ieee_division():
    with tempfile.TemporaryDirectory() as d:
        c = os.path.join(d, "div.c")
        exe = os.path.join(d, "div")
        open(c, "w").write(SRC)
        subprocess.run(["gcc", "-O2", "-ffp-contract=off", "-fno-fast-math", "-o", exe, c, "-lm"], check=True)
        r = subprocess.run([exe, "3000000"], capture_output=True, text=True)
        assert r.returncode == 0, r.stdout
        assert "mismatches 0" in r.stdout
