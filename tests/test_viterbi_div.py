"""The batched engine's Viterbi division (csrc/kernels.cuh `vit_div`, reading Q13) must equal
the binary32 quotient RN(x / w) bit for bit.  Its fast path replaces the division by
q = RN(x * RN(1/w)), e = x - q*w (one FMA, exact) and RN(q + e * RN(1/w)) (Markstein's
correction) for w <= 64 and x >= 2^-64.  Within that range the quotient, the product and the
residual stay normal, so each result scales exactly with x's exponent: checking every
significand of a few binades for every w decides the whole range.  The check is written in C
(IEEE binary32 with hardware / libm FMA, no contraction), independent of the CUDA source and of
the oracle.
"""
import ctypes
import os
import subprocess
import tempfile

import numpy as np
import pytest

C_SRC = r"""
#include <math.h>
#include <stdint.h>
#include <string.h>
static float f(uint32_t b) { float x; memcpy(&x, &b, 4); return x; }
static uint32_t u(float x) { uint32_t b; memcpy(&b, &x, 4); return b; }
/* mismatches of the fast path over all significands of the binade [2^e, 2^(e+1)) for w = 1..wmax */
long long check(int e, int wmax) {
    long long bad = 0;
    #pragma omp parallel for reduction(+:bad) schedule(static)
    for (int w = 1; w <= wmax; ++w) {
        const float b = (float)w;
        const volatile float one = 1.0f;
        const float r = one / b;                       /* RN(1/w) */
        for (uint32_t m = 0; m < (1u << 23); ++m) {
            const float x = f(((uint32_t)(e + 127) << 23) | m);
            const volatile float qv = x * r;           /* RN(x*r), no contraction */
            const float q = qv;
            const float res = fmaf(-q, b, x);           /* exact residual */
            const float q2 = fmaf(res, r, q);
            const volatile float ref = x / b;           /* RN(x/w) */
            if (u(q2) != u(ref)) ++bad;
        }
    }
    return bad;
}
"""


@pytest.fixture(scope="module")
def lib():
    d = tempfile.mkdtemp()
    src, so = os.path.join(d, "vd.c"), os.path.join(d, "vd.so")
    with open(src, "w") as fh:
        fh.write(C_SRC)
    subprocess.check_call(["gcc", "-O2", "-fopenmp", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared",
                           src, "-o", so, "-lm"])
    lb = ctypes.CDLL(so)
    lb.check.restype = ctypes.c_longlong
    lb.check.argtypes = [ctypes.c_int, ctypes.c_int]
    return lb


@pytest.mark.parametrize("exp", [0, -1, -64])
def test_fast_division_is_correctly_rounded(lib, exp):
    # binades [1,2), [1/2,1) (Viterbi values are <= 1) and the fast path's lower edge [2^-64, 2^-63)
    assert lib.check(exp, 64) == 0


def test_fast_path_guard_matches_kernel():
    """The constants the proof above relies on are the ones the kernel uses."""
    csrc = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                        "paper_conf_eurosys_0002a0a024_b200", "csrc")
    src = open(os.path.join(csrc, "kernels.cuh")).read()
    eng = open(os.path.join(csrc, "engine_batch.cu")).read()
    assert "w <= 64u ? s_rcp[w] : 0.0f" in eng                                           # fast path: w <= 64
    assert "s_rcp[threadIdx.x] = threadIdx.x ? __frcp_rn((float)threadIdx.x) : 0.0f" in eng  # r = RN(1/w)
    assert "threadIdx.x <= 64" in eng                                                      # table covers 0..64
    assert "x >= 0x1p-64f" in src                                                          # vit_div's guard
    assert "lo < 0x1F7FFFFFu" in src and "lo = min(lo, a[i] - 1u)" in src                  # vit_div4's guard
    assert np.float32(2.0 ** -64).view(np.uint32) == 0x1F800000                            # = x >= 2^-64
