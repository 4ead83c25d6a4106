"""Host constants of the CRT ("Ozaki scheme II") FP64-class engine (csrc/crt.cu), pinned against
exact big-integer arithmetic — the Chinese remainder theorem itself, not a retyped formula:
  * the moduli are pairwise coprime and M = prod p_t;
  * for the paired moduli m_j = p_2j p_2j+1, w_j = H_j + L_j reproduces the CRT basis
    (w_j == 1 mod m_j, == 0 mod m_i, i != j) up to the rounding of L_j (< 2^-53 relative), and H_j is
    a multiple of 2^sh with < 2^33 units (so sum_j R_j H_j is exact in FP64 for R_j < 2^16);
  * the operand bit budget b keeps K 2^{2b} < M/2 (the reconstructed integer is unique);
  * a pure-Python model of the device epilogue (modulus reduction, pair combination
    R = r_a + a((r_b - r_a) a^-1 mod b), FP64 reconstruction with exactly the kernel's operations)
    returns sum_k x'_k y'_k to within its final FP64 rounding + 2^64 (relative 2^-58 of the operand
    scale K 2^{2b}) for random full-budget integer dot products.
No GPU needed (the constants are host code of libmpgeo)."""
import ctypes as C
import math
from fractions import Fraction

import numpy as np
import pytest


def _consts(nmod, K):
    from paper_conf_cluster_caoalgkb23_b200._lib import lib
    bits = C.c_int()
    mod = (C.c_int * 16)()
    H = (C.c_double * 16)()
    L = (C.c_double * 16)()
    Mhl = (C.c_double * 2)()
    assert lib.mp_test_crt_constants(nmod, K, C.byref(bits), mod, H, L, Mhl) == 0
    return bits.value, list(mod)[:nmod], list(H)[:nmod // 2], list(L)[:nmod // 2], list(Mhl)


@pytest.mark.parametrize("nmod,K", [(16, 2048), (16, 512), (14, 2048), (8, 2048)])
def test_crt_constants_exact(nmod, K):
    bits, p, H, L, (Mh, Ml) = _consts(nmod, K)
    for i in range(nmod):
        for j in range(i):
            assert math.gcd(p[i], p[j]) == 1
    assert all(2 <= q <= 256 for q in p)
    M = math.prod(p)
    sh = M.bit_length() - 33
    assert int(Fraction(Mh)) % (1 << sh) == 0 and int(Fraction(Mh)) <= M < int(Fraction(Mh)) + (1 << sh)
    assert abs(Fraction(M - int(Fraction(Mh))) - Fraction(Ml)) <= Fraction(Ml) * Fraction(1, 1 << 53)
    m = [p[2 * j] * p[2 * j + 1] for j in range(nmod // 2)]
    for j, mj in enumerate(m):
        Mj = M // mj
        w = Mj * pow(Mj, -1, mj)  # exact CRT basis element for the paired modulus
        assert w % mj == 1 and all(w % m[i] == 0 for i in range(len(m)) if i != j)
        hh = int(Fraction(H[j]))
        assert hh % (1 << sh) == 0 and (hh >> sh) < (1 << 33)
        assert abs(Fraction(w - hh) - Fraction(L[j])) <= Fraction(w - hh) * Fraction(1, 1 << 52) + 1
    assert K * 4**bits < M // 2
    assert not (K * 4 ** (bits + 1) * 2 ** 0.05 < M // 2)


def _mod_canon(a, p):
    """Device mod_canon: q = round(a/p) by a 32-bit multiply-high, then one correction."""
    mq = ((1 << 32) + p // 2) // p
    q = (a * mq + (1 << 31)) >> 32
    r = a - q * p
    assert -p // 2 - 1 <= r <= p // 2 + 1
    return r + p if r < 0 else r


def _device_epilogue(accs, p, H, L, Mh, Ml):
    """Residue reduction, pair combination and FP64 reconstruction exactly as crt_gemm_kernel
    (fma = exact product + one rounding, emulated with Fraction)."""
    def fma(a, b, c):
        return float(Fraction(a) * Fraction(b) + Fraction(c))
    sh = sl = 0.0
    for j in range(len(p) // 2):
        a, b = p[2 * j], p[2 * j + 1]
        ra = _mod_canon(accs[2 * j], a)
        rb = _mod_canon(accs[2 * j + 1], b)
        tt = _mod_canon((rb - ra) * pow(a, -1, b), b)
        R = ra + a * tt
        assert 0 <= R < a * b
        sh = fma(float(R), H[j], sh)
        sl = fma(float(R), L[j], sl)
    invM = 1.0 / float(math.prod(p))
    q = float(round((sh + sl) * invM))
    return fma(-q, Mh, sh) + fma(-q, Ml, sl)


def test_crt_epilogue_model_exact_to_final_rounding():
    nmod, K = 16, 2048
    bits, p, H, L, (Mh, Ml) = _consts(nmod, K)
    rng = np.random.default_rng(5)
    worst = 0.0
    for trial in range(200):
        k = 64
        x = [int(v) >> (62 - bits) for v in rng.integers(-(1 << 62), 1 << 62, k)]
        y = [int(v) >> (62 - bits) for v in rng.integers(-(1 << 62), 1 << 62, k)]
        if trial % 3 == 0:
            y = [abs(v) * (1 if a >= 0 else -1) for v, a in zip(y, x)]  # no cancellation
        X = sum(a * b for a, b in zip(x, y)) * (K // k)
        # INT32 accumulators of the residue GEMMs: any value == X (mod p) with |acc| <= K 128^2
        accs = []
        for q in p:
            r = X % q
            r = r - q if r > 127 else r
            accs.append(r + q * int(rng.integers(-(K * 128 * 128) // q // 2, (K * 128 * 128) // q // 2)))
        got = _device_epilogue(accs, p, H, L, Mh, Ml)
        # error: the L-part FP64 sums (< 2^64 absolute) plus the final rounding of X
        assert abs(Fraction(got) - X) <= Fraction(abs(X)) * Fraction(1, 1 << 52) + (1 << 64), (trial, got, X)
        worst = max(worst, float(abs(Fraction(got) - X)) / (K * 4.0**bits))
    # relative to the operand scale K 2^(2b): at most the final rounding, far below an FP64 GEMM's K u = 2^-42
    assert worst <= 2.0**-52


def test_exact_barrett_reduction_of_the_epilogue():
    """crt.cu mod_canon: r = a' - floor(a' m / 2^38) p with a' = a + p 2^20 and m = ceil(2^38 / p) equals
    a mod p for every |a| <= 2^27 (the INT32 accumulator bound at K <= 8192) and every modulus of the
    engine (dense samples + both ends of the range, exact integer arithmetic)."""
    import numpy as np
    moduli = [256, 255, 253, 251, 247, 241, 239, 233, 229, 227, 223, 217, 211, 199, 197, 193]
    rng = np.random.default_rng(0)
    lim = 1 << 27
    a = np.concatenate([np.arange(-lim, -lim + 50000), np.arange(-50000, 50000), np.arange(lim - 50000, lim + 1),
                        rng.integers(-lim, lim + 1, 500000)]).astype(np.int64)
    for p in moduli:
        m = ((1 << 38) + p - 1) // p
        assert m < (1 << 32)
        ap = (a + (p << 20)).astype(np.uint64)
        assert int(ap.max()) < (1 << 29)
        q = ((ap * np.uint64(m)) >> np.uint64(32)) >> np.uint64(6)  # __umulhi(a', m) >> 6
        r = (ap - q * np.uint64(p)).astype(np.int64)
        assert np.array_equal(r, np.mod(a, p)), p
