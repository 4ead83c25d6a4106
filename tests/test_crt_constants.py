"""Host constants of the CRT ("Ozaki scheme II") FP64-class engine (csrc/crt.cu), pinned against
exact big-integer arithmetic — the Chinese remainder theorem itself, not a retyped formula:
  * the moduli are pairwise coprime and M = prod p_t;
  * for the paired moduli m_j = p_2j p_2j+1, w_j = H_j + L_j reproduces the CRT basis
    (w_j == 1 mod m_j, == 0 mod m_i, i != j) up to the rounding of L_j (< 2^-53 relative), and H_j is
    a multiple of 2^sh with < 2^33 units (so sum_j R_j H_j is exact in FP64 for R_j < 2^16);
  * the operand bit budget b keeps K 2^{2b} < M/2 (the reconstructed integer is unique);
  * the element reconstruction the GEMM epilogue runs (crt_recon_bits, integer + FP32 arithmetic;
    called on the host through mp_test_crt_recon) returns X 2^e0 for every integer X with
    |X| <= K 2^{2b} given only its pair residues, to within one FP64 rounding + 2^(51.6 + e0) (the
    dropped low limb, ld = 1) — exact quotient included — checked against Python big integers on
    random, extreme (+-K 2^{2b}, the 0.3 M edge), tiny and zero values;
  * the bit budget b is the largest with K 2^{2b} <= 0.3 M (the quotient estimate's margin).
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
    assert 10 * K * 4**bits <= 3 * M and not (10 * K * 4 ** (bits + 1) <= 3 * M)


def _recon(nmod, K, X, e0, neg=0):
    """crt_recon_bits on the host for integers X (Python ints): pair residues in, FP64 out."""
    from paper_conf_cluster_caoalgkb23_b200._lib import lib
    _, p, _, _, _ = _consts(nmod, K)
    m = [p[2 * j] * p[2 * j + 1] for j in range(nmod // 2)]
    R = (C.c_uint32 * (len(X) * len(m)))(*[x % mj for x in X for mj in m])
    E = (C.c_int * len(X))(*e0)
    out = (C.c_double * len(X))()
    assert lib.mp_test_crt_recon(nmod, K, R, E, len(X), neg, out) == 0
    return list(out)


@pytest.mark.parametrize("nmod,K", [(16, 2048), (16, 512), (14, 2048), (8, 2048)])
def test_crt_reconstruction_exact_to_final_rounding(nmod, K):
    bits, p, _, _, _ = _consts(nmod, K)
    M = math.prod(p)
    Xmax = K * 4**bits
    ld = 1 if M.bit_length() > 64 else 0
    rng = np.random.default_rng(7 + nmod)
    X = [0, 1, -1, Xmax, -Xmax, Xmax - 1, -(Xmax - 1), 3 * M // 10, -(3 * M // 10)]
    X += [s * (1 << k) + int(rng.integers(0, 1 << 20)) for k in range(0, Xmax.bit_length(), 3) for s in (1, -1)]
    X += [int.from_bytes(rng.bytes(16), "little") % (2 * Xmax + 1) - Xmax for _ in range(3000)]
    # quotient-estimate stress: X near the integer multiples' edges +-0.3 M (S/M = q +- 0.3)
    X += [3 * M // 10 - int(rng.integers(0, 1 << 40)) for _ in range(200)]
    X += [-(3 * M // 10) + int(rng.integers(0, 1 << 40)) for _ in range(200)]
    e0 = [int(v) for v in rng.integers(-2 * bits - 200, -2 * bits + 100, len(X))]
    for neg in (0, 1):
        got = _recon(nmod, K, X, e0, neg)
        for x, e, g in zip(X, e0, got):
            exact = Fraction(-x if neg else x) * Fraction(2) ** e
            tol = abs(exact) * Fraction(1, 1 << 52) + (Fraction(2) ** (e + 52) if ld else 0)
            assert abs(Fraction(g) - exact) <= tol, (nmod, x, e, g, float(exact))
            if x == 0:
                assert g == 0.0


def test_crt_reconstruction_flushes_below_fp64_range():
    nmod, K = 16, 2048
    bits, _, _, _, _ = _consts(nmod, K)
    got = _recon(nmod, K, [12345, -12345], [-1300, -1300])
    assert got == [0.0, 0.0]


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


def test_shoup_pair_combination_of_the_epilogue():
    """crt.cu residue step of the second modulus b of each pair: t = ((acc_b - r_a) a^-1) mod b by Shoup's
    multiplication — x = acc_b - r_a + b 2^21 (in [0, 2^32) for |acc_b| <= 2^27, r_a < 256),
    r = x ia - floor(x floor(ia 2^32 / b) / 2^32) b (mod 2^32) in [0, 2b), t = min(r, r - b) unsigned —
    equals the exact modular value for every pair of the engine (both range ends + random samples)."""
    moduli = [256, 255, 253, 251, 247, 241, 239, 233, 229, 227, 223, 217, 211, 199, 197, 193]
    rng = np.random.default_rng(1)
    lim = 1 << 27
    acc = np.concatenate([np.arange(-lim, -lim + 20000), np.arange(-20000, 20000), np.arange(lim - 20000, lim + 1),
                          rng.integers(-lim, lim + 1, 300000)]).astype(np.int64)
    ra = rng.integers(0, 256, acc.size).astype(np.int64)
    M32 = np.uint64(0xFFFFFFFF)
    for j in range(8):
        a, b = moduli[2 * j], moduli[2 * j + 1]
        ia = pow(a, -1, b)
        ra_j = ra % a
        sh = (ia << 32) // b
        x = (acc - ra_j + (b << 21)).astype(np.uint64)
        assert int(x.min()) >= 0 and int(x.max()) < (1 << 32)
        q = (x * np.uint64(sh)) >> np.uint64(32)
        r = (x * np.uint64(ia) - q * np.uint64(b)) & M32
        assert int(r.max()) < 2 * b
        t = np.minimum(r, (r - np.uint64(b)) & M32).astype(np.int64)
        assert np.array_equal(t, np.mod((acc - ra_j) * ia, b)), (a, b)
        R = ra_j + a * t  # the combined pair residue
        assert np.array_equal(R % a, np.mod(acc * 0 + ra_j, a)) and np.array_equal(R % b, np.mod(acc, b))
