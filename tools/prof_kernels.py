"""Launch the hot kernels in isolation (for ncu --set full): K5 DMMA GEMM at a trailing-update shape
and the two tcgen05 GEMMs; also measures the 3xTF32 error growth with K (reading C13)."""
import ctypes as C
import sys
import os

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_cluster_caoalgkb23_b200._lib import lib  # noqa: E402


def p(t):
    return C.c_void_p(t.data_ptr())


def main(which):
    torch.cuda.set_device(0)
    if which in ("dgemm", "all"):
        M, N, K = 8192, 8192, 2048
        A = torch.randn(M, K, dtype=torch.float64, device="cuda")
        B = torch.randn(N, K, dtype=torch.float64, device="cuda")
        Cm = torch.randn(M, N, dtype=torch.float64, device="cuda")
        for _ in range(3):
            assert lib.mp_test_dgemm(p(A), p(B), p(Cm), M, N, K, K, K, N, 0, -1.0, 1.0, 0, 0) == 0
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record()
        for _ in range(5):
            lib.mp_test_dgemm(p(A), p(B), p(Cm), M, N, K, K, K, N, 0, -1.0, 1.0, 0, 0)
        e.record()
        torch.cuda.synchronize()
        print("dgemm TF/s", 5 * 2 * M * N * K / (s.elapsed_time(e) / 1e3) / 1e12)
    if which in ("tc", "all"):
        nb, nt = 2048, 4
        P = torch.randn(nt * nb, nb, dtype=torch.float64, device="cuda") * 0.1
        Cf = torch.zeros(nb, nb, device="cuda")
        hi = torch.randn(nt * nb, nb, device="cuda")
        lo = torch.randn(nt * nb, nb, device="cuda") * 1e-4
        for _ in range(3):
            assert lib.mp_test_tc_gemm_split(0, p(P), p(Cf), nb, nt, 1, 0, 0) == 0
            assert lib.mp_test_tc_gemm_split(2, p(P), p(Cf), nb, nt, 1, 0, 0) == 0
            assert lib.mp_test_tc_gemm(1, p(hi), p(lo), p(Cf), nb, nt, 1, 0) == 0
    if which in ("tf32err", "all"):
        from tests.test_gpu_kernels import tf32_rna
        for K in (64, 256, 1024, 2048):
            rng = np.random.default_rng(K)
            A32 = rng.standard_normal((2 * 256, K)).astype(np.float32)
            h = tf32_rna(A32)
            l = tf32_rna((A32 - h).astype(np.float32))
            # panel rows = 2 tiles of K rows, nb = K (square tiles), use tiles (1, 0)
            nbk = K
            Ab = np.zeros((2 * nbk, nbk), np.float32)
            Ab[: 2 * 256] = A32[:, :nbk] if K >= 512 else 0
            rng2 = np.random.default_rng(1)
            Af = rng2.standard_normal((2 * nbk, nbk)).astype(np.float32)
            H, L = tf32_rna(Af), tf32_rna((Af - tf32_rna(Af)).astype(np.float32))
            dH, dL = torch.from_numpy(H).cuda(), torch.from_numpy(L).cuda()
            Cz = torch.zeros(nbk, nbk, device="cuda")
            if nbk % 256:
                continue
            assert lib.mp_test_tc_gemm(1, p(dH), p(dL), p(Cz), nbk, 2, 1, 0) == 0
            got = -Cz.cpu().numpy().astype(np.float64)
            Ad = Af.astype(np.float64)
            ex = Ad[nbk:] @ Ad[:nbk].T
            sg = (Af[nbk:] @ Af[:nbk].T).astype(np.float64)
            print(f"K={nbk}: 3xTF32 rel.err {np.linalg.norm(got-ex)/np.linalg.norm(ex):.3e}  "
                  f"SGEMM {np.linalg.norm(sg-ex)/np.linalg.norm(ex):.3e}")
    torch.cuda.synchronize()


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else "all")
