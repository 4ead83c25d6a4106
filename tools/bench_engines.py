"""Isolated CRT engine timing (mp_bench_fp64_engine): batched nb = 2048 tile-GEMMs with 16 (FP64 class)
or 8 moduli; prints FP64-equivalent TFLOP/s of the GEMM launch and the split cost."""
import ctypes as C
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_cluster_caoalgkb23_b200._lib import lib  # noqa: E402


def run(nb=2048, nt=8, njobs=64, nmod=16, reps=5):
    ms = (C.c_float * 2)()
    st = lib.mp_bench_fp64_engine(nb, nt, njobs, nmod, reps, ms)
    assert st == 0, st
    tf = njobs * 2 * nb**3 / (ms[1] * 1e-3) / 1e12
    print(f"crt nmod {nmod:2d} njobs {njobs:4d}: gemm {ms[1]:8.3f} ms = {tf:6.1f} TFLOP/s FP64-equiv "
          f"({ms[1] / njobs * 1e3:.1f} us/tile-GEMM); split {ms[0] / nt * 1e3:.1f} us/tile", flush=True)
    return tf


if __name__ == "__main__":
    import torch
    torch.cuda.init()
    for nm in [int(a) for a in sys.argv[1:]] or [16, 8]:
        for nj in (16, 64, 148):
            run(njobs=nj, nmod=nm)
