"""Isolated INT8 engine timing (mp_bench_fp64_engine): 8-slice splitting vs CRT, batched
nb = 2048 tile-GEMMs; prints FP64-equivalent TFLOP/s of the GEMM launch and the split cost."""
import ctypes as C
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_cluster_caoalgkb23_b200._lib import lib  # noqa: E402


def run(engine, nb=2048, nt=8, njobs=64, nmod=16, reps=5):
    ms = (C.c_float * 2)()
    st = lib.mp_bench_fp64_engine(engine, nb, nt, njobs, nmod, reps, ms)
    assert st == 0, st
    tf = njobs * 2 * nb**3 / (ms[1] * 1e-3) / 1e12
    print(f"engine {engine:2d} nmod {nmod:2d} njobs {njobs:4d}: gemm {ms[1]:8.3f} ms = {tf:6.1f} TFLOP/s FP64-equiv "
          f"({ms[1] / njobs * 1e3:.1f} us/tile-GEMM); split {ms[0] / nt * 1e3:.1f} us/tile", flush=True)
    return tf


if __name__ == "__main__":
    import torch
    torch.cuda.init()
    args = sys.argv[1:] or ["8", "16", "16/8"]  # "16/8": CRT with 8 moduli (the FP32-class instantiation)
    for a in args:
        eng, _, nm = a.partition("/")
        for nj in (16, 64, 148):
            run(int(eng), njobs=nj, nmod=int(nm) if nm else 16)
