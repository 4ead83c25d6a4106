import ctypes as C, sys, os
sys.path.insert(0, os.getcwd())
import numpy as np, torch
from paper_conf_cluster_caoalgkb23_b200._lib import lib
def dev(a): return torch.from_numpy(np.ascontiguousarray(a)).cuda()
def run(P, Cm, nb, nt, m, n, nmod, lower=0):
    dP, dC = dev(P), dev(Cm)
    st = lib.mp_test_crt_gemm(C.c_void_p(dP.data_ptr()), C.c_void_p(dC.data_ptr()), nb, nt, m, n, nmod, lower)
    return st, dC.cpu().numpy()
nb, nt = 512, 2
rng = np.random.default_rng(0)
for nmod in (16, 4, 2):
    P = rng.integers(-7, 8, (nt*nb, nb)).astype(np.float64)
    P[:, 0] = 7.0
    Cm = np.zeros((nb, nb))
    st, got = run(P, Cm, nb, nt, 1, 0, nmod)
    ref = -(P[nb:] @ P[:nb].T)
    d = got - ref
    bad = np.abs(d) > 1e-6
    print("nmod", nmod, "status", st, "bad frac", bad.mean(), "max", np.abs(d).max())
    if bad.any():
        rows = np.where(bad.any(1))[0]; cols = np.where(bad.any(0))[0]
        print(" bad rows", rows[:10], len(rows), " bad cols", cols[:10], len(cols))
        i, j = np.argwhere(bad)[0]
        print(" first", i, j, got[i, j], ref[i, j])
        # does got match some permutation of rows?
        for di in (1, 2, 4, 8, 16, 32, 64, 128, 256):
            if np.allclose(got[:nb-di], ref[di:]) or np.allclose(got[di:], ref[:nb-di]):
                print(" row shift", di)
        for dj in (1, 2, 4, 8, 16, 32, 64, 128, 256):
            if np.allclose(got[:, :nb-dj], ref[:, dj:]) or np.allclose(got[:, dj:], ref[:, :nb-dj]):
                print(" col shift", dj)
        print(" got[0,:8]", got[0, :8]); print(" ref[0,:8]", ref[0, :8])
        print(" ratio sample", (got[:4,:4] / ref[:4,:4]))
