import ctypes as C, os, sys
sys.path.insert(0, os.getcwd())
import torch
from paper_conf_cluster_caoalgkb23_b200._lib import lib
torch.cuda.init()
ms = (C.c_float * 2)()
eng = int(sys.argv[1]) if len(sys.argv) > 1 else 16
assert lib.mp_bench_fp64_engine(eng, 2048, 8, 32, 16, 1, ms) == 0
print(ms[0], ms[1])
