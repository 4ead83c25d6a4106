#!/bin/bash
# ncu --set full of one isolated 148-job CRT-16 launch (tools/bench_engines.py), summary to gpurun_out/$1_summary.txt
cd "$(dirname "$0")/.."
tag=${1:-ncu_crt_iso}
ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k 'regex:crt_gemm_kernel<\(int\)16' -s 1 -c 1 \
  -o gpurun_out/$tag python -c "
import sys; sys.path.insert(0, '.')
import torch; torch.cuda.init()
from tools.bench_engines import run
run(njobs=148, nmod=16, reps=1)
" > gpurun_out/$tag.log 2>&1
python tools/ncu_summary.py gpurun_out/$tag.ncu-rep > gpurun_out/${tag}_summary.txt
