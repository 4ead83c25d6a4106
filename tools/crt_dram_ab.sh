#!/bin/bash
# DRAM bytes of one isolated 148-job CRT-16 launch per compile-time variant (ncu, 3 metrics only):
# tools/crt_dram_ab.sh "" "-DCRT_DISCARD=0" ...; rebuilds the default at the end.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
i=0
for v in "$@"; do
  (cd paper_conf_cluster_caoalgkb23_b200 && make clean >/dev/null && make -j16 EXTRA="$v" >/dev/null 2>&1)
  ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct \
    --clock-control none --kernel-name-base demangled -k 'regex:crt_gemm_kernel<\(int\)16' -s 1 -c 1 --csv \
    python -c "
import sys; sys.path.insert(0, '.')
import torch; torch.cuda.init()
from tools.bench_engines import run
run(njobs=148, nmod=16, reps=1)
" > gpurun_out/dram_ab_$i.csv 2>/dev/null
  echo "[$v] $(grep -E 'dram__bytes|gpu__time|hit_rate' gpurun_out/dram_ab_$i.csv | awk -F'","' '{print $(NF-2), $(NF-1), $NF}' | tr -d '"' | tr '\n' ' ')"
  i=$((i+1))
done
(cd paper_conf_cluster_caoalgkb23_b200 && make clean >/dev/null && make -j16 >/dev/null 2>&1)
