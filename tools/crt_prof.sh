#!/bin/bash
# CRT-16 epilogue cycle counters (crt.cu CRT_PROF): isolated launches of 16/64/148 nb = 2048 jobs
# (tools/bench_engines.py); rebuilds the default library at the end.  Output: gpurun_out/crt_prof*.txt
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
tag=${1:-}
(cd paper_conf_cluster_caoalgkb23_b200 && make clean >/dev/null && make -j16 EXTRA=-DCRT_PROF >/dev/null 2>&1)
timeout 600 python tools/bench_engines.py 16 > gpurun_out/crt_prof$tag.txt 2>&1
grep -E "crt nmod|recon detail" gpurun_out/crt_prof$tag.txt | head -20
(cd paper_conf_cluster_caoalgkb23_b200 && make clean >/dev/null && make -j16 >/dev/null 2>&1)
timeout 600 python tools/bench_engines.py 16 > gpurun_out/crt_noprof$tag.txt 2>&1
cat gpurun_out/crt_noprof$tag.txt
