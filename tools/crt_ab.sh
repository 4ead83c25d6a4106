#!/bin/bash
# A/B of CRT kernel compile-time variants: tools/crt_ab.sh "-DX=0" "-DX=1" ...  For each EXTRA: isolated
# CRT-16 launches (bench_engines) and one short C3 evaluation bench; rebuilds the default at the end.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
i=0
for v in "$@"; do
  (cd paper_conf_cluster_caoalgkb23_b200 && make clean >/dev/null && make -j16 EXTRA="$v" >/dev/null 2>&1)
  timeout 300 python -m pytest tests/test_gpu_kernels.py -q -x -k crt > gpurun_out/ab_${i}_tests.txt 2>&1
  timeout 300 python tools/bench_engines.py 16 > gpurun_out/ab_${i}_engines.txt 2>&1
  timeout 900 python bench.py --config c3 --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ab_${i}_c3.json 2>/dev/null
  echo "[$v] tests: $(tail -1 gpurun_out/ab_${i}_tests.txt | cut -c1-40) | $(grep 'njobs  148' gpurun_out/ab_${i}_engines.txt | cut -c1-80) | C3 $(python -c "import json; d=json.load(open('gpurun_out/ab_${i}_c3.json')); print(round(d['value'],1), 'Tflop/s', d['clocks']['sm_mhz'], 'MHz frac', round(d['roofline']['frac'],3), 'upd64', round(d['profile']['upd_fp64']['tflops'],1))")"
  i=$((i+1))
done
(cd paper_conf_cluster_caoalgkb23_b200 && make clean >/dev/null && make -j16 >/dev/null 2>&1)
