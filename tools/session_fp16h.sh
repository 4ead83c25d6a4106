#!/bin/bash
# One GPU session: TMEM F16-accumulator layout probe, ALU/DMMA-vs-tcgen05 contention, the pure-FP16 /
# four-level tests, the FP16_32 epsilon experiment and a C3 A/B of the persistent 3xFP16 kernel.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o /tmp/tp tools/dbg/tmem_f16acc.cu && timeout 60 /tmp/tp > gpurun_out/tmem_f16acc.txt 2>&1
cat gpurun_out/tmem_f16acc.txt
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/mc tools/dbg/mma_contention.cu && timeout 300 /tmp/mc > gpurun_out/mma_contention2.txt 2>&1
grep -E "DMMA|DFMA" gpurun_out/mma_contention2.txt
timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_parity.py -q -x -k "pure_fp16 or four_level" -s > gpurun_out/t_fp16h.log 2>&1
grep -E "scale|beta|passed|failed|Error|assert" gpurun_out/t_fp16h.log | head -20
timeout 900 python tools/fp16_eps.py 40000 24 > gpurun_out/fp16_eps.log 2>&1; tail -1 gpurun_out/fp16_eps.log | cut -c1-400
for e in "" "f16x3_persistent=1"; do
  timeout 900 python bench.py --config c3 --steps 2 --warmup 3 --no-cpu-baseline --no-e2e ${e:+--engine $e} > gpurun_out/c3_p$e.json 2>/dev/null
  echo "[$e] $(python -c "import json; d=json.load(open('gpurun_out/c3_p$e.json')); print(round(d['value'],1), d['clocks']['sm_mhz'], round(d['roofline']['frac'],3), {k: round(v['ms']) for k, v in d['profile'].items() if isinstance(v, dict)})")"
done
