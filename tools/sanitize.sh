#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck of one small evaluation (n = 4096, nb = 512,
# adaptive map: every default kernel, CRT-16, CRT-8 TRSM product, 3xFP16, FP16, DMMA, solve) and of the
# all-FP64 map; logs to gpurun_out/sanitizer_<tool>.log.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck initcheck; do
  timeout 1200 compute-sanitizer --tool $tool --print-limit 20 --error-exitcode 9 python tools/one_eval.py c0 1 \
    > gpurun_out/sanitizer_$tool.log 2>&1
  echo "$tool rc=$?" | tee -a gpurun_out/sanitizer_$tool.log
done
# the four-level map (pure-FP16 kernel with the F16 accumulator, hs planes)
for tool in memcheck synccheck; do
  timeout 1200 compute-sanitizer --tool $tool --print-limit 20 --error-exitcode 9 python tools/one_eval.py c0q 1 \
    > gpurun_out/sanitizer_${tool}_c0q.log 2>&1
  echo "$tool c0q rc=$?" | tee -a gpurun_out/sanitizer_${tool}_c0q.log
done
