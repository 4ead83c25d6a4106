#!/bin/bash
# One gpurun session of ncu evidence (B200_PROFILING.md recipe).  Usage: tools/ncu_session.sh <what...>
#   launches  — per-launch list of one C5 evaluation (gpu__time_duration, clock-control none)
#   crt       — --set full of one mid-evaluation CRT-16 launch at C5 (DRAM traffic, tensor pipe, stalls)
#   f16x3     — --set full of one 3xFP16 launch at C5
#   membound  — --set full of the HBM-bound kernels (generation, conversions, solve) at C2
# Reports land in gpurun_out/ (scratch); summaries are copied to profiles/r02 by hand.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
for what in "$@"; do
  case $what in
    launches)
      timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
        --log-file gpurun_out/ncu_launches_c5.csv python tools/one_eval.py c5 0 > gpurun_out/ncu_launches_c5.log 2>&1
      python tools/launch_summary.py gpurun_out/ncu_launches_c5.csv "one C5 evaluation (n=250k, adaptive)" \
        > gpurun_out/ncu_launches_c5_summary.md 2>&1 ;;
    crt)
      timeout 1500 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
        -k 'regex:crt_gemm_kernel<\(int\)16' -s 23 -c 1 -o gpurun_out/ncu_crt16_c5 -f \
        python tools/one_eval.py c5 0 > gpurun_out/ncu_crt16_c5.log 2>&1
      python tools/ncu_summary.py gpurun_out/ncu_crt16_c5.ncu-rep > gpurun_out/ncu_crt16_c5_summary.txt 2>&1 ;;
    f16x3)
      timeout 1500 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
        -k 'regex:tc_gemm_kernel<\(int\)2' -s 11 -c 1 -o gpurun_out/ncu_f16x3_c5 -f \
        python tools/one_eval.py c5 0 > gpurun_out/ncu_f16x3_c5.log 2>&1
      python tools/ncu_summary.py gpurun_out/ncu_f16x3_c5.ncu-rep > gpurun_out/ncu_f16x3_c5_summary.txt 2>&1 ;;
    membound)
      timeout 1500 ncu --set full --clock-control none --kernel-name-base demangled \
        -k 'regex:matern|crt_split|split16|panel_in|panel_out|gemv_sub|trsv|logdiag' -c 16 \
        -o gpurun_out/ncu_membound_c2 -f python tools/one_eval.py c2a 0 > gpurun_out/ncu_membound_c2.log 2>&1
      python tools/ncu_summary.py gpurun_out/ncu_membound_c2.ncu-rep > gpurun_out/ncu_membound_c2_summary.txt 2>&1 ;;
  esac
done
