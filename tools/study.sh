#!/bin/bash
# Batch of bench.py lines for the DESIGN.md studies (one gpurun session).  Each line: name + bench args.
# Output: gpurun_out/study_<name>.json (+ .err).  Usage: tools/study.sh <set>
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
run() {
  local name=$1; shift
  timeout 1500 python bench.py --no-cpu-baseline --no-e2e --steps 2 --warmup 3 "$@" \
    > gpurun_out/study_$name.json 2> gpurun_out/study_$name.err
  echo "$name rc=$? $(python -c "import json,sys; d=json.load(open('gpurun_out/study_$name.json')); print(round(d['value'],1), 'Tflop/s', round(d['ms_per_step']/1e3,2), 's', round(d['joules_per_eval'] or 0), 'J', d['loglik'], d['tiles_fp64_fp32_fp16'], 'stc', d['stc_tiles'])" 2>/dev/null)"
}
case $1 in
  conv_c5)
    run c5_auto --config c5 --policy auto
    run c5_ttc --config c5 --policy ttc
    run c5_ext_auto --config c5 --map extreme --policy auto
    run c5_ext_ttc --config c5 --map extreme --policy ttc ;;
  c2)
    for m in adaptive band fp64 extreme; do run c2_${m}_auto --config c2 --map $m --policy auto; done
    run c2_extreme_ttc --config c2 --map extreme --policy ttc
    run c2_fp64_dmma --config c2 --map fp64 --engine fp64_engine=1
    run c2b01_band --config c2 --map band --theta 1,0.1,0.5
    run c2b01_fp64 --config c2 --map fp64 --theta 1,0.1,0.5
    run c2b01_adaptive --config c2 --map adaptive --theta 1,0.1,0.5 ;;
  c3)
    run c3_adaptive --config c3
    run c3_fp64_crt --config c3 --map fp64
    run c3_fp64_dmma --config c3 --map fp64 --engine fp64_engine=1
    run c3_adaptive_dmma --config c3 --engine fp64_engine=1
    run c3_nolook --config c3 --engine lookahead=0 ;;
  r3)  # refresh after the integer CRT reconstruction (session 3) + the four-level map + reserve pairs at C5
    run c3_adaptive_v3 --config c3
    run c3_fp64_crt_v3 --config c3 --map fp64
    run c3_fp64_dmma_v3 --config c3 --map fp64 --engine fp64_engine=1
    run c3_adaptive4_v3 --config c3 --map adaptive4
    run c2_adaptive_v3 --config c2 --map adaptive
    run c2_fp64_v3 --config c2 --map fp64
    run c2_adaptive4_v3 --config c2 --map adaptive4
    run c5_rp3_v3 --config c5 --engine reserve_pairs=3
    run c5_rp9_v3 --config c5 --engine reserve_pairs=9
    python tools/mc_check.py profiles/r02/mc/montecarlo_n40000_R8_b0.03_nu1.0_f1000.json 0 > gpurun_out/mc_check.log 2>&1; tail -1 gpurun_out/mc_check.log
    bash tools/sanitize.sh ;;
  rp)  # reserve_pairs sweep at C5 on one box (CTA pairs the persistent CRT grid leaves to the panel stream)
    for r in 6 3 2 4 0; do run c5_rp${r}_sweep --config c5 --engine reserve_pairs=$r; done ;;
  sens)
    run c3_ureq1e-8 --config c3 --u-req 1e-8
    run c3_nu1 --config c3 --theta 1,0.03,1.0
    run c3_nu1_fp64 --config c3 --theta 1,0.03,1.0 --map fp64
    run c5_ureq1e-8 --config c5 --u-req 1e-8
    run c5_nu1 --config c5 --theta 1,0.03,1.0 ;;
esac
