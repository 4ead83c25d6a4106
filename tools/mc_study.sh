#!/bin/bash
# Monte-Carlo theta-recovery study: n = 40,000, 20 replicas per setting, MP map
# for every replica, FP64 map for the first 3 (MP-vs-FP64 comparison), COBYQA from the lower bounds
# (reading C19), maxfev 200; beta in {0.03, 0.3} x nu in {0.5, 1}.  Output: gpurun_out/montecarlo_*.json
#   tools/mc_study.sh [betas] [nus] [replicas] [fp64_replicas] [maxfev]   e.g. tools/mc_study.sh "0.03" "0.5 1.0" 10 2 1000
# (maxfev 200 stops COBYQA before convergence on the sigma^2-beta ridge: C3 needed 287 / 505 evaluations)
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
for b in ${1:-0.03 0.3}; do
  for nu in ${2:-0.5 1.0}; do
    timeout ${MC_TIMEOUT:-3000} python tools/montecarlo.py 40000 ${3:-20} 1e-9 $b $nu ${4:-3} ${5:-200} > gpurun_out/mc_b${b}_nu${nu}_f${5:-200}.log 2>&1
    echo "beta=$b nu=$nu rc=$? $(tail -c 400 gpurun_out/mc_b${b}_nu${nu}_f${5:-200}.log | tr '\n' ' ' | cut -c1-300)"
  done
done
