#!/bin/bash
# Monte-Carlo theta-recovery study: n = 40,000, 20 replicas per setting, MP map
# for every replica, FP64 map for the first 3 (MP-vs-FP64 comparison), COBYQA from the lower bounds
# (reading C19), maxfev 200; beta in {0.03, 0.3} x nu in {0.5, 1}.  Output: gpurun_out/montecarlo_*.json
#   tools/mc_study.sh [betas] [nus]     e.g. tools/mc_study.sh "0.03" "0.5 1.0"
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
for b in ${1:-0.03 0.3}; do
  for nu in ${2:-0.5 1.0}; do
    timeout 2400 python tools/montecarlo.py 40000 20 1e-9 $b $nu 3 200 > gpurun_out/mc_b${b}_nu${nu}.log 2>&1
    echo "beta=$b nu=$nu rc=$? $(tail -c 400 gpurun_out/mc_b${b}_nu${nu}.log | tr '\n' ' ' | cut -c1-300)"
  done
done
