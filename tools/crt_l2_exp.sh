#!/bin/bash
# A/B of the CRT operand L2 eviction hint (crt.cu CRT_L2HINT = 0 / 1 / 2): C3 evaluation rate and the DRAM
# bytes of one mid-evaluation CRT-16 launch; rebuilds the default library at the end.
cd "$(dirname "$0")/.."
for v in 0 1 2; do
  (cd paper_conf_cluster_caoalgkb23_b200 && make clean >/dev/null && make -j16 EXTRA=-DCRT_L2HINT=$v >/dev/null 2>&1)
  timeout 900 python bench.py --config c3 --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --no-profile \
    > gpurun_out/crt_l2_$v.json 2>/dev/null
  timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct \
    --clock-control none --kernel-name-base demangled -k 'regex:crt_gemm_kernel<\(int\)16' -s 11 -c 1 --csv python tools/one_eval.py c3 0 \
    > gpurun_out/crt_l2_ncu_$v.csv 2>/dev/null
  echo "L2HINT=$v $(python -c "import json; d=json.load(open('gpurun_out/crt_l2_$v.json')); print(round(d['value'],1), 'Tflop/s', d['clocks']['sm_mhz'], 'MHz')") $(grep -E 'dram__bytes|gpu__time|hit_rate' gpurun_out/crt_l2_ncu_$v.csv | awk -F'","' '{print $(NF-2), $(NF-1), $NF}' | tr '\n' ' ')"
done
(cd paper_conf_cluster_caoalgkb23_b200 && make clean >/dev/null && make -j16 >/dev/null 2>&1)
