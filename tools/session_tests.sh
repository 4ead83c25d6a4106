#!/bin/bash
# GPU tests + smoke + 2-rank bench (shared device) — the quick half of the round-end evidence.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_final.log 2>&1; tail -2 gpurun_out/smoke_final.log
timeout 1500 python -m pytest tests -m gpu -q --durations=10 > gpurun_out/pytest_gpu_final.log 2>&1; grep -E "passed|failed|FAILED|Error" gpurun_out/pytest_gpu_final.log | tail -8
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 \
  bench.py --gpus 2 --config c0 --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/bench_2rank_c0.json 2> gpurun_out/bench_2rank_c0.err
python -c "import json; d=json.load(open('gpurun_out/bench_2rank_c0.json')); print('2-rank c0:', d['value'], d.get('grid'), [r['ms_per_step'] for r in d.get('per_rank', [])])" || tail -5 gpurun_out/bench_2rank_c0.err
