#!/bin/bash
# Round-end evidence on one B200: full GPU test suite, smoke, a 2-rank bench on the shared device (N > 1 path
# validation: grid + per-rank fields), and the default bench line.  Outputs in gpurun_out/.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_final.log 2>&1; tail -2 gpurun_out/smoke_final.log
timeout 1500 python -m pytest tests -m gpu -q -x --durations=10 > gpurun_out/pytest_gpu_final.log 2>&1; tail -2 gpurun_out/pytest_gpu_final.log
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 \
  bench.py --gpus 2 --config c0 --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/bench_2rank_c0.json 2> gpurun_out/bench_2rank_c0.err
python -c "import json; d=json.load(open('gpurun_out/bench_2rank_c0.json')); print('2-rank c0:', d['value'], d.get('grid'), [r['ms_per_step'] for r in d.get('per_rank', [])])"
python bench.py > gpurun_out/bench_final.json 2> gpurun_out/bench_final.err
python -c "import json; d=json.load(open('gpurun_out/bench_final.json')); print('C5:', d['value'], d['ms_per_step'], d['joules_per_eval'], d['clocks'], d['roofline']['frac'])"
