#!/bin/bash
# A/B timing of runtime parameters on the bench workload (one GPU): each argument is an
# env assignment list, e.g. tools/ab_env.sh "MSCCL_WARP_FLAGS=0" "MSCCL_WARP_FLAGS=1"
for cfg in "$@"; do
  echo "== $cfg"
  env $cfg timeout 300 python bench.py --no-cpu --no-e2e --steps 10 --warmup 3 $BENCH_ARGS | python -c "import json,sys; d=json.loads(sys.stdin.readlines()[-1]); print(d['value'], d['ms_per_step'], d['parity'], d.get('extras'))"
done
