#!/bin/bash
# A/B timing of library variants on the bench workload (one GPU).
for lib in "" tools/variants/*.so; do
  echo "== ${lib:-default}"
  MSCCL_LIB=$lib timeout 300 python bench.py --no-cpu --no-e2e --steps 10 --warmup 3 "$@" | python -c "import json,sys; d=json.loads(sys.stdin.readlines()[-1]); print(d['value'], d['ms_per_step'], d['parity'])"
done
