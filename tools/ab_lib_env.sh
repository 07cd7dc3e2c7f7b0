#!/bin/bash
# A/B of (library, env) pairs on the bench workload: each argument is "LIB ENV..." e.g.
#   tools/ab_lib_env.sh "default MSCCL_DIRECT_HINTS=0" "tools/variants/x.so MSCCL_DIRECT_HINTS=1"
for cfg in "$@"; do
  lib=${cfg%% *}; envs=${cfg#* }; [ "$lib" = "$cfg" ] && envs=""
  [ "$lib" = default ] && lib=""
  echo "== $cfg"
  env MSCCL_LIB=$lib $envs timeout 300 python bench.py --no-cpu --no-e2e --quiet-extra --steps 10 --warmup 3 $BENCH_ARGS | python -c "import json,sys; d=json.loads(sys.stdin.readlines()[-1]); print(d['value'], d['ms_per_step'])"
done
