#!/bin/bash
# Sweep slot count x slot size (and the L2 persisting set-aside) on the bench workload.
for cfg in "4 256 0" "2 256 0" "3 256 0" "2 512 0" "4 512 0" "2 1024 0" "4 256 32" "4 256 64" "2 512 64"; do
  set -- $cfg
  r=$(MSCCL_WARP_FLAGS=0 MSCCL_L2_PERSIST_MIB=$3 timeout 120 python bench.py --no-cpu --no-e2e --quiet-extra --steps 10 --warmup 3 \
      --slots $1 --slot-kib $2 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'], d['parity']['mismatches'])")
  echo "slots=$1 slot_kib=$2 l2persist=$3 -> $r"
done
