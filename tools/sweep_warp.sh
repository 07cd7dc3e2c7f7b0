#!/bin/bash
# Sweep warp flags x slot size x instances x threads on the bench workload (one GPU).
for w in 0 1; do for kib in 64 128 256; do for inst in 16 32; do for thr in 256 512; do
  if [ $thr = 512 ] && [ $inst = 32 ]; then continue; fi
  r=$(MSCCL_WARP_FLAGS=$w timeout 120 python bench.py --no-cpu --no-e2e --quiet-extra --steps 10 --warmup 3 \
      --slot-kib $kib --instances $inst --threads $thr 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'], d['parity']['mismatches'])")
  echo "warp=$w slot_kib=$kib inst=$inst thr=$thr -> $r"
done; done; done; done
