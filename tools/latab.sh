for i in 1 2 3; do for lib in "" tools/variants/v9.so; do
  echo "== ${lib:-new}"; MSCCL_LIB=$lib timeout 300 python bench.py --no-cpu --no-e2e --steps 5 --warmup 3 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.readlines()[-1]); e=d['extras']['allreduce_1KiB_fp16_latency_us']; print(d['value'], e['oneshot_LL'], e['allpairs_LL'], e['ring_LL'])"
done; done
