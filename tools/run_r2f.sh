timeout 1500 python -m pytest tests/test_gpu_nvls.py -x -q > gpurun_out/nvls_r2f.log 2>&1; tail -3 gpurun_out/nvls_r2f.log
timeout 1500 python -m pytest tests/test_gpu_multiprocess.py -x -q > gpurun_out/mp_r2f.log 2>&1; tail -3 gpurun_out/mp_r2f.log
timeout 1200 python tools/ab.py "ag|--program allgather" "ag_s384|--program allgather --slot-kib 384" "ag_s192|--program allgather --slot-kib 192" "ar|" "a2a|--program alltoall --instances 2" "nvls_dummy|--program allgather --instances 16" --reps 2 > gpurun_out/ab_r2f.log 2>&1; grep SUMMARY gpurun_out/ab_r2f.log
