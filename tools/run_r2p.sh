timeout 900 python -m pytest tests/test_gpu_nvls.py -x -q > gpurun_out/nvls_r2p.log 2>&1; tail -2 gpurun_out/nvls_r2p.log
timeout 900 python tools/ab.py "nvls32|--program nvls --instances 32" "nvls36|--program nvls --instances 36" "ring|" --reps 2 > gpurun_out/ab_r2p.log 2>&1; grep SUMMARY gpurun_out/ab_r2p.log
