python -c "
from paper_conf_asplos_cowanmmsx23_b200 import runtime
import torch
print('devices', torch.cuda.device_count(), 'multicast supported', [runtime.nvls_supported(d) for d in range(torch.cuda.device_count())])"
timeout 900 python -m pytest tests/test_gpu_nvls.py -x -q -rs > gpurun_out/nvls_r2j.log 2>&1; tail -8 gpurun_out/nvls_r2j.log
