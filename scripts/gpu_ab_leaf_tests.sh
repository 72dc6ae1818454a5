bash scripts/gpu_ableaf.sh
timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_factor_device.py tests/test_gpu_dist.py -q -x 2>&1 | tail -3
