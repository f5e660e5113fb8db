timeout 900 python -m pytest tests/test_gpu_scale.py -q -x > gpurun_out/gpu_scale.log 2>&1
