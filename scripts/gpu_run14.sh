timeout 600 python -m pytest tests/test_gpu_parity.py -q -x > gpurun_out/gpu_tests.log 2>&1
timeout 900 python -m pytest tests/test_gpu_scale.py -q -x > gpurun_out/gpu_scale.log 2>&1
timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/o_auto.json 2> gpurun_out/o_auto.err
