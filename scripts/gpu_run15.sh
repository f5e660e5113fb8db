timeout 1200 python -m pytest tests/test_gpu_scale.py -q -x > gpurun_out/gpu_scale.log 2>&1
timeout 2400 python bench.py --workload sbm4m --steps 5 --warmup 3 --no-cpu-baseline --sweep 2,0.05,0.03,0.02,0.01,0.005,0.002 > gpurun_out/c4.json 2> gpurun_out/c4.err
