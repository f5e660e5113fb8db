timeout 600 python -m pytest tests/test_gpu_parity.py -q -x > gpurun_out/gpu_tests.log 2>&1
timeout 900 python -m pytest tests/test_gpu_scale.py -q -x > gpurun_out/gpu_scale.log 2>&1
for pm in 0 1; do PCGCN_DENSE_PAIR=$pm timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --sweep 2,0.04,0.028,0.02,0.014,0.01 > gpurun_out/pair$pm.json 2> gpurun_out/pair$pm.err; done
