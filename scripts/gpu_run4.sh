timeout 400 python -m pytest tests/test_gpu_parity.py tests/test_dist.py -q -x > gpurun_out/r1_gpu_tests.log 2>&1
for th in 0.02 0.04; do timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --theta $th > gpurun_out/r1_e_th$th.json 2>/dev/null; done
timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --theta 2.0 > gpurun_out/r1_e_sparse.json 2>/dev/null
