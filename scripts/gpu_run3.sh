timeout 120 python tests/debug_dense.py > gpurun_out/r1_debug_dense.log 2>&1
timeout 400 python -m pytest tests/test_gpu_parity.py -q -x > gpurun_out/r1_gpu_tests.log 2>&1
for u in 1 2 4; do PCGCN_TC_U=$u timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --theta 0.02 > gpurun_out/r1_d_u$u.json 2>/dev/null; done
for th in 0.01 0.04; do timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --theta $th > gpurun_out/r1_d_th$th.json 2>/dev/null; done
timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/r1_d_auto.json 2> gpurun_out/r1_d_auto.err
