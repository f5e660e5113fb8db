set -x
timeout 120 python tests/debug_dense.py > gpurun_out/r1_debug_dense.log 2>&1
timeout 300 python -m pytest tests/test_gpu_parity.py -q -x > gpurun_out/r1_gpu_tests.log 2>&1
for th in 0.01 0.02 0.04; do timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --theta $th > gpurun_out/r1_b_th$th.json 2>/dev/null; done
timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/r1_b_auto.json 2> gpurun_out/r1_b_auto.err
for gv in 16,2 8,4 32,1; do PCGCN_SPARSE_GV=$gv timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --theta 0.04 > gpurun_out/r1_b_gv$gv.json 2>/dev/null; done
