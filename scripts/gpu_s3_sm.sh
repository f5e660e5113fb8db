# 4-lanes-per-row softmax (C <= 32) + GEMM epilogue mask words in registers: parity, C3 + C5 epochs
set -x
export PCGCN_GRAPH_CACHE=/tmp/pcgcn_graphs
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/s3s_pytest.log 2>&1
timeout 900 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e > gpurun_out/s3s_c3.json 2> gpurun_out/s3s_c3.err
timeout 1500 python bench.py --workload pl32m --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/s3s_c5.json 2> gpurun_out/s3s_c5.err
