# staged GEMM epilogue + in-kernel B conversion for xtg: parity, then C3/C5 epoch A/B (PCGCN_XTG_PRESPLIT)
set -x
export PCGCN_GRAPH_CACHE=/tmp/pcgcn_graphs
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_dist.py -x -q > gpurun_out/s3g_pytest.log 2>&1
timeout 900 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e --theta 0.05 > gpurun_out/s3g_c3.json 2> gpurun_out/s3g_c3.err
PCGCN_XTG_PRESPLIT=1 timeout 900 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e --theta 0.05 > gpurun_out/s3g_c3_pre.json 2> gpurun_out/s3g_c3_pre.err
timeout 1500 python bench.py --workload pl32m --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --theta 0.0693 > gpurun_out/s3g_c5.json 2> gpurun_out/s3g_c5.err
