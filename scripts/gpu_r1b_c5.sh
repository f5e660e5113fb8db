# C5 (clustered power-law, 33.5M vertices, 1.03B nnz) bench on 1 GPU, then the full-size sampled parity test
set -x
free -g > gpurun_out/c5_mem.txt
timeout 1800 python bench.py --workload pl32m --steps 10 --warmup 3 > gpurun_out/bench_c5.json 2> gpurun_out/bench_c5.err
timeout 1500 python -m pytest tests/test_gpu_scale.py -m gpu -x -q -k c5 > gpurun_out/pytest_c5.log 2>&1
