# sparse kernel v2: parity suite, then bench (fixed theta for A/B vs v1, and default)
set -x
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_v2.log 2>&1
timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --theta 0.028 > gpurun_out/bench_v2_t028.json 2> gpurun_out/bench_v2_t028.err
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/bench_v2.json 2> gpurun_out/bench_v2.err
