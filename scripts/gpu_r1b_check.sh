# Re-entry check: GPU parity suite + default bench on the current HEAD.
set -x
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1
timeout 900 python bench.py > gpurun_out/bench_now.json 2> gpurun_out/bench_now.err
