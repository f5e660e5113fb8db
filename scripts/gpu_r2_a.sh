#!/bin/bash
# round 2, call A: full GPU suite (incl. the C3 bench-configuration oracle epoch) + baseline bench
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/r2a_smi.txt 2>&1
timeout 1500 python -m pytest tests/test_gpu_scale.py -x -q -s -k "c3_bench" > gpurun_out/r2a_c3epoch.log 2>&1
echo "c3 rc=$?" >> gpurun_out/r2a_c3epoch.log
timeout 1800 python -m pytest tests -m gpu -x -q --durations=20 --deselect tests/test_gpu_scale.py::test_c3_bench_epoch_all_rows > gpurun_out/r2a_pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r2a_pytest.log
timeout 600 python bench.py --steps 20 --warmup 5 > gpurun_out/r2a_bench.json 2> gpurun_out/r2a_bench.err
echo "bench rc=$?" >> gpurun_out/r2a_bench.err
