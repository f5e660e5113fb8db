#!/bin/bash
# round 2, call C: new GPU tests (partial-warp layout, tile grain, halo epochs, knobs) + bench G6 A/B
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q --durations=15 --deselect tests/test_gpu_scale.py::test_c3_bench_epoch_all_rows \
   -k "partial_warp or rmat or epoch_parity or dist or hybrid_tile or knobs or calibrate or integer_exact" > gpurun_out/r2c_pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r2c_pytest.log
timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e > gpurun_out/r2c_bench_g6.json 2> gpurun_out/r2c_bench_g6.err
PCGCN_SPARSE_G6=0 timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e > gpurun_out/r2c_bench_nog6.json 2> gpurun_out/r2c_bench_nog6.err
