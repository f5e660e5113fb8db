#!/bin/bash
# round 2, call D: bf16x3 full mode + halo epochs + the rest of the new GPU tests; bench with bf16x3
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "bf3 and (aggregation and cliques)" > gpurun_out/r2d_bf3_first.log 2>&1
echo "rc=$?" >> gpurun_out/r2d_bf3_first.log
timeout 1500 python -m pytest tests -m gpu -q --durations=15 --deselect tests/test_gpu_scale.py::test_c3_bench_epoch_all_rows \
   -k "partial_warp or rmat or epoch_parity or dist or hybrid_tile or knobs or calibrate or integer_exact or bf3 or long_accumulation" > gpurun_out/r2d_pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r2d_pytest.log
timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e --dense bf16x3 > gpurun_out/r2d_bench_bf3.json 2> gpurun_out/r2d_bench_bf3.err
