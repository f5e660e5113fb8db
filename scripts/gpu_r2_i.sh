#!/bin/bash
# round 2, call I: full GPU suite, C3 bench (fused split + dynamic tiles), C5-shape GEMM timings + ncu
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e > gpurun_out/r2i_bench.json 2> gpurun_out/r2i_bench.err
timeout 2400 python -m pytest tests -m gpu -q --durations=25 > gpurun_out/r2i_pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r2i_pytest.log
timeout 600 python scripts/profile_gemms.py > gpurun_out/r2i_gemms.json 2>&1
timeout 1200 ncu --profile-from-start off --set full --clock-control none --import-source on -c 12 \
  -o gpurun_out/r2i_gemms python scripts/profile_gemms.py 8388608 > gpurun_out/r2i_gemms_ncu.log 2>&1
