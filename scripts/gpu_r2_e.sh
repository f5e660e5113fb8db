#!/bin/bash
# round 2, call E: C3 bench-config epoch parity (tile, bf16x3), tile order A/B, ncu of the new default
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_scale.py -q -s -k "c3_bench and tile" > gpurun_out/r2e_c3epoch.log 2>&1
echo "rc=$?" >> gpurun_out/r2e_c3epoch.log
timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e > gpurun_out/r2e_bench.json 2> gpurun_out/r2e_bench.err
PCGCN_TC_ORDER=plan timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e > gpurun_out/r2e_bench_plan.json 2> gpurun_out/r2e_bench_plan.err
TH=$(python -c "import json;print(json.load(open('gpurun_out/r2e_bench.json'))['config']['theta'])")
THC=$(python -c "import json;print(json.load(open('gpurun_out/r2e_bench.json'))['config']['theta_c'])")
timeout 600 ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/r2e_launches.csv python scripts/profile_epoch.py --theta $TH --theta-c $THC > gpurun_out/r2e_prof_plan.json 2>&1
timeout 1500 ncu --profile-from-start off --set full --clock-control none --import-source on \
  -k regex:"sparse_row|sparse_seg|tc_engine_kernel<0" -c 6 -o gpurun_out/r2e_full python scripts/profile_epoch.py --theta $TH --theta-c $THC > gpurun_out/r2e_ncu.log 2>&1
echo done >> gpurun_out/r2e_ncu.log
