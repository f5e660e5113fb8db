#!/bin/bash
# round 2, call H: dynamic full-mode tile claiming A/B + knob tests, engine ncu, C5 bench with auto options
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "knobs" > gpurun_out/r2h_knobs.log 2>&1
echo "rc=$?" >> gpurun_out/r2h_knobs.log
timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e > gpurun_out/r2h_bench.json 2> gpurun_out/r2h_bench.err
PCGCN_TC_DYN=1 timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e > gpurun_out/r2h_bench_dyn.json 2> gpurun_out/r2h_bench_dyn.err
timeout 1200 ncu --profile-from-start off --set full --clock-control none --import-source on --kernel-name-base demangled \
  -k 'regex:tc_engine_kernel<\(int\)0' -c 2 -o gpurun_out/r2h_engine python scripts/profile_epoch.py --theta 0.04 --theta-c 0.08 > gpurun_out/r2h_ncu.log 2>&1
PCGCN_TC_DYN=1 timeout 1200 ncu --profile-from-start off --set full --clock-control none --import-source on --kernel-name-base demangled \
  -k 'regex:tc_engine_kernel<\(int\)0' -c 2 -o gpurun_out/r2h_engine_dyn python scripts/profile_epoch.py --theta 0.04 --theta-c 0.08 > gpurun_out/r2h_ncu_dyn.log 2>&1
export PCGCN_GRAPH_CACHE=/tmp/pcgcn_graphs
timeout 2400 python bench.py --workload pl32m --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/r2h_c5.json 2> gpurun_out/r2h_c5.err
