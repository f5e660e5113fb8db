#!/bin/bash
# round 2, call F: ncu of the full-mode engine (default config), C5 bench (P = 16384 and 4096)
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 1200 ncu --profile-from-start off --set full --clock-control none --import-source on --kernel-name-base demangled \
  -k regex:"tc_engine_kernel<0" -c 2 -o gpurun_out/r2f_engine python scripts/profile_epoch.py --theta 0.04 --theta-c 0.08 > gpurun_out/r2f_ncu.log 2>&1
export PCGCN_GRAPH_CACHE=/tmp/pcgcn_graphs
timeout 2400 python bench.py --workload pl32m --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/r2f_c5.json 2> gpurun_out/r2f_c5.err
timeout 2400 python bench.py --workload pl32m --P 4096 --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/r2f_c5_p4096.json 2> gpurun_out/r2f_c5_p4096.err
