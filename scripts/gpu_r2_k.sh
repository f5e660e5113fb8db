#!/bin/bash
# round 2, call K (final measurements): C3 bench line (default config, e2e, cpu baseline), reference arm,
# ncu launch list + --set full of the default configuration, C4 bench + launch list, C5 bench
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 1200 python bench.py > gpurun_out/r2k_bench.json 2> gpurun_out/r2k_bench.err
TH=$(python -c "import json;print(json.load(open('gpurun_out/r2k_bench.json'))['config']['theta'])")
THC=$(python -c "import json;print(json.load(open('gpurun_out/r2k_bench.json'))['config']['theta_c'])")
timeout 900 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/r2k_ref.json 2> gpurun_out/r2k_ref.err
timeout 600 ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/r2k_launches.csv python scripts/profile_epoch.py --theta $TH --theta-c $THC > gpurun_out/r2k_prof.json 2>&1
timeout 1500 ncu --profile-from-start off --set full --clock-control none --import-source on \
  -k regex:"sparse_row|sparse_seg|tc_engine_kernel" -c 14 -o gpurun_out/r2k_full python scripts/profile_epoch.py --theta $TH --theta-c $THC > gpurun_out/r2k_ncu.log 2>&1
export PCGCN_GRAPH_CACHE=/tmp/pcgcn_graphs
timeout 1800 python bench.py --workload sbm4m --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/r2k_c4.json 2> gpurun_out/r2k_c4.err
TH4=$(python -c "import json;print(json.load(open('gpurun_out/r2k_c4.json'))['config']['theta'])")
timeout 900 ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/r2k_c4_launches.csv python scripts/profile_epoch.py --workload sbm4m --theta $TH4 --order id --grain block > gpurun_out/r2k_c4_prof.json 2>&1
timeout 2400 python bench.py --workload pl32m --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/r2k_c5.json 2> gpurun_out/r2k_c5.err
timeout 1200 python bench.py --table3 --order id --grain block --dense tf32x2 --steps 20 --warmup 5 > gpurun_out/r2k_table3_block.json 2> gpurun_out/r2k_table3_block.err
timeout 1200 python bench.py --workload pubmed --f3 200 --f3-signal 0.011 --f3-seeds 3 > gpurun_out/r2k_f3_pubmed.json 2> gpurun_out/r2k_f3_pubmed.err
