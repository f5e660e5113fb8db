#!/bin/bash
# round 2, call B: C3 θ sweeps for vertex order x mode grain (forward aggregation times per θ)
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
export PCGCN_GRAPH_CACHE=/tmp/pcgcn_graphs
for cfg in "id block 2.0,0.028,0.04,0.056" "degree block 2.0,0.028,0.04,0.056" "degree tile 0.02,0.03,0.045,0.06,0.08,0.11,0.15,0.2" "id tile 0.03,0.06,0.1"; do
  set -- $cfg
  timeout 900 python bench.py --steps 10 --warmup 3 --order $1 --grain $2 --sweep $3 --no-cpu-baseline --no-e2e \
     > gpurun_out/r2b_${1}_${2}.json 2> gpurun_out/r2b_${1}_${2}.err
done
