#!/bin/bash
# round 2, call M: C3 partition count sweep with the default plan options
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
for P in 41 64 256; do
  timeout 900 python bench.py --P $P --steps 20 --warmup 5 --no-cpu-baseline --no-e2e > gpurun_out/r2m_P$P.json 2> gpurun_out/r2m_P$P.err
done
