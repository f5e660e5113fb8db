#!/bin/bash
# round 2, call J: fused split (smem-transposed epilogue) A/B + bitwise test
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -q -k "fused_split or gemms" > gpurun_out/r2j_pytest.log 2>&1
echo "rc=$?" >> gpurun_out/r2j_pytest.log
for fs in on off; do
  timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e --fuse-split $fs --theta 0.038 --theta-c 0.06 > gpurun_out/r2j_bench_$fs.json 2> gpurun_out/r2j_bench_$fs.err
done
