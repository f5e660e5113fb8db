# session 4, call I: warp-wide MMA issue (elected lane, no per-MMA elect loop): full-mode / GEMM parity tests,
# C3 at the fixed theta of call H, bf16x1
set -x
timeout 1500 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "aggregation_parity or integer_exact or long_accumulation or closed_forms or fused or epoch_parity or gemms or knobs or dense_pair" > gpurun_out/s4i_pytest.log 2>&1
B3="python bench.py --no-cpu-baseline --no-e2e --steps 30 --warmup 5 --theta 0.0326 --theta-c 0.045"
for rep in 1 2; do timeout 600 $B3 > gpurun_out/s4i_c3_$rep.json 2> gpurun_out/s4i_c3.err; done
timeout 600 python bench.py --no-cpu-baseline --no-e2e --steps 30 --warmup 5 --dense bf16x1 --theta 0.026 --theta-c 0.045 > gpurun_out/s4i_bf1.json 2> /dev/null
