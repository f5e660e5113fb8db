# session 4, call K: bf16x3 parts stacked along N (one MMA per K-step for F <= 64): full-mode parity, C3 A/B
set -x
timeout 1500 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "aggregation_parity or integer_exact or long_accumulation or closed_forms or fused or epoch_parity or rmat" > gpurun_out/s4k_pytest.log 2>&1
timeout 1500 python -m pytest tests/test_gpu_scale.py -m gpu -q -x -k "c3_bench_epoch_all_rows and bf3" > gpurun_out/s4k_pytest_scale.log 2>&1
B3="python bench.py --no-cpu-baseline --no-e2e --steps 30 --warmup 5 --theta 0.0315 --theta-c 0.045"
for rep in 1 2; do
  timeout 600 $B3 > gpurun_out/s4k_stack_$rep.json 2> gpurun_out/s4k.err
  PCGCN_TC_STACK=0 timeout 600 $B3 > gpurun_out/s4k_nostack_$rep.json 2> /dev/null
done
