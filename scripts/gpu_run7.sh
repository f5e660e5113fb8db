timeout 120 python tests/debug_dense.py > gpurun_out/r1_debug_dense.log 2>&1
timeout 500 python -m pytest tests/test_gpu_parity.py -q -x > gpurun_out/r1_gpu_tests.log 2>&1
for th in 0.01 0.02 0.04 auto; do timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --theta $th > gpurun_out/r1_h_th$th.json 2>/dev/null; done
timeout 600 ncu --metrics gpu__time_duration.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active --clock-control none -k regex:"tc_engine|sparse_agg" --csv --log-file gpurun_out/r1_h_list.csv python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-e2e --eager --theta 0.02 > /dev/null 2>&1
