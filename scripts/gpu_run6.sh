timeout 500 python -m pytest tests/test_gpu_parity.py -q -x > gpurun_out/r1_gpu_tests.log 2>&1
for th in 0.03 0.04 auto; do timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --theta $th > gpurun_out/r1_g_th$th.json 2>/dev/null; done
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:sparse_agg --csv --log-file gpurun_out/r1_sparse_dram2.csv python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-e2e --eager --theta 0.04 > /dev/null 2>&1
