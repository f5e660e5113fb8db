# round-end style run: tests, smoke, bench (default), launch list, ncu full on the top kernels
timeout 600 python -m pytest tests -m gpu -q > gpurun_out/r1_gpu_tests.log 2>&1
timeout 120 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r1_smoke.log 2>&1
timeout 900 python bench.py > gpurun_out/r1_bench_full.json 2> gpurun_out/r1_bench_full.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/r1_bench_ref.json 2> gpurun_out/r1_bench_ref.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r1_launch_list.csv python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-e2e --eager --theta 0.04 > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"sparse_agg|tc_engine" -s 0 -c 6 -o gpurun_out/r1_full python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-e2e --eager --theta 0.04 > /dev/null 2>&1
