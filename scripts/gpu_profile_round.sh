# Round-end measurement: bench (calibrated theta), then ncu launch list and a --set full capture of the
# aggregation kernels on the SAME plan (theta read back from the bench line), 1 GPU.
set -x
timeout 900 python bench.py > gpurun_out/bench_final.json 2> gpurun_out/bench_final.err
TH=$(python -c "import json;print(json.load(open('gpurun_out/bench_final.json'))['config']['theta'])")
timeout 900 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launch_list.csv python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-e2e --eager --theta $TH > /dev/null 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"sparse_agg|tc_engine" -s 0 -c 8 -o gpurun_out/full python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-e2e --eager --theta $TH > /dev/null 2>&1
