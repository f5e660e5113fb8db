# session-3 verification of HEAD: full GPU test suite, smoke, default bench, reference arm, launch list
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/s3_gpu.txt
timeout 2400 python -m pytest tests/ -m gpu -x -q --durations=25 > gpurun_out/s3_pytest.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/s3_smoke.log 2>&1
timeout 900 python bench.py > gpurun_out/s3_bench.json 2> gpurun_out/s3_bench.err
timeout 900 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/s3_ref.json 2> gpurun_out/s3_ref.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/s3_launches.csv python bench.py --steps 2 --warmup 1 --eager --no-cpu-baseline --no-e2e > gpurun_out/s3_ncu_bench.log 2>&1
