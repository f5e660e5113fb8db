# session-4 verification of HEAD: GPU test suite, smoke, default bench line
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/s4_gpu.txt
timeout 2400 python -m pytest tests/ -m gpu -q --durations=25 > gpurun_out/s4_pytest.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/s4_smoke.log 2>&1
timeout 900 python bench.py > gpurun_out/s4_bench.json 2> gpurun_out/s4_bench.err
