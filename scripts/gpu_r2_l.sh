#!/bin/bash
# round 2, call L: the whole GPU suite on the final code (incl. F4 peer tests) + smoke
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 3000 python -m pytest tests -m gpu -q --durations=10 > gpurun_out/r2l_pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r2l_pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2l_smoke.log 2>&1
echo "smoke rc=$?" >> gpurun_out/r2l_smoke.log
