timeout 90 python tests/debug_dense.py > gpurun_out/pair_debug.log 2>&1; echo "debug rc=$?" >> gpurun_out/pair_debug.log
timeout 90 python tests/debug_dense2.py > gpurun_out/pair_debug2.log 2>&1; echo "debug2 rc=$?" >> gpurun_out/pair_debug2.log
