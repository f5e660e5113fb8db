# Focused ncu capture of the selective gather (both widths) on the C3 plan, with source counters.
set -x
B="python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-e2e --eager --theta 0.028"
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"sparse_agg" -s 0 -c 2 -o gpurun_out/sp_full $B > gpurun_out/ncu_sp.log 2>&1
nvidia-smi --query-gpu=memory.total --format=csv > gpurun_out/box_info.txt; free -g >> gpurun_out/box_info.txt; nproc >> gpurun_out/box_info.txt
