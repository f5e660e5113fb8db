# ncu of the v2 selective gather (segment + row passes, both widths) and the epoch launch list
set -x
B="python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-e2e --eager --theta 0.04"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launch_list_v2.csv $B > /dev/null 2>&1
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"sparse_(row|seg)" -s 0 -c 4 -o gpurun_out/sp2_full $B > gpurun_out/ncu_sp2.log 2>&1
