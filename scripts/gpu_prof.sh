# ncu captures of the aggregation kernels on the C3 (Reddit-shaped) epoch, theta fixed
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"dense_tc|sparse_agg" -s 2 -c 4 -o gpurun_out/r1_prof2 python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-e2e --eager --theta 0.02 > gpurun_out/r1_ncu2.log 2>&1
