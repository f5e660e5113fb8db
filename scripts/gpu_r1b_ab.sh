# GEMM a11 changes (dwt on the engine, balanced xtg slices): parity; then sparse knob A/B on C3
set -x
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "gemms or epoch or long_rows or graph" > gpurun_out/pytest_ab.log 2>&1
B="timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --theta 0.04"
for i in 1 2; do
$B > gpurun_out/ab_base_$i.json 2>/dev/null
PCGCN_IDX_EF=1 $B > gpurun_out/ab_ef_$i.json 2>/dev/null
PCGCN_SPARSE_FSPLIT=64 $B > gpurun_out/ab_fs64_$i.json 2>/dev/null
PCGCN_SPARSE_FSPLIT=64 PCGCN_IDX_EF=1 $B > gpurun_out/ab_fs64ef_$i.json 2>/dev/null
done
# C5 partition locality vs LP sweeps (host only), then ncu of the C5 selective passes
timeout 1500 python scripts/c5_locality.py > gpurun_out/c5_locality.log 2>&1
timeout 1800 ncu --set full --clock-control none -k regex:"sparse_(row|seg)" -s 0 -c 4 -o gpurun_out/c5_sp python bench.py --workload pl32m --steps 1 --warmup 0 --no-cpu-baseline --no-e2e --eager > gpurun_out/ncu_c5.log 2>&1
