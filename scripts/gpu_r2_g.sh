#!/bin/bash
# round 2, call G: C1/C2 bench lines, full oracle epochs on the host, F3 study, Table III replica,
# compute-sanitizer on tiny graphs
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
for wl in cora pubmed; do
  timeout 600 python bench.py --workload $wl --steps 50 --warmup 10 > gpurun_out/r2g_bench_$wl.json 2> gpurun_out/r2g_bench_$wl.err
done
timeout 900 python tests/oracle_epoch_time.py cora pubmed reddit > gpurun_out/r2g_oracle_epoch.json 2> gpurun_out/r2g_oracle_epoch.err
timeout 1200 python bench.py --workload pubmed --f3 200 --f3-signal 0.015 --f3-seeds 3 > gpurun_out/r2g_f3_pubmed.json 2> gpurun_out/r2g_f3_pubmed.err
timeout 1200 python bench.py --table3 --steps 20 --warmup 5 > gpurun_out/r2g_table3.json 2> gpurun_out/r2g_table3.err
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python scripts/sanitize_case.py > gpurun_out/r2g_san_$tool.log 2>&1
  echo "rc=$?" >> gpurun_out/r2g_san_$tool.log
done
