# A/B of the full-mode || segment-pass overlap (high-priority side stream), C3 epoch; parity first
set -x
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_dist.py -x -q > gpurun_out/s3o_pytest.log 2>&1
for ov in 0 1; do
  PCGCN_OVERLAP=$ov timeout 900 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e > gpurun_out/s3o_ov$ov.json 2> gpurun_out/s3o_ov$ov.err
done
PCGCN_OVERLAP=1 PCGCN_TC_GRID=132 timeout 900 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e --theta 0.04 > gpurun_out/s3o_ov1_g132.json 2> gpurun_out/s3o_ov1_g132.err
PCGCN_OVERLAP=1 timeout 900 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e --theta 0.028 > gpurun_out/s3o_ov1_t028.json 2> gpurun_out/s3o_ov1_t028.err
timeout 300 python -c "
from paper_conf_ipps_tianmyd20_b200 import _lib as L
for rb in (512, 256, 192, 128, 64, 16):
    print(rb, {lvl: round(max(L.probe_gather_gbs(nb, rb, 256) for _ in range(3))) for lvl, nb in (('l1', 64<<10), ('l1b', 160<<10), ('l2', 64<<20), ('l2b', 100<<20), ('hbm', 4<<30))}, flush=True)
print('read', {mb: round(L.probe_read_gbs(mb<<20, 20)) for mb in (16, 64, 4096)})
" > gpurun_out/s3o_probe.log 2>&1
