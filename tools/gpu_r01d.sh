# round-1 GPU batch d: watermark re-test + bench, HA thread sweep, maintenance sweep
timeout 600 python -m pytest tests/test_gpu_watermark.py -x -q 2>&1 | tail -5 > gpurun_out/pytest_d.log
B="python bench.py --no-cpu-baseline --no-e2e"
timeout 300 $B --config cfg2 --watermarks 0.95,0.9 > gpurun_out/d_cfg2_wm95_90.json 2>/dev/null
for th in 8 15; do
  FLECHE_HA_THREADS=$th timeout 300 $B --config cfg5 --steps 300 --host-assist --ha-frac 0.5 > gpurun_out/d_cfg5_ha_t$th.json 2>/dev/null
done
timeout 300 $B --config cfg5 --steps 300 --host-assist --ha-frac 0.6 > gpurun_out/d_cfg5_ha0.6.json 2>/dev/null
timeout 900 python tools/maintenance_sweep.py > gpurun_out/maintenance_sweep.jsonl 2> gpurun_out/maintenance_sweep.err
nproc > gpurun_out/nproc.txt
cat gpurun_out/pytest_d.log
