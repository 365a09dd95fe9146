# round-1 GPU batch: new tests, host-assist split sweep, watermark bench
timeout 600 python -m pytest tests/test_gpu_watermark.py tests/test_gpu_host_assist.py -x -q 2>&1 | tail -15 > gpurun_out/pytest_c.log
B="python bench.py --no-cpu-baseline --no-e2e"
for f in 0.25 0.5 0.75; do
  timeout 300 $B --config cfg5 --steps 300 --host-assist --ha-frac $f > gpurun_out/c_cfg5_ha$f.json 2>/dev/null
  timeout 300 $B --config cfg2 --host-assist --ha-frac $f > gpurun_out/c_cfg2_ha$f.json 2>/dev/null
done
timeout 300 $B --config cfg2 --watermarks 0.95,0.9 > gpurun_out/c_cfg2_wm95_90.json 2>/dev/null
timeout 300 $B --config cfg2 --watermarks 0.9,0.8 > gpurun_out/c_cfg2_wm90_80.json 2>/dev/null
timeout 300 $B --config cfg2 > gpurun_out/c_cfg2_default.json 2>/dev/null
cat gpurun_out/pytest_c.log
