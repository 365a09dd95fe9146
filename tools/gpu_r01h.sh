timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "early or graph" 2>&1 | tail -5 > gpurun_out/pytest_h.log
B="python bench.py --no-cpu-baseline --no-e2e"
FLECHE_EARLY_FETCH=1 timeout 300 $B > gpurun_out/h_cfg2_early.json 2>gpurun_out/h_cfg2_early.err
timeout 300 $B > gpurun_out/h_cfg2_base.json 2>/dev/null
FLECHE_EARLY_FETCH=1 timeout 300 $B --config cfg5 --steps 300 > gpurun_out/h_cfg5_early.json 2>/dev/null
FLECHE_EARLY_FETCH=1 timeout 300 $B --config cfg1 > gpurun_out/h_cfg1_early.json 2>/dev/null
timeout 300 $B --config cfg1 > gpurun_out/h_cfg1_base.json 2>/dev/null
cat gpurun_out/pytest_h.log
