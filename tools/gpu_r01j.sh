B="python bench.py --no-cpu-baseline --no-e2e"
for i in 1 2; do
timeout 200 $B > gpurun_out/j_base_$i.json 2>/dev/null
FLECHE_TS_FIRST=1 timeout 200 $B > gpurun_out/j_tsfirst_$i.json 2>/dev/null
done
timeout 200 $B --config cfg1 > gpurun_out/j_cfg1.json 2>/dev/null
FLECHE_TS_FIRST=1 timeout 200 $B --config cfg1 > gpurun_out/j_cfg1_tsfirst.json 2>/dev/null
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q 2>&1 | tail -3
