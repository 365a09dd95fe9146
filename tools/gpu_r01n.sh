timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "km_wide or address_ordered" 2>&1 | tail -3 > gpurun_out/pytest_n.log
B="python bench.py --no-cpu-baseline --no-e2e"
for i in 1 2; do
  FLECHE_KM_WIDE=1 timeout 200 $B > gpurun_out/n_wide_$i.json 2>/dev/null
  timeout 200 $B > gpurun_out/n_base_$i.json 2>/dev/null
done
FLECHE_KM_WIDE=1 timeout 300 $B --config cfg5 --steps 300 > gpurun_out/n_cfg5_wide.json 2>/dev/null
cat gpurun_out/pytest_n.log
