timeout 600 python -m pytest tests/test_gpu_host_assist.py -x -q 2>&1 | tail -4 > gpurun_out/pytest_l.log
B="python bench.py --no-cpu-baseline --no-e2e"
for f in 1 0.75 0.5; do
  FLECHE_HA_PUSH=1 timeout 200 $B --host-assist --ha-frac $f > gpurun_out/l_cfg2_push$f.json 2>/dev/null
done
FLECHE_HA_PUSH=1 FLECHE_HA_THREADS=15 timeout 200 $B --host-assist --ha-frac 1 > gpurun_out/l_cfg2_push1_t15.json 2>/dev/null
timeout 200 $B > gpurun_out/l_cfg2_base.json 2>/dev/null
FLECHE_HA_PUSH=1 timeout 300 $B --config cfg5 --steps 300 --host-assist --ha-frac 1 > gpurun_out/l_cfg5_push1.json 2>/dev/null
FLECHE_HA_PUSH=1 timeout 300 $B --config cfg5 --steps 300 --host-assist --ha-frac 0.6 > gpurun_out/l_cfg5_push0.6.json 2>/dev/null
cat gpurun_out/pytest_l.log
