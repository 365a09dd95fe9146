set -x
B="python bench.py --no-cpu-baseline --steps 1000"
for cfg in cfg2 cfg5; do
  timeout 300 $B --config $cfg > gpurun_out/ab_${cfg}_default.json 2>/dev/null
  FLECHE_FUSED_GATHER=1 timeout 300 $B --config $cfg > gpurun_out/ab_${cfg}_fused.json 2>/dev/null
  timeout 300 $B --config $cfg --host-assist > gpurun_out/ab_${cfg}_ha.json 2>/dev/null
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:km_kernel -s 320 -c 1 -o gpurun_out/ncu_km_r01b python bench.py --steps 5 --no-cpu-baseline --no-e2e > gpurun_out/ncu_km.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"kq_kernel|kg_kernel" -s 640 -c 2 -o gpurun_out/ncu_kq_r01b python bench.py --steps 5 --no-cpu-baseline --no-e2e > gpurun_out/ncu_kq.log 2>&1
ls -la gpurun_out
