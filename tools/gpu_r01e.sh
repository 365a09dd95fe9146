# round-1 GPU batch e: host-assist timelines at cfg2 (experiment build), default bench at HEAD
for f in 1 0.25; do
  FLECHE_HA_FRAC=$f timeout 300 python tools/ha_timeline.py cfg2 > gpurun_out/e_ha_timeline_f$f.txt 2>&1
done
timeout 300 python tools/km_timeline.py > gpurun_out/e_km_timeline.txt 2>&1
timeout 300 python bench.py > gpurun_out/e_bench_default.json 2>/dev/null
timeout 300 python bench.py --no-cpu-baseline --no-e2e --host-assist --ha-frac 0.25 > gpurun_out/e_cfg2_ha0.25.json 2>/dev/null
timeout 300 python bench.py --no-cpu-baseline --no-e2e --config cfg5 --steps 300 > gpurun_out/e_cfg5_default.json 2>/dev/null
tail -3 gpurun_out/e_ha_timeline_f1.txt
