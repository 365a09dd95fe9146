# round-1 final evidence at HEAD: default bench line, launch list, ncu --set full of KQ and KM,
# other configs' lines
timeout 400 python bench.py > gpurun_out/fin_default.json 2> gpurun_out/fin_default.err
timeout 400 ncu --metrics gpu__time_duration.sum --clock-control none -s 1200 -c 80 --csv --log-file gpurun_out/fin_launches.csv python bench.py --steps 30 --no-cpu-baseline --no-e2e > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"kq_kernel|km_kernel" -s 640 -c 2 -o gpurun_out/fin_kq_km python bench.py --steps 5 --no-cpu-baseline --no-e2e > /dev/null 2>&1
B="python bench.py --no-cpu-baseline --no-e2e"
timeout 300 $B --config cfg1 > gpurun_out/fin_cfg1.json 2>/dev/null
timeout 300 $B --config cfg5 --steps 300 > gpurun_out/fin_cfg5.json 2>/dev/null
timeout 300 $B --config cfg5 --steps 300 --host-assist --ha-frac 0.5 > gpurun_out/fin_cfg5_ha.json 2>/dev/null
timeout 400 $B --config cfg4 --steps 100 > gpurun_out/fin_cfg4.json 2>/dev/null
ls -la gpurun_out/fin_*
