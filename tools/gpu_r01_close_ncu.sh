# ncu evidence at the round-1 close: launch list + one KQ/KM --set full capture (cfg2)
timeout 400 ncu --metrics gpu__time_duration.sum --clock-control none -s 1200 -c 80 --csv --log-file gpurun_out/close_launches.csv python bench.py --steps 30 --no-cpu-baseline --no-e2e > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"kq_kernel|km_kernel" -s 640 -c 2 -o gpurun_out/close_kq_km python bench.py --steps 5 --no-cpu-baseline --no-e2e > /dev/null 2>&1
ls -la gpurun_out
