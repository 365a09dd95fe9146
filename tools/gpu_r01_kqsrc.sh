# KQ source-level stall capture (cfg2 steady state) + D2H output-copy probe for the e2e bound
./tools/d2h_probe > gpurun_out/d2h_probe.jsonl 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"kq_kernel" -s 640 -c 1 -o gpurun_out/ncu_kq_src python bench.py --steps 5 --no-cpu-baseline --no-e2e > gpurun_out/ncu_kq_src.log 2>&1
ncu -i gpurun_out/ncu_kq_src.ncu-rep --page source --csv --print-source sass > gpurun_out/kq_src_sass.csv 2>&1
ncu -i gpurun_out/ncu_kq_src.ncu-rep --page source --csv > gpurun_out/kq_src_cuda.csv 2>&1
ls -la gpurun_out; cat gpurun_out/d2h_probe.jsonl
