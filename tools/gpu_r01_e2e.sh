# fleche_query_host pipelining fix: GPU suite, default bench twice (e2e), D2H probe, KQ source capture
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/e_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/e_pytest.log
tail -3 gpurun_out/e_pytest.log
for r in 1 2; do timeout 400 python bench.py > gpurun_out/e_default_$r.json 2> gpurun_out/e_default_$r.err
python -c "import json,sys; d=json.load(open(sys.argv[1])); print(sys.argv[1], round(d['value']), 'e2e', round(d['e2e']['value'],1))" gpurun_out/e_default_$r.json; done
timeout 400 ncu --metrics gpu__time_duration.sum --clock-control none -s 1200 -c 80 --csv --log-file gpurun_out/e_launches.csv python bench.py --steps 30 --no-cpu-baseline --no-e2e > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"kq_kernel" -s 320 -c 1 -o gpurun_out/ncu_kq_src python bench.py --steps 5 --no-cpu-baseline --no-e2e > gpurun_out/ncu_kq_src.log 2>&1
ncu -i gpurun_out/ncu_kq_src.ncu-rep --page source --csv --print-source sass > gpurun_out/kq_src_sass.csv 2>&1
ncu -i gpurun_out/ncu_kq_src.ncu-rep --page raw --csv > gpurun_out/kq_raw.csv 2>&1
ls -la gpurun_out | head -30
