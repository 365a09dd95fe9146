# closing check after FL_KQ_TS_DEFER=1 became the default: GPU suite, smoke, default bench line
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/f3_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/f3_pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/f3_smoke.log 2>&1
timeout 400 python bench.py > gpurun_out/f3_default.json 2> gpurun_out/f3_default.err
tail -2 gpurun_out/f3_pytest.log; tail -1 gpurun_out/f3_smoke.log
python -c "import json,sys; d=json.load(open(sys.argv[1])); k=d['roofline']['kernels']; print(sys.argv[1], round(d['value']), 'e2e', round(d['e2e']['value'],1), 'frac', round(d['roofline']['frac'],3), 'kq_us', round(k['kq_kernel']['ms']*1000,1))" gpurun_out/f3_default.json
