# round-1 closing check at HEAD: GPU suite, smoke, default bench line (e2e overlapped by default)
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/f2_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/f2_pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/f2_smoke.log 2>&1
timeout 400 python bench.py > gpurun_out/f2_default.json 2> gpurun_out/f2_default.err
timeout 300 python bench.py --config cfg5 --steps 300 --no-cpu-baseline > gpurun_out/f2_cfg5.json 2>/dev/null
tail -2 gpurun_out/f2_pytest.log; tail -1 gpurun_out/f2_smoke.log
for f in gpurun_out/f2_default.json gpurun_out/f2_cfg5.json; do python -c "import json,sys; d=json.load(open(sys.argv[1])); print(sys.argv[1], round(d['value']), 'e2e', round(d['e2e']['value'],1), 'frac', round(d['roofline']['frac'],3))" $f; done
