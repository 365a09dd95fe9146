# round-1 re-entry check at HEAD: GPU suite, smoke, default bench line, reference arm
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/v_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/v_pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/v_smoke.log 2>&1
timeout 400 python bench.py > gpurun_out/v_default.json 2> gpurun_out/v_default.err
timeout 400 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/v_ref.json 2> gpurun_out/v_ref.err
tail -3 gpurun_out/v_pytest.log; cat gpurun_out/v_smoke.log | tail -2; cat gpurun_out/v_default.json; cat gpurun_out/v_ref.json
