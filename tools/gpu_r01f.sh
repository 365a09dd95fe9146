# round-1 GPU batch f: L2 prefetch-from-KQ A/B, full-size tests
B="python bench.py --no-cpu-baseline --no-e2e"
timeout 300 $B > gpurun_out/f_cfg2_pf0.json 2>/dev/null
for m in 2 3; do
  FLECHE_PREFETCH_MODE=$m timeout 300 $B > gpurun_out/f_cfg2_pf$m.json 2>/dev/null
done
FLECHE_PREFETCH_MODE=2 timeout 300 $B --config cfg5 --steps 300 > gpurun_out/f_cfg5_pf2.json 2>/dev/null
timeout 900 python -m pytest tests/test_gpu_fullsize.py tests/test_gpu_parity.py -x -q 2>&1 | tail -5 > gpurun_out/pytest_f.log
cat gpurun_out/pytest_f.log
