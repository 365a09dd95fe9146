# KQ A/B: timestamp-exchange result consumed late (FL_KQ_TS_DEFER=1, libfleche_tsd.so) vs default
FLECHE_LIB=libfleche_tsd.so timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py tests/test_gpu_mixed.py -x -q 2>&1 | tail -1
B="python bench.py --no-cpu-baseline --no-e2e"
for rep in 1 2; do
for lib in libfleche.so libfleche_tsd.so; do
  for cfg in cfg2 cfg5 cfg1; do
    FLECHE_LIB=$lib timeout 300 $B --config $cfg > gpurun_out/tsd_${rep}_${lib%.so}_$cfg.json 2>/dev/null
    python -c "import json,sys; d=json.load(open(sys.argv[1])); k=d['roofline']['kernels']; print(sys.argv[1], round(d['value']), round(d['ms_per_step']*1000,1), 'kq_us', round(k['kq_kernel']['ms']*1000,1), 'km_us', round(k['km_kernel']['ms']*1000,1))" gpurun_out/tsd_${rep}_${lib%.so}_$cfg.json
  done
done
done
