# KQ occupancy A/B: probe lines in flight per lane (FL_KQ_PROBE) x CTAs per SM (FL_KQ_MIN_BLOCKS),
# same box, back to back; then parity of the variants on the quick GPU parity file
B="python bench.py --no-cpu-baseline --no-e2e"
for rep in 1 2; do
for lib in libfleche.so libfleche_p16b10.so libfleche_p8b12.so libfleche_p4b12.so libfleche_p8b16.so; do
  for cfg in cfg2 cfg5 cfg1; do
    FLECHE_LIB=$lib timeout 300 $B --config $cfg > gpurun_out/kqab_${rep}_${lib%.so}_$cfg.json 2>/dev/null
    python -c "import json,sys; d=json.load(open(sys.argv[1])); k=d['roofline']['kernels']; print(sys.argv[1], round(d['value']), round(d['ms_per_step']*1000,1), 'kq_us', round(k['kq_kernel']['ms']*1000,1), 'km_us', round(k['km_kernel']['ms']*1000,1))" gpurun_out/kqab_${rep}_${lib%.so}_$cfg.json
  done
done
done
for lib in libfleche_p8b12.so libfleche_p8b16.so; do
  FLECHE_LIB=$lib timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_mixed.py -x -q 2>&1 | tail -2
done
