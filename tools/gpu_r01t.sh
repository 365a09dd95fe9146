B="python bench.py --no-cpu-baseline --no-e2e"
for f in 0.7 0.85; do
  timeout 900 $B --config cfg3h --steps 200 --cache-frac 0.01 --host-assist --ha-frac $f > gpurun_out/t_cfg3h_ha$f.json 2>/dev/null
done
timeout 900 $B --config cfg3h --steps 200 --cache-frac 0.05 --host-assist > gpurun_out/t_cfg3h5_ha.json 2>/dev/null
timeout 900 $B --config cfg3h --steps 200 --cache-frac 0.05 > gpurun_out/t_cfg3h5.json 2>/dev/null
for i in 1 2; do
  for v in kq6 kq8 base; do
    if [ $v = base ]; then timeout 200 $B > gpurun_out/t_$v.$i.json 2>/dev/null; else FLECHE_LIB=libfleche_$v.so timeout 200 $B > gpurun_out/t_$v.$i.json 2>/dev/null; fi
  done
done
for f in gpurun_out/t_*.json; do python -c "import json,sys; d=json.load(open(sys.argv[1])); r=d['roofline']; print(sys.argv[1], round(d['value']), round(d['ms_per_step']*1000,1), {k:round(v['ms']*1000,1) for k,v in r['kernels'].items()})" $f; done
