timeout 1500 python -m pytest tests -m gpu -q -rf 2>&1 | grep -E "FAILED|passed|failed" | head -10
timeout 400 python bench.py > gpurun_out/u_default.json 2>/dev/null
B="python bench.py --no-cpu-baseline --no-e2e"
timeout 900 $B --config cfg3h --steps 200 --cache-frac 0.01 --host-assist > gpurun_out/u_cfg3h_ha.json 2>/dev/null
timeout 300 $B --config cfg5 --steps 300 --host-assist > gpurun_out/u_cfg5_ha.json 2>/dev/null
for f in gpurun_out/u_*.json; do python -c "import json,sys; d=json.load(open(sys.argv[1])); r=d['roofline']; print(sys.argv[1], round(d['value']), round(d['ms_per_step']*1000,1), {k:round(v['ms']*1000,1) for k,v in r['kernels'].items()}, round(r['frac'],3))" $f; done
