B="python bench.py --no-cpu-baseline --no-e2e --config cfg3h --steps 200"
timeout 900 $B --cache-frac 0.01 > gpurun_out/s_cfg3h_001.json 2>gpurun_out/s_err1.txt
timeout 900 $B --cache-frac 0.01 --host-assist > gpurun_out/s_cfg3h_001_ha.json 2>gpurun_out/s_err2.txt
for f in gpurun_out/s_cfg3h_*.json; do python -c "import json,sys; d=json.load(open(sys.argv[1])); print(sys.argv[1], round(d['value']), round(d['ms_per_step']*1000,1), d['hit_ratio'], d['assisted_rows_per_step'])" $f; done
tail -2 gpurun_out/s_err1.txt
