# round-1 final matrix at HEAD (one box, back to back)
B="python bench.py --no-cpu-baseline --no-e2e"
timeout 300 $B --config cfg1 > gpurun_out/mx_cfg1.json 2>/dev/null
timeout 300 $B --flags 2 > gpurun_out/mx_cfg2_static.json 2>/dev/null
timeout 300 $B --flags 6 > gpurun_out/mx_cfg2_static_pt.json 2>/dev/null
timeout 300 $B --config cfg5 --steps 300 > gpurun_out/mx_cfg5.json 2>/dev/null
timeout 300 $B --mode sharded --p2p 2>/dev/null | tail -1 > gpurun_out/mx_cfg2_sharded_p2p.json
timeout 500 $B --config cfg4 --steps 60 --flags 2 > gpurun_out/mx_cfg4_static.json 2>/dev/null
for f in gpurun_out/mx_*.json; do python -c "import json,sys; d=json.load(open(sys.argv[1])); r=d['roofline']; print(sys.argv[1], round(d['value']), round(d['ms_per_step']*1000,1), round(d['hit_ratio'],4), round(r['frac'],3))" $f; done
