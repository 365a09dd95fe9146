# e2e A/B (round-1 builds): fleche_query_host ordered vs FLECHE_HOST_OVERLAP=1 (now the default; FLECHE_HOST_ORDERED=1 gives the old order), alternating, same box
B="python bench.py --no-cpu-baseline"
for r in 4 5 6 7 8; do
  timeout 300 $B > gpurun_out/eab_ordered_$r.json 2>/dev/null
  FLECHE_HOST_OVERLAP=1 timeout 300 $B > gpurun_out/eab_overlap_$r.json 2>/dev/null
done
for f in gpurun_out/eab_*.json; do python -c "import json,sys; d=json.load(open(sys.argv[1])); print(sys.argv[1], round(d['value']), 'e2e', round(d['e2e']['value'],1))" $f; done
