for tool in memcheck racecheck synccheck; do
  NB=4 timeout 900 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_run.py > gpurun_out/sanitizer_${tool}_r01b.log 2>&1
done
B="python bench.py --no-cpu-baseline --no-e2e"
timeout 400 $B --config cfg4 --steps 100 > gpurun_out/k_cfg4.json 2>/dev/null
timeout 400 $B --config cfg4 --steps 100 --host-assist --ha-frac 0.5 > gpurun_out/k_cfg4_ha.json 2>/dev/null
tail -n 3 gpurun_out/sanitizer_*_r01b.log
