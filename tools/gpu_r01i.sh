timeout 150 python tools/early_diag.py 1 8 > gpurun_out/i_k1.txt 2>&1
timeout 150 python tools/early_diag.py 16 64 > gpurun_out/i_k16.txt 2>&1
for f in gpurun_out/i_k1.txt gpurun_out/i_k16.txt; do echo "== $f"; tail -n 4 $f; done
B="python bench.py --no-cpu-baseline --no-e2e"
FLECHE_EARLY_FETCH=1 timeout 200 $B > gpurun_out/i_cfg2_early.json 2>/dev/null
FLECHE_EARLY_FETCH=1 timeout 200 $B --config cfg5 --steps 300 > gpurun_out/i_cfg5_early.json 2>/dev/null
FLECHE_EARLY_FETCH=1 timeout 200 $B --config cfg1 > gpurun_out/i_cfg1_early.json 2>/dev/null
head -c 300 gpurun_out/i_cfg2_early.json
