#!/bin/bash
# Round-2 close (run under gpurun from the repo root): GPU suite, default bench line, the
# Terabyte-shape (cfg3h) and key-sharded (one rank) lines, then an ncu launch list and one
# --set full capture of KQ and KM at cfg2.  Outputs gpurun_out/${TAG}_*.
TAG=${TAG:-fin}
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -x -q -m gpu > gpurun_out/${TAG}_pytest.txt 2>&1; tail -2 gpurun_out/${TAG}_pytest.txt
timeout 900 python bench.py > gpurun_out/${TAG}_def.json 2> gpurun_out/${TAG}_def.err; python tools/show_bench.py gpurun_out/${TAG}_def.json | head -3
A="--steps 200 --warmup 10 --no-cpu-baseline --no-e2e --no-also --no-graph"
timeout 900 python bench.py --config cfg3h --cache-frac 0.01 $A > gpurun_out/${TAG}_cfg3h.json 2> gpurun_out/${TAG}_cfg3h.err; python tools/show_bench.py gpurun_out/${TAG}_cfg3h.json | head -1
timeout 600 python bench.py --mode sharded --p2p $A > gpurun_out/${TAG}_sharded_p2p.json 2> gpurun_out/${TAG}_sharded_p2p.err; python tools/show_bench.py gpurun_out/${TAG}_sharded_p2p.json | head -1
timeout 600 python bench.py $A > gpurun_out/${TAG}_replicated.json 2> gpurun_out/${TAG}_replicated.err; python tools/show_bench.py gpurun_out/${TAG}_replicated.json | head -1
CMD="python bench.py --steps 20 --warmup 5 --reps 1 --no-cpu-baseline --no-e2e --no-also --no-graph"
$CMD > gpurun_out/${TAG}_plain.log 2>&1 && \
ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"kq_kernel|km_kernel" -s 700 -c 40 --csv \
    --log-file gpurun_out/${TAG}_launches.csv $CMD > gpurun_out/${TAG}_ncu_list.log 2>&1 && \
ncu --set full --clock-control none --import-source on -k regex:"kq_kernel|km_kernel" -s 700 -c 2 \
    -o gpurun_out/${TAG}_prof $CMD > gpurun_out/${TAG}_ncu_full.log 2>&1
echo "ncu rc=$?"
