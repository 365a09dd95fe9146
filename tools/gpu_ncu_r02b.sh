#!/bin/bash
# Round-2 closing evidence at HEAD (run under gpurun from the repo root): GPU suite, the
# default bench line, an ncu launch list and one --set full capture of KQ and KM (cfg2).
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -x -q -m gpu > gpurun_out/${TAG:-z}_pytest.txt 2>&1; tail -2 gpurun_out/${TAG:-z}_pytest.txt
timeout 900 python bench.py > gpurun_out/${TAG:-z}_def.json 2> gpurun_out/${TAG:-z}_def.err; python tools/show_bench.py gpurun_out/${TAG:-z}_def.json | head -4
CMD="python bench.py --steps 20 --warmup 5 --reps 1 --no-cpu-baseline --no-e2e --no-also --no-graph"
$CMD > gpurun_out/${TAG:-z}_plain.log 2>&1 && \
ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"kq_kernel|km_kernel" -s 700 -c 40 --csv \
    --log-file gpurun_out/${TAG:-z}_launches.csv $CMD > gpurun_out/${TAG:-z}_ncu_list.log 2>&1 && \
ncu --set full --clock-control none --import-source on -k regex:"kq_kernel|km_kernel" -s 700 -c 2 \
    -o gpurun_out/${TAG:-z}_prof $CMD > gpurun_out/${TAG:-z}_ncu_full.log 2>&1
echo "ncu rc=$?"
