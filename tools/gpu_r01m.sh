B="python bench.py --no-cpu-baseline --no-e2e"
for d in 16 32 128; do timeout 300 $B --dim $d > gpurun_out/m_dim$d.json 2>/dev/null; done
for bs in 1024 2048 4096 16384 32768; do timeout 300 $B --batch $bs > gpurun_out/m_batch$bs.json 2>/dev/null; done
ls gpurun_out/m_*
