#!/bin/bash
# One parameterised GPU batch (run under gpurun from the repo root):
#   tools/gpu_r02.sh TAG "pytest args (e.g. tests -m gpu)|-" "bench-variant ..." 
# Each bench variant is "name:ENV=V,ENV2=V2:bench args" and writes gpurun_out/<TAG>_<name>.json.
TAG=$1; shift
PYT=$1; shift
mkdir -p gpurun_out
if [ "$PYT" != "-" ]; then
  timeout 1500 python -m pytest -x -q $PYT > gpurun_out/${TAG}_pytest.txt 2>&1
  tail -3 gpurun_out/${TAG}_pytest.txt
fi
for v in "$@"; do
  name=${v%%:*}; rest=${v#*:}; envs=${rest%%:*}; args=${rest#*:}
  ( [ -n "$envs" ] && export $(echo $envs | tr ',' ' ');
    timeout 600 python bench.py $args > gpurun_out/${TAG}_${name}.json 2> gpurun_out/${TAG}_${name}.err )
  python tools/show_bench.py gpurun_out/${TAG}_${name}.json 2>/dev/null | head -6 || tail -3 gpurun_out/${TAG}_${name}.err
done
