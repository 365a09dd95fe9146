# compute-sanitizer over HEAD's changed paths (deferred KQ timestamp exchange, overlapped host entry point)
timeout 900 compute-sanitizer --tool memcheck --error-exitcode 9 python tools/sanitize_run.py > gpurun_out/san2_memcheck.log 2>&1; echo "memcheck rc=$?" >> gpurun_out/san2_memcheck.log
timeout 900 compute-sanitizer --tool racecheck --error-exitcode 9 python tools/sanitize_run.py > gpurun_out/san2_racecheck.log 2>&1; echo "racecheck rc=$?" >> gpurun_out/san2_racecheck.log
timeout 900 compute-sanitizer --tool memcheck --error-exitcode 9 python -m pytest tests/test_gpu_parity.py -q -x -k "query_host or back_to_back" > gpurun_out/san2_host.log 2>&1; echo "memcheck host rc=$?" >> gpurun_out/san2_host.log
tail -n 3 gpurun_out/san2_memcheck.log gpurun_out/san2_racecheck.log gpurun_out/san2_host.log
