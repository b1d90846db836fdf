mkdir -p gpurun_out
( echo '$ NITRO_CSRV_HOT=2 compute-sanitizer --tool memcheck python tools/sanitize_run.py'
  NITRO_CSRV_HOT=2 timeout 1500 compute-sanitizer --tool memcheck python tools/sanitize_run.py 2>&1 | tail -5
  echo; echo '$ NITRO_CSRV_HOT=2 compute-sanitizer --tool racecheck python tools/sanitize_run.py'
  NITRO_CSRV_HOT=2 timeout 1500 compute-sanitizer --tool racecheck python tools/sanitize_run.py 2>&1 | tail -5 ) > gpurun_out/sanitizers_r02.txt
cat gpurun_out/sanitizers_r02.txt
