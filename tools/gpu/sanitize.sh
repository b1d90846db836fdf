# compute-sanitizer over tools/sanitize_run.py: memcheck on everything; racecheck
# on the single-thread part and on the 2-host-thread loopback part separately
mkdir -p gpurun_out
( echo '$ NITRO_CSRV_HOT=2 compute-sanitizer --tool memcheck python tools/sanitize_run.py'
  NITRO_CSRV_HOT=2 timeout 1500 compute-sanitizer --tool memcheck python tools/sanitize_run.py 2>&1 | tail -3
  echo; echo '$ NITRO_CSRV_HOT=2 SANITIZE_PARTS=single compute-sanitizer --tool racecheck python tools/sanitize_run.py'
  NITRO_CSRV_HOT=2 SANITIZE_PARTS=single timeout 1500 compute-sanitizer --tool racecheck python tools/sanitize_run.py 2>&1 | tail -3
  for i in 1 2 3; do
    echo; echo "\$ NITRO_CSRV_HOT=2 SANITIZE_PARTS=loopback compute-sanitizer --tool racecheck python tools/sanitize_run.py   # run $i"
    NITRO_CSRV_HOT=2 SANITIZE_PARTS=loopback timeout 1500 compute-sanitizer --tool racecheck python tools/sanitize_run.py 2>&1 | tail -5
  done ) > gpurun_out/sanitizers_r02.txt
cat gpurun_out/sanitizers_r02.txt
