# GPU-box check: parity tests, smoke, bench, ncu launch list + full captures.
# usage (from the repo root on the box): bash tools/gpu_check.sh [quick]
set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv
nproc
timeout 1500 python -m pytest tests -m gpu -q -rf --durations=10 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"
tail -25 gpurun_out/pytest_gpu.log
timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"; tail -3 gpurun_out/smoke.log
timeout 600 python bench.py --steps 20 --warmup 5 > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
cat gpurun_out/bench.json; tail -5 gpurun_out/bench.err
if [ "$1" != "quick" ]; then
  # launch list of the bench command (cold-cache, serialised: compare shares)
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
      --log-file gpurun_out/launches_bench.csv python bench.py --steps 5 --warmup 3 --no-cpu > /dev/null 2>&1
  echo "ncu launches rc=$?"
  for cfg in c1 c2a c2b; do
    timeout 900 ncu --set full --clock-control none --import-source on \
        -k 'regex:k_(features|csr_scalar|csr_vector|ell|dia|hyb_tail)' -c 16 \
        -o gpurun_out/prof_$cfg -f python tools/profile_variants.py $cfg > gpurun_out/prof_$cfg.log 2>&1
    echo "ncu full $cfg rc=$?"
  done
fi
