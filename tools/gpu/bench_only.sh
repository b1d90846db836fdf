mkdir -p gpurun_out
timeout 900 python bench.py > gpurun_out/bench_r02.json 2> gpurun_out/bench_r02.err; echo "bench rc=$?"; tail -14 gpurun_out/bench_r02.err
