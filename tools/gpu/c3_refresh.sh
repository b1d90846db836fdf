# after a configs[3] recipe change: GPU tests, feature study, bench line (selection leg + picks)
mkdir -p gpurun_out/artifacts
timeout 1500 python -m pytest tests -m gpu -q -x -rf > gpurun_out/pytest_full.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_full.log
timeout 1200 python tools/feature_study.py --gpu > gpurun_out/feature_study.log 2>&1; echo "fstudy rc=$?"; tail -8 gpurun_out/feature_study.log
cp artifacts/feature_study.json gpurun_out/artifacts/
timeout 900 python bench.py > gpurun_out/bench_r02.json 2> gpurun_out/bench_r02.err; echo "bench rc=$?"; tail -14 gpurun_out/bench_r02.err
