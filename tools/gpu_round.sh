# Full GPU refresh after a kernel change: parity suite, smoke, configs[3]
# retrain + incremental tuning + feature study, bench, variant table, configs[4].
# usage: bash tools/gpu_round.sh [steps...]  (default: all)
mkdir -p gpurun_out
ALL="$*"
[ -z "$ALL" ] && ALL="tests c3 bench table c4"
want() { for a in $ALL; do [ "$a" = "$1" ] && return 0; done; return 1; }
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv,noheader
if want tests; then
  timeout 1800 python -m pytest tests -m gpu -q -rf --durations=15 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"
  tail -22 gpurun_out/pytest_gpu.log
  timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/smoke.log
fi
if want c3; then
  timeout 1800 python tools/train_select.py > gpurun_out/c3_train_select.log 2>&1; echo "c3 rc=$?"; tail -4 gpurun_out/c3_train_select.log
  timeout 600 python tools/itune_c3.py > gpurun_out/c3_itune.log 2>&1; echo "itune rc=$?"; tail -3 gpurun_out/c3_itune.log
  timeout 1200 python tools/feature_study.py --gpu > gpurun_out/feature_study.log 2>&1; echo "fstudy rc=$?"; tail -4 gpurun_out/feature_study.log
  mkdir -p gpurun_out/artifacts; cp artifacts/* gpurun_out/artifacts/
fi
if want fstudy; then
  timeout 1200 python tools/feature_study.py --gpu > gpurun_out/feature_study.log 2>&1; echo "fstudy rc=$?"; tail -4 gpurun_out/feature_study.log
  mkdir -p gpurun_out/artifacts; cp artifacts/feature_study.json gpurun_out/artifacts/
fi
if want bench; then
  timeout 600 python bench.py --steps 20 --warmup 5 > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
  cat gpurun_out/bench.json; tail -3 gpurun_out/bench.err
fi
if want table; then
  timeout 900 python tools/profile_variants.py --time --csr-ab c1 c2a c2b short band01 uvar3 > gpurun_out/variant_table.json 2> gpurun_out/variant_table.err
  echo "table rc=$?"; python -c "
import json; t=json.load(open('gpurun_out/variant_table.json'))
for c,r in t.items(): print(c, round(r['feature_ms'],3), {k: round(v['GBps']) for k,v in r['variants'].items()})"
fi
if want prof; then
  bash tools/gpu_check.sh prof
fi
if want c4; then
  timeout 1200 python tools/c4_probe.py --out gpurun_out/c4_probe.json > gpurun_out/c4_probe.log 2>&1; echo "c4 rc=$?"; tail -12 gpurun_out/c4_probe.log
fi
