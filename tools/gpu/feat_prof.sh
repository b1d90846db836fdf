# K1 timing A/B (ab/libnitro_head.so vs in-tree) + ncu SASS-level source page of k_features on c1 / c4
mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -q -x -k "feature or canonical or c1 or c4 or smoke" > gpurun_out/pytest_feat.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_feat.log
CFGS="${CFGS:-c1 c4 c2a c2b short band01 uvar3 band48}" bash tools/gpu/feat_ab2.sh
for cfg in ${PCFG:-c1 c4}; do
  timeout 900 ncu --set full --clock-control none --import-source on -k 'regex:k_features$|k_features<' -c 1 \
      -o /tmp/feat_$cfg -f python tools/profile_variants.py $cfg none > gpurun_out/featprof_$cfg.log 2>&1
  echo "ncu $cfg rc=$?"
  ncu -i /tmp/feat_$cfg.ncu-rep --page raw --csv > gpurun_out/featprof_${cfg}_raw.csv 2>/dev/null
  ncu -i /tmp/feat_$cfg.ncu-rep --page source --csv --print-source cuda,sass > gpurun_out/featprof_${cfg}_src.csv 2>/dev/null
done
