# ncu full capture of the feature-pass kernels on c2a / c2b (CSV exported on the box)
mkdir -p gpurun_out
for cfg in ${CFGS:-c2a c2b}; do
  timeout 900 ncu --set full --clock-control none --import-source on -k 'regex:k_features' -c 2 \
      -o /tmp/feat_$cfg -f python tools/profile_variants.py $cfg none > gpurun_out/featprof_$cfg.log 2>&1
  echo "ncu $cfg rc=$?"
  ncu -i /tmp/feat_$cfg.ncu-rep --page raw --csv > gpurun_out/featprof_${cfg}_raw.csv 2>/dev/null
  ncu -i /tmp/feat_$cfg.ncu-rep --page source --csv -k regex:k_features$ -c 1 > gpurun_out/featprof_${cfg}_src.csv 2>/dev/null
  ncu -i /tmp/feat_$cfg.ncu-rep --page details --csv > gpurun_out/featprof_${cfg}_details.csv 2>/dev/null
done
ls -la gpurun_out | grep featprof
