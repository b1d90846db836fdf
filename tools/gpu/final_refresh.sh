# final round-2 refresh after the feature-pass changes: tests, smoke, feature study,
# variant table, bench line, ncu launch list + full captures (c2b with hot-x staging)
mkdir -p gpurun_out/artifacts
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
timeout 1500 python -m pytest tests -m gpu -q -x -rf --durations=5 > gpurun_out/pytest_full.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_full.log
timeout 300 python __graft_entry__.py smoke 2>&1 | tail -1
timeout 1200 python tools/feature_study.py --gpu > gpurun_out/feature_study.log 2>&1; echo "fstudy rc=$?"; tail -4 gpurun_out/feature_study.log
timeout 600 python tools/profile_variants.py --time c1 c2a c2b short band01 uvar3 band48 c4 > gpurun_out/variant_table_r02.json 2>/dev/null; echo "table rc=$?"
cp artifacts/feature_study.json gpurun_out/artifacts/
timeout 900 python bench.py > gpurun_out/bench_r02.json 2> gpurun_out/bench_r02.err; echo "bench rc=$?"; tail -12 gpurun_out/bench_r02.err
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv -c 600 \
    --log-file gpurun_out/launches_r02_bench.csv python bench.py --steps 5 --warmup 3 --quick --no-cpu > gpurun_out/bench_under_ncu.log 2>&1
echo "ncu launches rc=$?"
for cfg in c1 c2a c2b c4; do
  case $cfg in
    c4) rx='regex:k_(features|dia)'; n=8 ;;
    *) rx='regex:k_(features|csr_scalar|csr_vector|csr_vec4|csr_stream|ell|dia|hyb_tail|hyb_fixup)'; n=24 ;;
  esac
  timeout 1200 ncu --set full --clock-control none --import-source on -k "$rx" -c $n \
      -o /tmp/prof_$cfg -f python tools/profile_variants.py $cfg > gpurun_out/prof_$cfg.log 2>&1
  echo "ncu full $cfg rc=$?"
  ncu -i /tmp/prof_$cfg.ncu-rep --page raw --csv > gpurun_out/prof_${cfg}_raw.csv 2>/dev/null
done
ncu -i /tmp/prof_c4.ncu-rep --page source --csv -k regex:k_dia -c 1 > gpurun_out/prof_c4_src_dia.csv 2>/dev/null
ncu -i /tmp/prof_c2b.ncu-rep --page source --csv -k regex:k_csr_stream -c 1 > gpurun_out/prof_c2b_src_csr_stream.csv 2>/dev/null
du -sh gpurun_out
