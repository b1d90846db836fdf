# GPU-box check: parity tests, smoke, bench, variant table, ncu launch list +
# full captures (exported to CSV on the box; the .ncu-rep files are too big
# to bring back).  usage: bash tools/gpu_check.sh [tests|bench|table|prof]...  (default: all)
set -x
mkdir -p gpurun_out
ALL="$*"
[ -z "$ALL" ] && ALL="tests bench table prof"
want() { for a in $ALL; do [ "$a" = "$1" ] && return 0; done; return 1; }
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv
if want tests; then
  timeout 1500 python -m pytest tests -m gpu -q -rf --durations=10 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"
  tail -25 gpurun_out/pytest_gpu.log
  timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"; tail -3 gpurun_out/smoke.log
fi
if want bench; then
  timeout 600 python bench.py --steps 20 --warmup 5 > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
  cat gpurun_out/bench.json; tail -5 gpurun_out/bench.err
fi
if want table; then
  timeout 900 python tools/profile_variants.py --time c1 c2a c2b short > gpurun_out/variant_table.json 2> gpurun_out/variant_table.err
  echo "table rc=$?"; cat gpurun_out/variant_table.json | python -c "import json,sys; t=json.load(sys.stdin); [print(c, round(r['feature_ms'],3), {k: round(v['GBps']) for k,v in r['variants'].items()}) for c,r in t.items()]"
fi
if want prof; then
  timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
      --log-file gpurun_out/launches_bench.csv python bench.py --steps 5 --warmup 3 --no-cpu > /dev/null 2>&1
  echo "ncu launches rc=$?"
  for cfg in c1 c2a c2b; do
    timeout 900 ncu --set full --clock-control none --import-source on \
        -k 'regex:k_(features|csr_scalar|csr_vector|ell|dia|hyb_tail|hyb_fixup)' -c 24 \
        -o /tmp/prof_$cfg -f python tools/profile_variants.py $cfg > gpurun_out/prof_$cfg.log 2>&1
    echo "ncu full $cfg rc=$?"
    ncu -i /tmp/prof_$cfg.ncu-rep --page raw --csv > gpurun_out/prof_${cfg}_raw.csv 2>/dev/null
    case $cfg in
      c1)  srcs="dia csr_vector features ell" ;;
      c2b) srcs="hyb_tail csr_vector" ;;
      *)   srcs="" ;;
    esac
    for k in $srcs; do
      ncu -i /tmp/prof_$cfg.ncu-rep --page source --csv -k regex:k_$k -c 1 > gpurun_out/prof_${cfg}_src_$k.csv 2>/dev/null
    done
  done
  du -sh gpurun_out
fi
