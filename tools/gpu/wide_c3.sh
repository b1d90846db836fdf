# experiment: configs[3] with a wider size range (train_select --wide), then the picks of both models on
# the bench's configs[4] / c2a / c2b feature vectors
mkdir -p gpurun_out/wide
timeout 3000 python tools/train_select.py --wide --wide-log2 ${WL:-26} --out gpurun_out/wide > gpurun_out/wide/train.log 2>&1; echo "rc=$?"
tail -28 gpurun_out/wide/train.log
python - <<'PY'
import json, sys
sys.path.insert(0, '.')
import paper_conf_ipps_muralidharanshgc14_b200 as nitro
d = json.loads(open('profiles/bench_r02.json').read().strip().splitlines()[-1])
cases = {'c4': (d['features'], [True] * 5)}
for c, v in d['configs'].items():
    cases[c] = (v['features'], [n in v['allowed'] for n in nitro.VARIANT_NAMES])
for tag, path in (('paper', 'gpurun_out/wide/spmv_model.txt'), ('r11x', 'gpurun_out/wide/spmv_model_r11x.txt')):
    ctx = nitro.Context(); cv = nitro.CodeVariant(ctx, 'spmv'); cv.register_spmv(); cv.load(path)
    print(tag, {c: nitro.VARIANT_NAMES[cv.predict([f[k] for k in nitro.FEATURE_NAMES], al)] for c, (f, al) in cases.items()})
PY
