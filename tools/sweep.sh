# DIA row-tiled layout vs column-major on configs[1] / 256^3 / short; tiled parity
t() { timeout 300 python tools/profile_variants.py --time $1 $2 2>/dev/null | python -c "import json,sys; t=json.load(sys.stdin); print({c: {k: (round(v['GBps']), round(v['ms']*1e3,1)) for k,v in r['variants'].items()} for c,r in t.items()})"; }
for tl in 0 1024 4096 16384; do echo "DIA_TILE=$tl"; NITRO_DIA_TILE=$tl t "c1 c1big short" "dia"; done
NITRO_DIA_TILE=1024 timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -m gpu 2>&1 | tail -3
python -c "
import torch
a=torch.ones(1<<28,device='cuda'); f=torch.empty(512<<20,dtype=torch.uint8,device='cuda')
s,e=torch.cuda.Event(enable_timing=True),torch.cuda.Event(enable_timing=True)
for mb in [242,470,1000]:
    v=a[:(mb<<20)//4]; ts=[]
    for r in range(23):
        f.fill_(r); s.record(); v.sum(); e.record(); torch.cuda.synchronize(); ts.append(s.elapsed_time(e))
    ts=sorted(ts[3:]); t=ts[len(ts)//2]*1e-3; print('read-only sum', mb, 'MB', round(t*1e6,1), 'us', round((mb<<20)/t/1e9), 'GB/s')
"
