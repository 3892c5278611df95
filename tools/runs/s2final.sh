timeout 1500 python bench.py > gpurun_out/bench_s2g.json 2> gpurun_out/bench_s2g.err
echo "bench rc=$?"; tail -2 gpurun_out/bench_s2g.err
python - <<'PY'
import json
d=json.load(open('gpurun_out/bench_s2g.json'))
r=d['roofline']
print('C5', round(d['value']/1e9,3), round(d['ms_per_step'],1), d['clocks'], 'frac', round(r['frac'],4), 'bfrac', round(r['binding_frac'],3), 'rtfrac', round(r.get('roundtrip_frac',0),3))
print('fp16', round(d['storage_fp16']['value']/1e9,3), d['storage_fp16']['roofline']['binding_frac'])
print('e2e', d['e2e'].get('value'), d['e2e'].get('s_per_step'), 'launches', d['gpu_launches'])
for k,v in d['legs'].items():
    print(k, round(v['value']/1e9,3), round(v['ms_per_step'],2), v['clocks'], v.get('e2e') and v['e2e'].get('value'), v['roofline'].get('binding_frac'))
PY
