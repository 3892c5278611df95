export HCCMF_BAND_REPORT=$PWD/gpurun_out/band_report4.jsonl
rm -f $HCCMF_BAND_REPORT
timeout 1800 python -m pytest tests -m gpu -q -k "c4_scaled or sanitizer or column_phases" > gpurun_out/gputest_4.log 2>&1
echo "pytest rc=$?"; tail -5 gpurun_out/gputest_4.log
timeout 1500 python bench.py > gpurun_out/bench_full4.json 2> gpurun_out/bench_full4.err
echo "bench rc=$?"; tail -3 gpurun_out/bench_full4.err
python - <<'PY'
import json
d=json.load(open('gpurun_out/bench_full4.json'))
print('C5', round(d['value']/1e9,3), round(d['ms_per_step'],1), d['clocks'], 'frac', round(d['roofline']['frac'],4), 'bfrac', round(d['roofline']['binding_frac'],3))
print('fp16', round(d['storage_fp16']['value']/1e9,3), d['storage_fp16']['roofline']['binding_frac'])
print('e2e', d['e2e'].get('value'), d['e2e'].get('s_per_step'))
for k,v in d['legs'].items():
    print(k, round(v['value']/1e9,3), round(v['ms_per_step'],2), v['clocks'], v.get('e2e') and v['e2e'].get('value'), v['roofline'].get('binding_frac'))
PY
