run() { timeout 600 python bench.py --config c4 --legs "" --no-e2e --no-cpu-baseline --fp16-leg none --steps 6 --warmup 2 "$@" > gpurun_out/c4n.json 2>gpurun_out/c4n.err; python -c "import json,sys;d=json.load(open('gpurun_out/c4n.json'));print(sys.argv[1:], round(d['ms_per_step'],2), [round(x,3) for x in d['rmse']['test_per_epoch']])" "$@"; }
run --grid 1,4
run --grid 1,8
run --grid 1,8 --warps 2368
run --grid 1,8 --warps 1184
run --grid 1,8 --warps 296
run --grid 1,1
run --grid 1,2
for lib in w40; do
HCCMF_LIB=paper_conf_icpp_huangylhbl21_b200/libhccmf_$lib.so timeout 600 python bench.py --legs "" --no-e2e --no-cpu-baseline --fp16-leg fp16sr --steps 5 --warmup 2 > gpurun_out/w.json 2>/dev/null
python -c "import json;d=json.load(open('gpurun_out/w.json'));print('$lib', round(d['value']/1e9,3), round(d['storage_fp16']['value']/1e9,3), d['roofline']['binding_frac'], d['clocks']['sm_mhz'])"
done
timeout 600 python bench.py --legs "" --no-e2e --no-cpu-baseline --fp16-leg fp16sr --steps 5 --warmup 2 > gpurun_out/w.json 2>/dev/null
python -c "import json;d=json.load(open('gpurun_out/w.json'));print('base', round(d['value']/1e9,3), round(d['storage_fp16']['value']/1e9,3), d['roofline']['binding_frac'], d['clocks']['sm_mhz'])"
