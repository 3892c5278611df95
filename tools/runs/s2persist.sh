for o in "l2_persist=0" "l2_persist=1"; do
timeout 900 python bench.py --legs "" --no-e2e --no-cpu-baseline --fp16-leg none --steps 6 --warmup 3 --opt $o > gpurun_out/ps.json 2>gpurun_out/ps.err; python -c "import json,sys;d=json.load(open('gpurun_out/ps.json'));print('$o', round(d['ms_per_step'],2), round(d['value']/1e9,3), d['clocks']['sm_mhz'])"
done
