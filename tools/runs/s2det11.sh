for g in 1024 1184 1280 1536 1792; do
timeout 600 python bench.py --config c3 --sched det --grid $g,$g --col-balance --legs "" --no-e2e --no-cpu-baseline --fp16-leg none --steps 5 --warmup 3 > gpurun_out/det11_$g.json 2>gpurun_out/det11.err; python -c "import json,sys;d=json.load(open('gpurun_out/det11_$g.json'));print('B=$g', round(d['ms_per_step'],2), round(d['value']/1e9,3), d['clocks'].get('sm_mhz'))"
done
timeout 900 python tools/trace_det_wave.py --wave 1 --B 1536 --bal 2>&1 | tail -1
