for g in 1024 1184 1280 1536 1792 2048; do
timeout 600 python bench.py --config c3 --sched det --grid $g,$g --col-balance --legs "" --no-e2e --no-cpu-baseline --fp16-leg none --steps 5 --warmup 3 > gpurun_out/det18_$g.json 2>gpurun_out/det18.err; python -c "import json,sys;d=json.load(open('gpurun_out/det18_$g.json'));print('B=$g', round(d['ms_per_step'],2), round(d['value']/1e9,3), d['clocks'].get('sm_mhz'))"
done
