# DET grid sweep with the record-ring slab wavefront (C3, balanced columns)
for g in 296 444 592 740 888 1184 1536 2048; do
timeout 600 python bench.py --config c3 --sched det --grid $g,$g --col-balance --legs "" --no-e2e --no-cpu-baseline --fp16-leg none --steps 3 --warmup 3 > gpurun_out/det3_$g.json 2>gpurun_out/det3.err; python -c "import json,sys;d=json.load(open('gpurun_out/det3_$g.json'));print('B=$g', round(d['ms_per_step'],2), round(d['value']/1e9,3), d['clocks']['sm_mhz'], d.get('det_path'))"
done
timeout 900 python tools/trace_det_wave.py --wave 1 --B 592 --bal 2>&1 | tail -1
