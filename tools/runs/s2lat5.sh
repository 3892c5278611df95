timeout 900 python -m pytest tests -m gpu -q -k "det or wave or slab or strata or balanced" > gpurun_out/det19_test.log 2>&1
echo "pytest rc=$?"; tail -2 gpurun_out/det19_test.log
timeout 300 python tools/det_chain_latency.py 2>&1 | tail -1
for g in 1536 2048; do
timeout 600 python bench.py --config c3 --sched det --grid $g,$g --col-balance --legs "" --no-e2e --no-cpu-baseline --fp16-leg none --steps 5 --warmup 3 > gpurun_out/det19_$g.json 2>gpurun_out/det19.err; python -c "import json,sys;d=json.load(open('gpurun_out/det19_$g.json'));print('B=$g', round(d['ms_per_step'],2), round(d['value']/1e9,3), d['clocks']['sm_mhz'])"
done
timeout 900 python tools/trace_det_wave.py --wave 1 --B 1536 --bal 2>&1 | tail -1
