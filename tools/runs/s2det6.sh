timeout 900 python -m pytest tests -m gpu -q -k "det or wave or slab or strata or balanced" > gpurun_out/det6_test.log 2>&1
echo "pytest rc=$?"; tail -12 gpurun_out/det6_test.log
for g in 1024 1536 2048; do
timeout 600 python bench.py --config c3 --sched det --grid $g,$g --col-balance --legs "" --no-e2e --no-cpu-baseline --fp16-leg none --steps 5 --warmup 3 > gpurun_out/det6_$g.json 2>gpurun_out/det6.err; python -c "import json,sys;d=json.load(open('gpurun_out/det6_$g.json'));print('B=$g', round(d['ms_per_step'],2), round(d['value']/1e9,3), d['clocks']['sm_mhz'], d['rmse']['test_per_epoch'])"
done
timeout 900 python tools/trace_det_wave.py --wave 1 --B 2048 --bal 2>&1 | tail -1
