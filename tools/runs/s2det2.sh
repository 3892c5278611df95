# DET record-ring body: parity, bench leg, ncu full capture + source page, trace of the critical path
timeout 900 python -m pytest tests -m gpu -q -k "det or wave or slab or strata or balanced" > gpurun_out/det2_test.log 2>&1
echo "pytest rc=$?"; tail -2 gpurun_out/det2_test.log
for g in 2048 1536 1024; do
timeout 600 python bench.py --config c3 --sched det --grid $g,$g --col-balance --legs "" --no-e2e --no-cpu-baseline --fp16-leg none --steps 5 --warmup 3 > gpurun_out/det2_$g.json 2>gpurun_out/det2.err; python -c "import json,sys;d=json.load(open('gpurun_out/det2_$g.json'));print('B=$g', round(d['ms_per_step'],2), round(d['value']/1e9,3), d['clocks'], d.get('det_path'))"
done
R=/tmp/ncu; mkdir -p $R
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:sgd_wave_slab -c 1 -f -o $R/det python bench.py --config c3 --sched det --grid 2048,2048 --col-balance --legs "" --no-e2e --no-cpu-baseline --fp16-leg none --steps 1 --warmup 1 > gpurun_out/ncu_det2.log 2>&1; echo "ncu det rc=$?"
cp $R/det.ncu-rep gpurun_out/r02_det_ring.ncu-rep
python tools/ncu_summary.py $R/det.ncu-rep --json gpurun_out/r02_ncu_det_ring_summary.json | tail -3
ncu -i $R/det.ncu-rep --page source --csv > gpurun_out/det_ring_source.csv 2>/dev/null; ls -la gpurun_out/det_ring_source.csv
timeout 900 python tools/trace_det_wave.py --wave 1 --B 2048 --bal 2>&1 | tail -1
