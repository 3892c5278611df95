timeout 900 python -m pytest tests/test_gpu_full_size.py -m gpu -q -k "det" > gpurun_out/d1184_test.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/d1184_test.log
for rep in 1 2; do for g in 1184 1536; do
timeout 600 python bench.py --config c3 --sched det --grid $g,$g --col-balance --legs "" --no-e2e --no-cpu-baseline --fp16-leg none --steps 5 --warmup 3 > gpurun_out/d_$g.json 2>gpurun_out/d.err; python -c "import json,sys;d=json.load(open('gpurun_out/d_$g.json'));print('B=$g', round(d['ms_per_step'],2), round(d['value']/1e9,3), round(d['roofline']['binding_frac'],3))"
done; done
R=/tmp/ncu; mkdir -p $R
timeout 1200 ncu --set full --clock-control none -k regex:sgd_wave_slab -c 1 -f -o $R/det python bench.py --config c3 --sched det --grid 1184,1184 --col-balance --legs "" --no-e2e --no-cpu-baseline --fp16-leg none --steps 1 --warmup 1 > gpurun_out/ncu_d1184.log 2>&1; echo "ncu rc=$?"
python tools/ncu_summary.py $R/det.ncu-rep --json gpurun_out/r02_ncu_det_B1184_summary.json | tail -1
