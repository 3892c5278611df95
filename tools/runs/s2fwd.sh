timeout 900 python -m pytest tests -m gpu -q -k "det or wave or slab or strata or balanced" > gpurun_out/fwd_test.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/fwd_test.log
timeout 300 python tools/det_chain_latency.py 2>&1 | tail -1
for rep in 1 2; do for g in 1184 1536; do
timeout 600 python bench.py --config c3 --sched det --grid $g,$g --col-balance --legs "" --no-e2e --no-cpu-baseline --fp16-leg none --steps 5 --warmup 3 > gpurun_out/f_$g.json 2>gpurun_out/f.err; python -c "import json,sys;d=json.load(open('gpurun_out/f_$g.json'));print('B=$g', round(d['ms_per_step'],2), round(d['roofline']['binding_frac'],3))"
done; done
