timeout 900 python -m pytest tests -m gpu -q -k "det or wave or slab or strata or balanced" > gpurun_out/y_test.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/y_test.log
run() { timeout 600 python bench.py --config c3 --sched det --grid 1536,1536 --col-balance --legs "" --no-e2e --no-cpu-baseline --fp16-leg none --steps 5 --warmup 3 > gpurun_out/y.json 2>gpurun_out/y.err; python -c "import json,sys;d=json.load(open('gpurun_out/y.json'));print(sys.argv[1:], round(d['ms_per_step'],2), round(d['value']/1e9,3), round(d['roofline'].get('binding_frac',0),3))" "$@"; }
run base
HCCMF_SLAB_ONE_CTA=1 run onecta
HCCMF_SLAB_ONE_CTA=1 HCCMF_SLAB_YIELD_NS=100 run onecta y100
HCCMF_SLAB_ONE_CTA=1 HCCMF_SLAB_YIELD_NS=300 run onecta y300
HCCMF_SLAB_ONE_CTA=1 HCCMF_SLAB_YIELD_NS=1000 run onecta y1000
HCCMF_SLAB_YIELD_NS=300 run y300
