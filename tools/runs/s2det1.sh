timeout 900 python -m pytest tests -m gpu -q -k "det or wave or slab or strata or balanced" > gpurun_out/det1_test.log 2>&1
echo "pytest rc=$?"; tail -5 gpurun_out/det1_test.log
run() { timeout 600 python bench.py --config c3 --sched det --grid 2048,2048 --col-balance --legs "" --no-e2e --no-cpu-baseline --fp16-leg none --steps 5 --warmup 3 > gpurun_out/det1.json 2>gpurun_out/det1.err; python -c "import json,sys;d=json.load(open('gpurun_out/det1.json'));print(sys.argv[1:], round(d['ms_per_step'],2), round(d['value']/1e9,3), d['clocks']['sm_mhz'], d.get('det_path'))" "$@"; }
run ring
HCCMF_SLAB_V1=1 run v1
run ring
HCCMF_SLAB_V1=1 run v1


