B=paper_conf_icpp_huangylhbl21_b200/build
run() { timeout 600 python bench.py --config c3 --sched det --grid 1184,1184 --col-balance --legs "" --no-e2e --no-cpu-baseline --fp16-leg none --steps 5 --warmup 3 > gpurun_out/hh.json 2>gpurun_out/hh.err; python -c "import json,sys;d=json.load(open('gpurun_out/hh.json'));print(sys.argv[1:], round(d['ms_per_step'],2), d['rmse']['test_per_epoch'][-1])" "$@"; }
echo base; timeout 300 python tools/det_chain_latency.py 2>&1 | tail -1
echo half; HCCMF_LIB=$B/diag_HALF.so timeout 300 python tools/det_chain_latency.py 2>&1 | tail -1
for rep in 1 2; do run base; HCCMF_LIB=$B/diag_HALF.so run half; done
