B=paper_conf_icpp_huangylhbl21_b200/build
run() { timeout 600 python bench.py --config c3 --sched det --grid 1184,1184 --col-balance --legs "" --no-e2e --no-cpu-baseline --fp16-leg none --steps 5 --warmup 3 > gpurun_out/pp.json 2>gpurun_out/pp.err; python -c "import json,sys;d=json.load(open('gpurun_out/pp.json'));print(sys.argv[1:], round(d['ms_per_step'],2))" "$@"; }
for rep in 1 2; do run P64; for d in 0 16 200; do HCCMF_LIB=$B/diag_P$d.so run P$d; done; done
