B=paper_conf_icpp_huangylhbl21_b200/build
run() { timeout 600 python bench.py --config c3 --sched det --grid 1184,1184 --col-balance --legs "" --no-e2e --no-cpu-baseline --fp16-leg none --steps 5 --warmup 3 > gpurun_out/dd.json 2>gpurun_out/dd.err; python -c "import json,sys;d=json.load(open('gpurun_out/dd.json'));print(sys.argv[1:], round(d['ms_per_step'],2), round(d['roofline']['binding_frac'],3))" "$@"; }
for rep in 1 2; do
run D12
for d in 6 8 14; do HCCMF_LIB=$B/diag_D$d.so run D$d; done
done
