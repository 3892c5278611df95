timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_full_size.py -q -x -k "wavefront or det or balance" 2>&1 | tail -3
run() { timeout 600 python bench.py --config c3 --sched det --legs "" --no-e2e --no-cpu-baseline --fp16-leg none --steps 3 --warmup 2 "$@" > gpurun_out/bal.json 2> gpurun_out/bal.err; python -c "import json,sys;d=json.load(open('gpurun_out/bal.json'));print(sys.argv[1:], round(d['ms_per_step'],2), round(d['value']/1e9,3), d['rmse']['test_per_epoch'][-1])" "$@"; tail -2 gpurun_out/bal.err; }
run --grid 2048,2048 --col-balance
run --grid 1024,1024 --col-balance
run --grid 1536,1536 --col-balance
run --grid 2048,2048
timeout 900 python tools/trace_det_wave.py --wave 1 --B 2048 --bal 2>&1 | tail -1
