timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "chain" > gpurun_out/chain1.log 2>&1; tail -15 gpurun_out/chain1.log
for w in 1 3; do
timeout 600 python bench.py --config c3 --sched det --grid 2048,2048 --det-wave $w --legs "" --no-e2e --no-cpu-baseline --fp16-leg none --steps 3 --warmup 2 > gpurun_out/chain_bench_w$w.json 2> gpurun_out/chain_bench_w$w.err
python -c "import json;d=json.load(open('gpurun_out/chain_bench_w$w.json'));print('wave $w', d['ms_per_step'], d['value']/1e9, d['rmse']['test_per_epoch'])"
tail -3 gpurun_out/chain_bench_w$w.err
done
