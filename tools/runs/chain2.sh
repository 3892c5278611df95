timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "chain" > gpurun_out/chain2.log 2>&1; tail -3 gpurun_out/chain2.log
for g in 2048 1024 512; do
for w in 3; do
timeout 600 python bench.py --config c3 --sched det --grid $g,$g --det-wave $w --legs "" --no-e2e --no-cpu-baseline --fp16-leg none --steps 3 --warmup 2 > gpurun_out/chain_bench_w${w}_$g.json 2> gpurun_out/chain_bench_w${w}_$g.err
python -c "import json;d=json.load(open('gpurun_out/chain_bench_w${w}_$g.json'));print('grid $g wave $w', d['ms_per_step'], d['value']/1e9, d['rmse']['test_per_epoch'])"
tail -3 gpurun_out/chain_bench_w${w}_$g.err
done; done
