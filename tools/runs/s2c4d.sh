for gr in 1,2 1,3; do
timeout 600 python bench.py --config c4 --grid $gr --legs "" --no-e2e --no-cpu-baseline --fp16-leg none --steps 6 --warmup 3 > gpurun_out/c4g.json 2>gpurun_out/c4g.err; python -c "import json,sys;d=json.load(open('gpurun_out/c4g.json'));print('grid $gr', round(d['ms_per_step'],2), round(d['value']/1e9,3), [round(x,3) for x in d['rmse']['test_per_epoch']][-3:])"
done
