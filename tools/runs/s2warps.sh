for w in 2960 3552 4144 4736; do
timeout 600 python bench.py --legs "" --no-e2e --no-cpu-baseline --fp16-leg none --steps 6 --warmup 3 --warps $w > gpurun_out/w_$w.json 2>gpurun_out/w.err; python -c "import json,sys;d=json.load(open('gpurun_out/w_$w.json'));print('warps $w', round(d['ms_per_step'],2), round(d['value']/1e9,3), d['clocks'])"
done
