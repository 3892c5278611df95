for st in 80 60; do
timeout 600 python bench.py --config c4 --legs "" --no-e2e --no-cpu-baseline --fp16-leg none --steps 6 --warmup 3 --opt staleness=$st > gpurun_out/c4s_$st.json 2>gpurun_out/c4s_$st.err; echo "rc=$?"; python -c "import json,sys;d=json.load(open('gpurun_out/c4s_$st.json'));print('st=$st', round(d['ms_per_step'],2), round(d['value']/1e9,3), [round(x,3) for x in d['rmse']['test_per_epoch']])"; tail -2 gpurun_out/c4s_$st.err
done
