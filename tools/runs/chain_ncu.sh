ncu --set full --import-source on --clock-control none -k regex:sgd_wave_chain -c 1 -f -o gpurun_out/chain_prof python bench.py --config c3 --sched det --grid 1024,1024 --det-wave 3 --legs "" --no-e2e --no-cpu-baseline --fp16-leg none --steps 1 --warmup 1 > gpurun_out/chain_ncu.log 2>&1
tail -5 gpurun_out/chain_ncu.log
ls -la gpurun_out/
