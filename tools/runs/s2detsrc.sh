R=/tmp/ncu; mkdir -p $R
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:sgd_wave_slab -c 1 -f -o $R/det python bench.py --config c3 --sched det --grid 1184,1184 --col-balance --legs "" --no-e2e --no-cpu-baseline --fp16-leg none --steps 1 --warmup 1 > gpurun_out/ncu_detsrc.log 2>&1; echo "ncu rc=$?"
ncu -i $R/det.ncu-rep --page source --csv > gpurun_out/det_final_source.csv 2>/dev/null; ls -la gpurun_out/det_final_source.csv
