R=/tmp/ncu; mkdir -p $R
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sgd_wave_slab -c 1 -f -o $R/lat python tools/det_chain_latency.py --ratings 400000 > gpurun_out/ncu_lat.log 2>&1; echo "ncu rc=$?"
ncu -i $R/lat.ncu-rep --page source --csv > gpurun_out/lat_source.csv 2>/dev/null; ls -la gpurun_out/lat_source.csv
