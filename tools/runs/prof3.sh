# ncu captures: reports stay in /tmp on the box, summaries come back (gpurun_out <= 64 MiB)
R=/tmp/ncu; mkdir -p $R
K='regex:sgd_warp_kernel|stream_kernel|roundtrip_kernel'
timeout 1200 ncu --set full --clock-control none -k "$K" -f -o $R/r02_l2split_c5 python tools/l2_split.py --config c5 > gpurun_out/ncu_c5.log 2>&1; echo "ncu c5 rc=$?"
timeout 1200 ncu --set full --clock-control none -k "$K" -f -o $R/r02_l2split_c4 python tools/l2_split.py --config c4 > gpurun_out/ncu_c4.log 2>&1; echo "ncu c4 rc=$?"
timeout 1200 ncu --set full --clock-control none -k regex:sgd_warp_kernel -c 2 -f -o $R/r02_c5_fp16sr python tools/l2_split.py --config c5 --storage fp16sr > gpurun_out/ncu_c5_16.log 2>&1; echo "ncu c5 fp16sr rc=$?"
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:sgd_wave_slab -c 1 -f -o $R/r02_det_slab_bal python bench.py --config c3 --sched det --grid 2048,2048 --col-balance --legs "" --no-e2e --no-cpu-baseline --fp16-leg none --steps 1 --warmup 1 > gpurun_out/ncu_det.log 2>&1; echo "ncu det rc=$?"
for f in r02_l2split_c5 r02_l2split_c4 r02_c5_fp16sr r02_det_slab_bal; do python tools/ncu_summary.py $R/$f.ncu-rep --json gpurun_out/$f.json > /dev/null; echo "$f $(wc -c < gpurun_out/$f.json)"; done
ncu -i $R/r02_l2split_c5.ncu-rep --page details --csv > gpurun_out/r02_l2split_c5_details.csv 2>/dev/null
ncu -i $R/r02_det_slab_bal.ncu-rep --page details --csv > gpurun_out/r02_det_slab_bal_details.csv 2>/dev/null
timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:hccmf -c 600 --csv --log-file gpurun_out/r02_launches_c5.csv python bench.py --steps 2 --warmup 1 --legs "" --no-e2e --no-cpu-baseline > gpurun_out/launch_run.log 2>&1; echo "launch list rc=$?"
du -sh gpurun_out
