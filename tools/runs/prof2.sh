# sanitizer logs (full workload), ncu captures, launch list, per-rank rates
for t in memcheck racecheck synccheck; do
  timeout 1500 compute-sanitizer --tool $t --print-limit 50 python tools/sanitize_workload.py > gpurun_out/r02_sanitizer_$t.log 2>&1
  echo "$t rc=$?"; tail -2 gpurun_out/r02_sanitizer_$t.log
done
timeout 1200 python tools/rank_rate.py --config c5 --G 1 2 4 8 2>&1 | tail -4
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"sgd_warp_kernel|stream_kernel|roundtrip_kernel" -f -o gpurun_out/r02_l2split_c5 python tools/l2_split.py --config c5 > gpurun_out/ncu_c5.log 2>&1; echo "ncu c5 rc=$?"; tail -2 gpurun_out/ncu_c5.log
timeout 1200 ncu --set full --clock-control none -k regex:"sgd_warp_kernel|stream_kernel|roundtrip_kernel" -f -o gpurun_out/r02_l2split_c4 python tools/l2_split.py --config c4 > gpurun_out/ncu_c4.log 2>&1; echo "ncu c4 rc=$?"
timeout 1200 ncu --set full --clock-control none -k regex:"sgd_warp_kernel" -c 2 -f -o gpurun_out/r02_c5_fp16sr python tools/l2_split.py --config c5 --storage fp16sr > gpurun_out/ncu_c5_16.log 2>&1; echo "ncu c5 fp16sr rc=$?"
timeout 1200 ncu --set full --clock-control none -k regex:"sgd_wave_slab" -c 1 -f -o gpurun_out/r02_det_slab_bal python bench.py --config c3 --sched det --grid 2048,2048 --col-balance --legs "" --no-e2e --no-cpu-baseline --fp16-leg none --steps 1 --warmup 1 > gpurun_out/ncu_det.log 2>&1; echo "ncu det rc=$?"
for f in gpurun_out/r02_l2split_c5 gpurun_out/r02_l2split_c4 gpurun_out/r02_c5_fp16sr gpurun_out/r02_det_slab_bal; do python tools/ncu_summary.py $f.ncu-rep --json $f.json > /dev/null; done
timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:hccmf -c 600 --csv --log-file gpurun_out/r02_launches_c5.csv python bench.py --steps 2 --warmup 1 --legs "" --no-e2e --no-cpu-baseline > gpurun_out/launch_run.log 2>&1; echo "launch list rc=$?"
