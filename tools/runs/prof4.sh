R=/tmp/ncu; mkdir -p $R
M=gpu__time_duration.sum,lts__t_sector_hit_rate.pct,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_srcunit_tex_op_read_lookup_hit.sum,lts__t_sectors_srcunit_tex_op_write.sum,lts__t_sectors_srcunit_tex_op_write_lookup_hit.sum,lts__t_sectors_srcunit_tex_op_red.sum,lts__t_sectors_srcunit_tex_op_red_lookup_hit.sum,dram__bytes_read.sum,dram__bytes_write.sum
for c in c5 c3; do
timeout 1200 ncu --metrics $M --clock-control none -k 'regex:sgd_warp_kernel|stream_kernel|roundtrip_kernel' --csv --log-file gpurun_out/r02_l2split_${c}_min.csv python tools/l2_split.py --config $c > gpurun_out/ncu_min_$c.log 2>&1; echo "ncu min $c rc=$?"
done
timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none --kernel-name-base demangled -k regex:hccmf -c 2000 --csv --log-file gpurun_out/r02_launches_c5.csv python bench.py --steps 2 --warmup 1 --legs "" --no-e2e --no-cpu-baseline > gpurun_out/launch_run.log 2>&1; echo "launch list rc=$?"; wc -l gpurun_out/r02_launches_c5.csv
for g in 1,4 1,6 1,8 1,12; do
timeout 600 python bench.py --config c4 --grid $g --legs "" --no-e2e --no-cpu-baseline --fp16-leg none --steps 5 --warmup 2 > gpurun_out/c4g.json 2>/dev/null
python -c "import json,sys;d=json.load(open('gpurun_out/c4g.json'));print('c4 grid', sys.argv[1], round(d['ms_per_step'],2), round(d['value']/1e9,3), d['rmse']['test_per_epoch'][-1])" $g
done
bash tools/runs/ratio1.sh
