set -x
timeout 300 python -m pytest tests/test_gpu_loopback.py -x -q -k "every_data_plane" > gpurun_out/lb2.log 2>&1; tail -3 gpurun_out/lb2.log
S="timeout 600 python tools/ring_band_sweep.py --config c2 --epochs 20"
$S --single > gpurun_out/sw_single.log 2>&1
$S --single --opt prefetch_depth=1 >> gpurun_out/sw_single.log 2>&1
$S --G 2 --Bc 2 >> gpurun_out/sw_g2.log 2>&1
$S --G 2 --Bc 2 --opt prefetch_depth=1 >> gpurun_out/sw_g2.log 2>&1
$S --G 2 --Bc 2 --opt conflict_ratio=6 >> gpurun_out/sw_g2.log 2>&1
$S --G 2 --Bc 2 --opt conflict_ratio=6 --opt prefetch_depth=1 >> gpurun_out/sw_g2.log 2>&1
$S --G 4 --Bc 4 >> gpurun_out/sw_g4.log 2>&1
$S --G 4 --Bc 4 --opt prefetch_depth=1 >> gpurun_out/sw_g4.log 2>&1
$S --G 8 --Bc 8 >> gpurun_out/sw_g8.log 2>&1
$S --G 8 --Bc 8 --opt prefetch_depth=1 >> gpurun_out/sw_g8.log 2>&1
grep -h max_gap gpurun_out/sw_*.log | python -c "
import sys,json
for l in sys.stdin:
    d=json.loads(l); print(d['G'],d['Bc'],d['opts'],'maxgap %.4f final %.4f'%(d['max_gap_e2plus'],d['final_gap']))"
