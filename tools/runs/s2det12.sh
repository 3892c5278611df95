timeout 900 python -m pytest tests/test_gpu_full_size.py -m gpu -q -k "det" > gpurun_out/det12_test.log 2>&1
echo "pytest rc=$?"; tail -2 gpurun_out/det12_test.log
R=/tmp/ncu; mkdir -p $R
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:sgd_wave_slab -c 1 -f -o $R/det python bench.py --config c3 --sched det --grid 1536,1536 --col-balance --legs "" --no-e2e --no-cpu-baseline --fp16-leg none --steps 1 --warmup 1 > gpurun_out/ncu_det12.log 2>&1; echo "ncu det rc=$?"
python tools/ncu_summary.py $R/det.ncu-rep --json gpurun_out/r02_ncu_det_s2_summary.json | tail -3
