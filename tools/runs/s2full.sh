# session 2 of round 2: whole GPU suite + the default bench line (the driver's command)
export HCCMF_BAND_REPORT=$PWD/gpurun_out/band_report_s2.jsonl
rm -f $HCCMF_BAND_REPORT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 2400 python -m pytest tests -m gpu -q --durations=15 > gpurun_out/gputest_s2.log 2>&1
echo "pytest rc=$?"; tail -22 gpurun_out/gputest_s2.log
timeout 1500 python bench.py > gpurun_out/bench_s2.json 2> gpurun_out/bench_s2.err
echo "bench rc=$?"; tail -3 gpurun_out/bench_s2.err; cat gpurun_out/bench_s2.json
