export HCCMF_BAND_REPORT=$PWD/gpurun_out/band_report.jsonl
rm -f $HCCMF_BAND_REPORT
timeout 2400 python -m pytest tests -m gpu -q -x --durations=25 > gpurun_out/gputest_full1.log 2>&1
echo "pytest rc=$?"
tail -40 gpurun_out/gputest_full1.log
timeout 1200 python bench.py > gpurun_out/bench_full1.json 2> gpurun_out/bench_full1.err
echo "bench rc=$?"
tail -c 3000 gpurun_out/bench_full1.json; tail -20 gpurun_out/bench_full1.err
