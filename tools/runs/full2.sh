export HCCMF_BAND_REPORT=$PWD/gpurun_out/band_report2.jsonl
rm -f $HCCMF_BAND_REPORT
timeout 3000 python -m pytest tests -m gpu -q --durations=30 > gpurun_out/gputest_full2.log 2>&1
echo "pytest rc=$?"; tail -45 gpurun_out/gputest_full2.log
timeout 1500 python bench.py > gpurun_out/bench_full2.json 2> gpurun_out/bench_full2.err
echo "bench rc=$?"; tail -c 600 gpurun_out/bench_full2.json; tail -5 gpurun_out/bench_full2.err
timeout 600 python tools/ring_timeline.py --config c3 --G 4 --Bc 8 2>&1 | tail -1
timeout 600 python tools/ring_timeline.py --config c3 --G 8 --Bc 8 2>&1 | tail -1
timeout 900 python tools/ring_timeline.py --config c5 --G 4 --Bc 4 2>&1 | tail -1
timeout 900 python tools/rank_rate.py --config c5 --G 1 2 4 8 2>&1 | tail -4
timeout 900 python tools/rank_rate.py --config c3 --G 1 2 4 8 2>&1 | tail -4
