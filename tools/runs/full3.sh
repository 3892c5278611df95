export HCCMF_BAND_REPORT=$PWD/gpurun_out/band_report3.jsonl
rm -f $HCCMF_BAND_REPORT
timeout 3000 python -m pytest tests -m gpu -q --durations=10 -k "not sanitizer" > gpurun_out/gputest_full3.log 2>&1
echo "pytest rc=$?"; tail -25 gpurun_out/gputest_full3.log
timeout 900 python tools/rank_rate.py --config c5 --G 1 2 4 8 2>&1 | tail -4
timeout 900 python tools/rank_rate.py --config c3 --G 1 2 4 8 2>&1 | tail -4
run() { timeout 600 python bench.py --config c4 --legs "" --no-e2e --no-cpu-baseline --fp16-leg none --steps 6 --warmup 2 "$@" > gpurun_out/c4n.json 2>gpurun_out/c4n.err; python -c "import json,sys;d=json.load(open('gpurun_out/c4n.json'));print(sys.argv[1:], round(d['ms_per_step'],2), round(d['value']/1e9,3), [round(x,3) for x in d['rmse']['test_per_epoch']])" "$@"; }
run --grid 1,4
run --grid 1,8
