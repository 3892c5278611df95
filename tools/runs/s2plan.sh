export HCCMF_BAND_REPORT=$PWD/gpurun_out/band_report_plan.jsonl
rm -f $HCCMF_BAND_REPORT
timeout 2400 python -m pytest tests -m gpu -q -x --durations=5 > gpurun_out/gputest_plan.log 2>&1
echo "pytest rc=$?"; tail -12 gpurun_out/gputest_plan.log
timeout 900 python tools/epoch_times.py --config c5 --epochs 4 2>&1 | tail -1
HCCMF_PROFILE=1 timeout 900 python tools/e2e_profile.py --config c5 --epochs 3 > gpurun_out/e2e_c5b.log 2>&1; grep 'rep\|tasks' gpurun_out/e2e_c5b.log
