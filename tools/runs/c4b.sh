export HCCMF_BAND_REPORT=$PWD/gpurun_out/band_report5.jsonl
rm -f $HCCMF_BAND_REPORT
timeout 1800 python -m pytest tests -m gpu -q -k "c4_scaled or partition" > gpurun_out/gputest_5.log 2>&1
echo "pytest rc=$?"; tail -3 gpurun_out/gputest_5.log
HCCMF_PROFILE=1 timeout 900 python tools/e2e_profile.py --config c5 --epochs 3 2>&1 | grep -v "^\[hccmf\]   " | tail -30
