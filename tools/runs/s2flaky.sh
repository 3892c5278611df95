for i in 1 2; do
export HCCMF_BAND_REPORT=$PWD/gpurun_out/band_report_flakyb$i.jsonl
rm -f $HCCMF_BAND_REPORT
timeout 2400 python -m pytest tests -m gpu -q -p no:randomly > gpurun_out/gputest_flakyb$i.log 2>&1
echo "pytest $i rc=$?"; tail -3 gpurun_out/gputest_flakyb$i.log
done
