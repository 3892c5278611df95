timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/gputest_last.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/gputest_last.log
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
