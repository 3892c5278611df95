HCCMF_PROFILE=1 timeout 900 python tools/e2e_profile.py --config c5 --epochs 3 > gpurun_out/e2e_c5.log 2>&1; echo rc=$?
tail -30 gpurun_out/e2e_c5.log
