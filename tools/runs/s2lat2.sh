B=paper_conf_icpp_huangylhbl21_b200/build
echo base; timeout 300 python tools/det_chain_latency.py 2>&1 | tail -1
for v in NO_DEPBAR SHFL_LEVELS_1 SHFL_LEVELS_3; do echo $v; HCCMF_LIB=$B/diag_$v.so timeout 300 python tools/det_chain_latency.py 2>&1 | tail -1; done
