for nw in 4 2; do
python paper_conf_icpp_huangylhbl21_b200/_build.py -DHCCMF_DIAG_TRACE -DHCCMF_CHAIN_NW=$nw --out=/tmp/libtrace$nw.so > /dev/null 2>&1
for B in 1024 2048; do
HCCMF_LIB=/tmp/libtrace$nw.so timeout 900 python tools/trace_det_wave.py --wave 3 --B $B --nobuild 2>&1 | tail -1 | sed "s/^/NW=$nw /"
done; done
