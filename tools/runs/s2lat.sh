timeout 600 python tools/det_chain_latency.py --ratings 2000000 2>&1 | tail -1
timeout 600 python tools/det_chain_latency.py --ratings 2000000 --per-user 8 2>&1 | tail -1
