timeout 900 python tools/epoch_times.py --config c5 --epochs 6 2>&1 | tail -2
timeout 900 python tools/epoch_times.py --config c3 --epochs 6 2>&1 | tail -2
