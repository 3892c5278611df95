timeout 1500 python tools/c4_stability.py --frac 0.05 --reps 8 --staleness 80 60 40 --heavy 1024 -1 2>&1 | tail -7
