for i in 1 2 3 4 5 6; do timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "c2_full or c4_scaled" 2>&1 | tail -1; done
timeout 900 python tools/c4_stability.py --frac 0.05 --reps 40 --staleness 80 2>&1 | tail -1 | cut -c1-200
