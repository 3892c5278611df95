timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "column_phases" 2>&1 | tail -5
cat > /tmp/c4small.py <<'PY'
import sys, numpy as np
sys.path.insert(0, '.')
import synth, paper_conf_icpp_huangylhbl21_b200 as pkg
for frac in (0.05, 0.2):
    cfg = synth.scaled(synth.CONFIGS["c4"], frac)
    (u, v, r), (tu, tv, tr) = synth.make(cfg)
    for Bc, W in ((1, 4736), (4, 4736), (8, 4736), (8, 2368), (16, 4736)):
        m = pkg.Model(cfg.m, cfg.n, 128, cfg.gamma, cfg.lam)
        m.set_option("hogwild_warps", W)
        m.load(u, v, r); m.partition(1, (1, Bc), seed=cfg.seed); m.init(1)
        c = [m.rmse(tu, tv, tr)]
        for _ in range(3):
            m.train_epoch("hogwild", "none"); c.append(m.rmse(tu, tv, tr))
        print(frac, Bc, W, [round(x, 3) for x in c], flush=True)
        m.close()
PY
timeout 900 python /tmp/c4small.py
