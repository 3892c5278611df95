# C3 G = 1 attribution of the steep-phase gap (heavy-first order vs concurrency) and C2 caps
S="timeout 900 python tools/ring_band_sweep.py --config c3 --epochs 10 --single"
$S > gpurun_out/sw2_c3.log 2>&1
$S --opt heavy_first=-1 >> gpurun_out/sw2_c3.log 2>&1
$S --opt conflict_ratio=6 >> gpurun_out/sw2_c3.log 2>&1
$S --opt conflict_ratio=6 --opt heavy_first=-1 >> gpurun_out/sw2_c3.log 2>&1
$S --opt hogwild_warps=1480 --opt heavy_first=-1 >> gpurun_out/sw2_c3.log 2>&1
S="timeout 900 python tools/ring_band_sweep.py --config c2 --epochs 20 --single"
$S --opt heavy_first=-1 > gpurun_out/sw2_c2.log 2>&1
$S --opt conflict_ratio=6 >> gpurun_out/sw2_c2.log 2>&1
$S --opt conflict_ratio=8 >> gpurun_out/sw2_c2.log 2>&1
$S --opt conflict_ratio=12 >> gpurun_out/sw2_c2.log 2>&1
$S --opt conflict_ratio=8 --opt heavy_first=-1 >> gpurun_out/sw2_c2.log 2>&1
python - <<'PY'
import json
for l in open("gpurun_out/ring_band_sweep.jsonl"):
    d = json.loads(l)
    print(d["config"], d["G"], d["Bc"], d["opts"], "maxgap %.4f final %.4f" % (d["max_gap_e2plus"], d["final_gap"]), d["gap"][:6])
PY
