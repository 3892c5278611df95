rm -f gpurun_out/ring_band_sweep.jsonl
for cr in 2 1; do
for G in 4 8; do
timeout 600 python tools/ring_band_sweep.py --config c3 --epochs 10 --G $G --Bc $G --opt conflict_ratio=$cr > /dev/null 2>&1
timeout 600 python tools/ring_band_sweep.py --config c2 --epochs 20 --G $G --Bc $G --opt conflict_ratio=$cr > /dev/null 2>&1
done; done
python - <<'PY'
import json
for l in open("gpurun_out/ring_band_sweep.jsonl"):
    d = json.loads(l)
    print(d["config"], d["G"], d["Bc"], d["opts"], "maxgap %.4f final %.4f" % (d["max_gap_e2plus"], d["final_gap"]))
PY
for cr in 2 1; do timeout 900 python tools/rank_rate.py --config c3 --G 2 4 8 --opt conflict_ratio=$cr 2>&1 | tail -3; done
