mkdir -p gpurun_out/tl
for w in C3 C4cc C2; do timeout 300 python tools/timeline.py $w paper_conf_hpdc_khorasanivgb14_b200/variant_TL.so gpurun_out/tl/$w.json > /dev/null 2>gpurun_out/tl/$w.err; echo "$w rc=$?"; done
python - <<'PY'
import json
for w in ("C3","C4cc","C2"):
    try: d=json.load(open(f"gpurun_out/tl/{w}.json"))["timeline"]
    except Exception as e: print(w, e); continue
    print(w, {k:(v["median_us"] if isinstance(v,dict) else v) for k,v in d.items()})
PY
