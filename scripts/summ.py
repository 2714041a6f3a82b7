import json, sys
for path in sys.argv[1:]:
    for l in open(path):
        if not l.startswith("{"): continue
        d = json.loads(l)
        if "metric" in d:
            ms = d.get("multislice") or {}
            print(path, round(d["value"], 1), "fwd", round(d["spmv"]["fwd_ms"], 4), "back", round(d["spmv"]["back_ms"], 4), "frac", round(d["roofline"]["frac"], 3), "ms", ms.get("value"), ms.get("fwd_ms"), ms.get("back_ms"))
        elif "P" in d:
            print(path, d["P"], round(d.get("max_fwd_us", d["fwd_us"][0])), round(d.get("max_back_us", d["back_us"][0])), round(d["max_us"]), round(d["E_spmv"], 3))
