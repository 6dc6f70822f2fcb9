import json,sys
for line in sys.stdin:
    line=line.strip()
    if not line.startswith('{'): 
        continue
    d=json.loads(line)
    print(d["config"]["workload"].split(' (')[0], "ms=%.1f"%d["ms_per_step"], {k:round(v,1) for k,v in d["phases_ms"].items()}, "frac=%.3f"%d["roofline"]["frac"], "n_ext=%d"%d["config"]["n_ext"])
