"""Print an optsweep output file as a compact table: opts, median us (pass 0 / pass 1), p10, GFLOPS, engine, CTA."""
import json, sys
for f in sys.argv[1:]:
    print("==", f)
    res = {}
    for l in open(f):
        try:
            d = json.loads(l)
        except Exception:
            print("  ", l.strip()[:160])
            continue
        k = json.dumps(d["opts"], sort_keys=True)
        res.setdefault(k, []).append(d)
    for k, ds in res.items():
        print("  %-62s %s  p10 %s  %s GF  eng %s cta %s" % (k, " / ".join("%.2f" % d["t_us"] for d in ds),
              min(d["p10"] for d in ds), ds[0]["gflops"], ds[0]["engine"], ds[0]["cta"]))
