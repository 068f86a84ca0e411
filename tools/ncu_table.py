"""Summarise ncu --page raw CSV captures: duration, DRAM bytes and GB/s, L2 hit rate, warps active, top stalls.
usage: python tools/ncu_table.py profiles/r01_final_*_raw.csv"""
import csv, sys

STALL = "smsp__pcsamp_warps_issue_stalled_"
print("| capture | kernel | µs | DRAM read+write MB | DRAM GB/s | L2 hit % | warps active % | top stalls (share of samples) |")
print("|---|---|---|---|---|---|---|---|")
for f in sys.argv[1:]:
    rows = list(csv.reader(open(f)))
    h, u, v = rows[0], rows[1], rows[2]
    g = lambda k: v[h.index(k)].replace(",", "") if k in h else None
    unit = lambda k: u[h.index(k)] if k in h else ""
    dur = float(g("gpu__time_duration.sum"))
    dur_us = dur * {"ms": 1e3, "us": 1.0, "ns": 1e-3, "usecond": 1.0, "msecond": 1e3, "nsecond": 1e-3}.get(unit("gpu__time_duration.sum"), 1.0)
    mb = lambda k: float(g(k)) * {"Mbyte": 1.0, "Kbyte": 1e-3, "Gbyte": 1e3, "byte": 1e-6}.get(unit(k), 1.0)
    dram = mb("dram__bytes_read.sum") + mb("dram__bytes_write.sum")
    st = {k[len(STALL):]: float(g(k)) for k in h if k.startswith(STALL) and not k.endswith("not_issued")}
    tot = sum(st.values()) or 1.0
    top = ", ".join("%s %.0f%%" % (k, 100 * x / tot) for k, x in sorted(st.items(), key=lambda kv: -kv[1])[:3])
    name = g("Kernel Name")
    name = name[name.find(" ") + 1:name.find("(")] if "(" in name else name
    print("| %s | `%s` | %.1f | %.1f | %.0f | %.1f | %.1f | %s |" % (f.split("/")[-1], name, dur_us, dram, dram / dur_us * 1e3,
          float(g("lts__t_sector_hit_rate.pct")), float(g("sm__warps_active.avg.pct_of_peak_sustained_active")), top))
