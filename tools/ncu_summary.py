"""Summarise ncu --set full captures (.ncu-rep) into a markdown table + raw csv extracts.

usage: python tools/ncu_summary.py OUT.md REP [REP ...]
For each report: kernel, duration, DRAM read / write bytes and throughput, L2 hit rate, warps active,
registers, and the top warp-stall reasons (per issue-active cycle).  Needs the ncu CLI (no GPU)."""
import csv
import io
import os
import subprocess
import sys

KEYS = {
    "gpu__time_duration.sum": "duration",
    "dram__bytes_read.sum": "dram_read",
    "dram__bytes_write.sum": "dram_write",
    "dram__bytes.sum.per_second": "dram_bw",
    "lts__t_sector_hit_rate.pct": "l2_hit_%",
    "sm__warps_active.avg.pct_of_peak_sustained_active": "warps_active_%",
    "launch__registers_per_thread": "regs",
    "launch__grid_size": "grid",
    "launch__block_size": "block",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed": "sm_thru_%",
    "lts__throughput.avg.pct_of_peak_sustained_elapsed": "l2_thru_%",
}
STALL = "smsp__average_warps_issue_stalled_"


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    return [dict(zip(hdr, r)) for r in rows[2:]], dict(zip(hdr, units))


def main():
    out_md, reps = sys.argv[1], sys.argv[2:]
    lines = ["| capture | kernel | " + " | ".join(KEYS.values()) + " | top stalls (per issue) |",
             "|" + "---|" * (len(KEYS) + 3)]
    for rep in reps:
        launches, units = raw(rep)
        for L in launches:
            vals = []
            for k in KEYS:
                v = L.get(k, "")
                u = units.get(k, "")
                vals.append(f"{v} {u}".strip())
            stalls = sorted(((float(L[k].replace(",", "")), k[len(STALL):].replace("_per_issue_active.ratio", ""))
                             for k in L if k.startswith(STALL) and k.endswith("_per_issue_active.ratio")
                             and L[k] not in ("", "n/a")), reverse=True)[:4]
            st = ", ".join(f"{n} {v:.2f}" for v, n in stalls)
            lines.append(f"| {os.path.basename(rep)} | {L.get('Kernel Name', '')[:40]} | " + " | ".join(vals) +
                         f" | {st} |")
        base = os.path.splitext(rep)[0]
        subprocess.run(f"ncu -i {rep} --page raw --csv > {base}_raw.csv", shell=True)
    open(out_md, "w").write("\n".join(lines) + "\n")
    print("\n".join(lines))


if __name__ == "__main__":
    main()
