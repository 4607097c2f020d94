#!/usr/bin/env python
"""Summarise an ncu --set full report (+ optional launch list) into
profiles/<name>.md and merge the DRAM traffic per launch into
profiles/ncu_traffic.json (read by bench.py for the roofline `traffic`)."""
import csv
import io
import json
import os
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "lts__throughput.avg.pct_of_peak_sustained_elapsed",
        "l1tex__throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
        "launch__grid_size", "launch__block_size", "smsp__average_warp_latency_per_inst_issued.ratio",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed"]


TIME_TO_MS = {"s": 1e3, "ms": 1.0, "us": 1e-3, "usecond": 1e-3, "msecond": 1.0, "second": 1e3, "ns": 1e-6,
              "nsecond": 1e-6}


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units, vals = rows[0], rows[1], rows[2]
    return {h: (vals[i], units[i]) for i, h in enumerate(hdr)}


def main():
    rep, name, key = sys.argv[1], sys.argv[2], sys.argv[3]
    launches = sys.argv[4] if len(sys.argv) > 4 else None
    r = raw(rep)
    unit_scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}
    dram = sum(float(r[k][0]) * unit_scale.get(r[k][1], 1) for k in ("dram__bytes_read.sum", "dram__bytes_write.sum"))
    stalls = sorted(((float(v[0]), k) for k, v in r.items()
                     if k.startswith("smsp__pcsamp_warps_issue_stalled") and not k.endswith("not_issued")
                     and v[0].replace('.', '', 1).isdigit()), reverse=True)[:8]
    lines = [f"# {name}", "", f"ncu --set full capture `{os.path.basename(rep)}` (kernel `{r.get('Kernel Name', ('?',))[0]}`)", "",
             "| metric | value | unit |", "|---|---|---|"]
    for k in KEYS:
        if k in r:
            lines.append(f"| {k} | {r[k][0]} | {r[k][1]} |")
    lines += ["", f"DRAM bytes per launch (read + write): {dram:.4g}", "", "Top stall reasons (pc samples):", ""]
    tot = sum(s for s, _ in stalls) or 1
    for s, k in stalls:
        lines.append(f"- {k.replace('smsp__pcsamp_warps_issue_stalled_', '')}: {100 * s / tot:.1f}%")
    if launches and os.path.exists(launches):
        lines += ["", "Launch list (ncu --metrics gpu__time_duration.sum, cold-cache, serialised):", "",
                  "| kernel | launches | total ms | share |", "|---|---|---|---|"]
        agg = {}
        with open(launches) as f:
            body = [ln for ln in f if ln.startswith('"')]
        for row in csv.DictReader(io.StringIO("".join(body))):
            if row.get("Metric Name") != "gpu__time_duration.sum":
                continue
            k = row["Kernel Name"].split("(")[0]
            ns = float(row["Metric Value"].replace(",", "")) * (1e3 if row.get("Metric Unit") == "us" else
                                                                 1e6 if row.get("Metric Unit") == "ms" else 1)
            c, t = agg.get(k, (0, 0.0))
            agg[k] = (c + 1, t + ns)
        total = sum(t for _, t in agg.values()) or 1
        for k, (c, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
            lines.append(f"| `{k}` | {c} | {t / 1e6:.3f} | {100 * t / total:.1f}% |")
    os.makedirs("profiles", exist_ok=True)
    with open(os.path.join("profiles", name + ".md"), "w") as f:
        f.write("\n".join(lines) + "\n")
    tj = os.path.join("profiles", "ncu_traffic.json")
    d = json.load(open(tj)) if os.path.exists(tj) else {}
    d[key] = {"dram_bytes_per_launch": dram, "report": os.path.basename(rep), "summary": name + ".md",
              "kernel_ms": float(r["gpu__time_duration.sum"][0]) * TIME_TO_MS[r["gpu__time_duration.sum"][1]]}
    json.dump(d, open(tj, "w"), indent=1)
    print("\n".join(lines))


if __name__ == "__main__":
    main()
