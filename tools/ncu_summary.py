"""Summarise an ncu --set full report: per launch duration, DRAM traffic and
throughput, occupancy, issue activity and the top warp-stall reasons.

    python tools/ncu_summary.py report.ncu-rep [--traffic-json profiles/ncu_traffic.json --config C5
                                                 --stage sort_pass_mid --scale 5.0]

--traffic-json records dram bytes per launch (x --scale, for a capture taken at a
smaller size than the bench) under traffic[config][stage] for bench.py's roofline."""
import argparse
import csv
import io
import json
import os
import subprocess

WANT = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "launch__grid_size", "launch__block_size", "smsp__inst_executed.sum"]
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12,
         "nsecond": 1e-6, "usecond": 1e-3, "msecond": 1.0, "second": 1e3, "ns": 1e-6, "us": 1e-3, "ms": 1.0, "s": 1e3}


def rows(rep):
    out = subprocess.check_output(["ncu", "-i", rep, "--page", "raw", "--csv"], stderr=subprocess.DEVNULL).decode()
    r = list(csv.reader(io.StringIO(out)))
    return r[0], r[1], r[2:]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("rep")
    ap.add_argument("--traffic-json")
    ap.add_argument("--config", default="C5")
    ap.add_argument("--stage")
    ap.add_argument("--scale", type=float, default=1.0)
    a = ap.parse_args()
    hdr, units, data = rows(a.rep)
    recs = []
    for r in data:
        d = {"kernel": r[hdr.index("Kernel Name")].split("(")[0]}
        for w in WANT:
            if w in hdr:
                i = hdr.index(w)
                v = r[i].replace(",", "")
                try:
                    v = float(v) * SCALE.get(units[i], 1)
                except ValueError:
                    pass
                d[w] = v
        stalls = []
        for i, h in enumerate(hdr):
            if "pcsamp_warps_issue_stalled" in h and "not_issued" not in h:
                try:
                    stalls.append((float(r[i].replace(",", "")), h.replace("smsp__pcsamp_warps_issue_stalled_", "")))
                except ValueError:
                    pass
        tot = sum(s for s, _ in stalls) or 1.0
        d["top_stalls"] = [f"{n} {100 * s / tot:.0f}%" for s, n in sorted(stalls, reverse=True)[:5]]
        recs.append(d)
    for d in recs:
        traffic = d.get("dram__bytes_read.sum", 0) + d.get("dram__bytes_write.sum", 0)
        print(f"{d['kernel']}: {d.get('gpu__time_duration.sum', 0):.3f} ms, grid {d.get('launch__grid_size')}, "
              f"dram {traffic / 1e9:.3f} GB ({d.get('gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed', 0):.1f}% "
              f"of peak), sm {d.get('sm__throughput.avg.pct_of_peak_sustained_elapsed', 0):.1f}%, issue "
              f"{d.get('smsp__issue_active.avg.pct_of_peak_sustained_active', 0):.1f}%, warps active "
              f"{d.get('sm__warps_active.avg.pct_of_peak_sustained_active', 0):.1f}%, regs "
              f"{d.get('launch__registers_per_thread')}, stalls {', '.join(d['top_stalls'])}")
    if a.traffic_json and a.stage and recs:
        t = {}
        if os.path.exists(a.traffic_json):
            t = json.load(open(a.traffic_json))
        vals = [(d.get("dram__bytes_read.sum", 0) + d.get("dram__bytes_write.sum", 0)) * a.scale for d in recs]
        t.setdefault(a.config, {})[a.stage] = sum(vals) / len(vals)
        json.dump(t, open(a.traffic_json, "w"), indent=1)


if __name__ == "__main__":
    main()
