"""Summarise ncu reports into profiles/ (JSON + markdown rows).

python tools/ncu_summary.py <report.ncu-rep | full_raw.csv> --variant site --local 32,32,32,32 [--out profiles/ncu_summary.json]
Reads `ncu -i ... --page raw --csv`, keeps the metrics the roofline uses, and merges one entry
per (variant, local_dims) into the JSON file bench.py reads for `roofline.traffic`.
"""
import argparse
import csv
import io
import json
import os
import subprocess

KEEP = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "dram__bytes.sum.per_second",
        "lts__t_sector_hit_rate.pct", "l1tex__t_sector_hit_rate.pct", "launch__registers_per_thread",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "sm__cycles_active.avg", "gpc__cycles_elapsed.max",
        "launch__grid_size", "launch__block_size", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "launch__waves_per_multiprocessor"]
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12,
         "us": 1e-6, "ms": 1e-3, "ns": 1e-9, "s": 1}


def rows(rep):
    if rep.endswith(".csv"):  # an exported `--page raw --csv` (gpu_ncu.sh full_raw.csv)
        with open(rep) as f:
            out = f.read()
    else:
        out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True,
                             check=True).stdout
    r = list(csv.reader(io.StringIO(out)))
    hdr, units = r[0], r[1]
    res = []
    for row in r[2:]:
        d = {"kernel": row[hdr.index("Kernel Name")]}
        for k in KEEP:
            if k in hdr:
                i = hdr.index(k)
                v = row[i].replace(",", "")
                try:
                    v = float(v) * SCALE.get(units[i], 1)
                except ValueError:
                    pass
                d[k] = v
        res.append(d)
    return res


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("report")
    ap.add_argument("--variant", required=True)
    ap.add_argument("--local", default="32,32,32,32")
    ap.add_argument("--out", default=os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                                  "profiles", "ncu_summary.json"))
    ap.add_argument("--note", default="")
    ap.add_argument("--bytes-per-site", type=int, default=2400, help="algorithmic bytes per target site")
    a = ap.parse_args()
    rs = rows(a.report)
    launches = [r for r in rs if "dslash" in r["kernel"]]
    dram = [r["dram__bytes_read.sum"] + r["dram__bytes_write.sum"] for r in launches]
    local = [int(v) for v in a.local.split(",")]
    vh = local[0] * local[1] * local[2] * local[3] // 2
    entry = {"variant": a.variant, "local_dims": local, "report": os.path.basename(a.report),
             "kernel": launches[0]["kernel"], "launches": len(launches),
             "dram_bytes_per_launch": int(sum(dram) / len(dram)),
             "algorithmic_bytes_per_launch": a.bytes_per_site * vh,
             "duration_us": [round(r["gpu__time_duration.sum"] * 1e6, 2) for r in launches],
             "metrics": launches[-1], "note": a.note}
    try:
        with open(a.out) as f:
            s = json.load(f)
    except Exception:
        s = {"about": "ncu --set full --clock-control none captures (cold cache, serialised); "
                      "dram_bytes_per_launch feeds bench.py roofline.traffic", "kernels": []}
    s["kernels"] = [e for e in s["kernels"] if not (e["variant"] == a.variant and e["local_dims"] == local)]
    s["kernels"].append(entry)
    with open(a.out, "w") as f:
        json.dump(s, f, indent=1)
    print(json.dumps({k: entry[k] for k in ("variant", "kernel", "dram_bytes_per_launch",
                                            "algorithmic_bytes_per_launch", "duration_us")}))


if __name__ == "__main__":
    main()
