"""Build profiles/rNN_traffic.json from one `ncu --set full` capture of a bench outer
iteration (the MTTKRP and ADMM launches of every mode, in launch order):
    python tools/traffic_json.py <report.ncu-rep> <workload> <out.json> [source-note]
Per kernel and mode: dram__bytes_read.sum + dram__bytes_write.sum, duration, and for
the ADMM the DMMA + FP64 pipe fractions (one shared FP64 datapath on B200)."""
import csv
import json
import os
import subprocess
import sys


def rows(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rs = list(csv.reader(out.splitlines()))
    hdr = rs[0]
    col = {h: i for i, h in enumerate(hdr)}
    unit = {h: rs[1][i] for i, h in enumerate(hdr)}
    return [dict(zip(hdr, r)) for r in rs[2:]], unit


def num(r, unit, k):
    v = float(r[k].replace(",", ""))
    u = unit[k]
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12,
             "ns": 1e-9, "us": 1e-6, "usecond": 1e-6, "msecond": 1e-3, "ms": 1e-3, "nsecond": 1e-9, "second": 1}.get(u, 1)
    return v * scale


def main(path, workload, out, note=""):
    rs, unit = rows(path)
    mt, ad = [], []
    for r in rs:
        name = r["Kernel Name"]
        d = {"kernel": name[:80],
             "bytes": num(r, unit, "dram__bytes_read.sum") + num(r, unit, "dram__bytes_write.sum"),
             "dram_read": num(r, unit, "dram__bytes_read.sum"), "dram_write": num(r, unit, "dram__bytes_write.sum"),
             "time_s": num(r, unit, "gpu__time_duration.sum")}
        if "k_admm_dmma" in name:
            d["dmma_pipe_pct"] = float(r["sm__pipe_tensor_subpipe_dmma_cycles_active.avg.pct_of_peak_sustained_active"])
            d["fp64_pipe_pct"] = float(r["sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active"])
            ad.append(d)
        elif "k_mttkrp" in name:
            mt.append(d)
    data = {}
    if os.path.exists(out):
        with open(out) as f:
            data = json.load(f)
    data["source"] = data.get("source") or out
    data.setdefault("how", "ncu --set full --clock-control none -k regex:'k_mttkrp_fast|k_admm_dmma' -s 24 -c 8 "
                           "python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e (one outer "
                           "iteration after 3 warm-up iterations); bytes = dram__bytes_read.sum + dram__bytes_write.sum")
    w = {"mttkrp": {"per_mode_bytes": [d["bytes"] for d in mt], "per_mode": mt},
         "admm": {"per_mode_bytes": [d["bytes"] for d in ad], "per_mode": ad}}
    tt = sum(d["time_s"] for d in ad)
    if tt > 0:
        w["admm"]["fp64_datapath_frac"] = sum((d["dmma_pipe_pct"] + d["fp64_pipe_pct"]) / 100 * d["time_s"]
                                             for d in ad) / tt
    if note:
        w["note"] = note
    data[workload] = w
    with open(out, "w") as f:
        json.dump(data, f, indent=1)
    print(json.dumps(w, indent=1)[:1500])


if __name__ == "__main__":
    main(*sys.argv[1:])
