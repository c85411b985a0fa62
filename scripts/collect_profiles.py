"""Turn gpurun_out/ ncu reports and bench JSONs into committed summaries under profiles/.

  python scripts/collect_profiles.py --round r1

* profiles/<round>_ncu_<config>_<policy>.txt : key metrics of one `ncu --set full` capture of k_spmm
* profiles/ncu_traffic.json                   : DRAM bytes per launch (read by bench.py as roofline.traffic)
* profiles/<round>_bench_<config>.json        : the bench JSON line(s)
* profiles/<round>_launches.txt               : per-kernel share of the launch list (ncu gpu__time_duration)
"""
import argparse
import csv
import glob
import io
import json
import os
import re
import shutil
import subprocess

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "gpurun_out")
PROF = os.path.join(ROOT, "profiles")
KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
        "l1tex__t_sector_hit_rate.pct", "derived__lts__lts2xbar_bytes.sum.per_second",
        "l1tex__m_xbar2l1tex_read_bytes.sum", "lts__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "smsp__inst_executed.sum", "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
        "sm__cycles_elapsed.avg.per_second", "smsp__average_warp_latency_issue_stalled_long_scoreboard"]


def ncu_raw(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    if len(rows) < 3:
        return None
    h, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = {"kernel": r[h.index("Kernel Name")] if "Kernel Name" in h else ""}
        for k in KEYS:
            if k in h:
                d[k] = (r[h.index(k)], units[h.index(k)])
        res.append(d)
    return res


def to_bytes(v, u):
    f = float(v.replace(",", ""))
    return f * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}.get(u, 1)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--round", default="r1")
    args = ap.parse_args()
    os.makedirs(PROF, exist_ok=True)
    traffic_path = os.path.join(PROF, "ncu_traffic.json")
    traffic = json.load(open(traffic_path)) if os.path.exists(traffic_path) else {}
    for rep in sorted(glob.glob(os.path.join(OUT, "prof_*.ncu-rep"))):
        m = re.match(r"prof_([a-z0-9]+)_(.+)\.ncu-rep", os.path.basename(rep))
        if not m:
            continue
        cfg, pol = m.groups()
        res = ncu_raw(rep)
        if not res:
            continue
        d = res[0]
        with open(os.path.join(PROF, f"{args.round}_ncu_{cfg}_{pol}.txt"), "w") as f:
            f.write(f"# ncu --set full --clock-control none, one launch of {d['kernel']}\n")
            f.write(f"# python scripts/profile_spmm.py --config {cfg} --policy {pol}\n")
            for k in KEYS:
                if k in d:
                    f.write(f"{k} {d[k][0]} {d[k][1]}\n")
        rd = to_bytes(*d["dram__bytes_read.sum"]) + to_bytes(*d["dram__bytes_write.sum"])
        traffic[f"{cfg}/{pol}"] = {"dram_bytes_per_launch": rd, "kernel": d["kernel"].split("(")[0],
                                   "duration": d["gpu__time_duration.sum"], "round": args.round}
    # raw-page CSV exports (scripts/gpu_prof_env.sh: prof_<config>_<policy>_<tag>.raw.csv; tag "def" = defaults)
    for rc in sorted(glob.glob(os.path.join(OUT, "prof_*.raw.csv"))):
        m = re.match(r"prof_([a-z0-9]+)_(.+)_([a-z0-9]+)\.raw\.csv", os.path.basename(rc))
        if not m:
            continue
        cfg, pol, tag = m.groups()
        rows = list(csv.reader(open(rc)))
        if len(rows) < 3:
            continue
        h, units, r = rows[0], rows[1], rows[2]
        d = {"kernel": r[h.index("Kernel Name")] if "Kernel Name" in h else ""}
        for k in KEYS:
            if k in h:
                d[k] = (r[h.index(k)], units[h.index(k)])
        name = f"{cfg}_{pol}" + ("" if tag == "def" else f"_{tag}")
        with open(os.path.join(PROF, f"{args.round}_ncu_{name}.txt"), "w") as f:
            f.write(f"# ncu --set full --clock-control none, one launch of {d['kernel']}\n")
            f.write(f"# python scripts/profile_spmm.py --config {cfg} --policy {pol} (env tag {tag})\n")
            for k in KEYS:
                if k in d:
                    f.write(f"{k} {d[k][0]} {d[k][1]}\n")
        if tag == "def":
            rd = to_bytes(*d["dram__bytes_read.sum"]) + to_bytes(*d["dram__bytes_write.sum"])
            traffic[f"{cfg}/{pol}"] = {"dram_bytes_per_launch": rd, "kernel": d["kernel"].split("(")[0],
                                       "duration": d["gpu__time_duration.sum"], "round": args.round}
    # one process, one k_spmm launch per policy (scripts/profile_policies.py): prof_multi_<config>.raw.csv rows in
    # the order of prof_multi_<config>.policies
    for rc in sorted(glob.glob(os.path.join(OUT, "prof_multi_*.raw.csv"))):
        cfg = re.match(r"prof_multi_([a-z0-9]+)\.raw\.csv", os.path.basename(rc)).group(1)
        pols = [l.strip() for l in open(os.path.join(OUT, f"prof_multi_{cfg}.policies")) if l.strip()]
        rows = list(csv.reader(open(rc)))
        if len(rows) < 3:
            continue
        h, units = rows[0], rows[1]
        for pol, r in zip(pols, rows[2:]):
            d = {"kernel": r[h.index("Kernel Name")] if "Kernel Name" in h else ""}
            for k in KEYS:
                if k in h:
                    d[k] = (r[h.index(k)], units[h.index(k)])
            with open(os.path.join(PROF, f"{args.round}_ncu_{cfg}_{pol}.txt"), "w") as f:
                f.write(f"# ncu --set full --clock-control none, one launch of {d['kernel']}\n")
                f.write(f"# python scripts/profile_policies.py --config {cfg} (launch of policy {pol})\n")
                for k in KEYS:
                    if k in d:
                        f.write(f"{k} {d[k][0]} {d[k][1]}\n")
            rd = to_bytes(*d["dram__bytes_read.sum"]) + to_bytes(*d["dram__bytes_write.sum"])
            traffic[f"{cfg}/{pol}"] = {"dram_bytes_per_launch": rd, "kernel": d["kernel"].split("(")[0],
                                       "duration": d["gpu__time_duration.sum"], "round": args.round}
    with open(traffic_path, "w") as f:
        json.dump(traffic, f, indent=1, sort_keys=True)
    for bj in sorted(glob.glob(os.path.join(OUT, "bench*.json"))):
        shutil.copy(bj, os.path.join(PROF, f"{args.round}_{os.path.basename(bj)}"))
    lc = os.path.join(OUT, "launches.csv")
    if os.path.exists(lc):
        txt = open(lc).read()
        start = txt.find('"ID"')
        rows = list(csv.reader(io.StringIO(txt[start:]))) if start >= 0 else []
        if rows:
            h = rows[0]
            ki, vi = h.index("Kernel Name"), h.index("Metric Value")
            tot = {}
            for r in rows[1:]:
                name = re.sub(r"\(.*", "", r[ki])
                tot[name] = tot.get(name, 0.0) + float(r[vi].replace(",", ""))
            s = sum(tot.values())
            with open(os.path.join(PROF, f"{args.round}_launches.txt"), "w") as f:
                f.write("# ncu --metrics gpu__time_duration.sum --clock-control none: share of device time per kernel\n")
                for k, v in sorted(tot.items(), key=lambda kv: -kv[1]):
                    f.write(f"{100 * v / s:6.2f}%  {v:14.0f}  {k}\n")
            shutil.copy(lc, os.path.join(PROF, f"{args.round}_launches.csv"))
    print("profiles updated")


if __name__ == "__main__":
    main()
