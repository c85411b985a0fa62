"""Summarise the locality-recovery run (scripts/gpu_locality.sh): per config and policy, the bench time, GFLOP/s,
step roofline fraction, LRU-model ceiling, and the ncu L2 / DRAM counters of one k_spmm launch, with the derived B
hit rate of SURVEY.md §5: 1 - (DRAM read bytes - A bytes - rowptr bytes) / (4 nnz K).

  python scripts/loc_table.py gpurun_out [--md]
"""
import csv
import json
import os
import sys


def ncu_metrics(path):
    if not os.path.exists(path):
        return None
    rows = [r for r in csv.reader(open(path)) if len(r) > 10]
    if not rows:
        return None
    h = rows[0]
    mi, ui, vi = h.index("Metric Name"), h.index("Metric Unit"), h.index("Metric Value")
    out = {}
    for r in rows[1:]:
        v = float(r[vi].replace(",", ""))
        u = r[ui]
        v *= {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12, "nsecond": 1e-9,
              "usecond": 1e-6, "msecond": 1e-3, "second": 1}.get(u, 1)
        out[r[mi]] = v
    return out


def main():
    d = sys.argv[1] if len(sys.argv) > 1 else "gpurun_out"
    md = "--md" in sys.argv
    res = {}
    for c in ("c3sh", "c3rl", "c5sh", "c5rl"):
        p = os.path.join(d, f"loc_{c}.json")
        if not os.path.exists(p):
            continue
        line = json.loads(open(p).read().strip().splitlines()[-1])
        nnz, K, M = line["config"]["nnz"], line["config"]["K"], line["config"]["M"]
        res[c] = {"nnz": nnz, "K": K, "M": M, "policies": {}}
        for pol, r in line["policies"].items():
            e = {"ms": r["ms"], "gflops": r["gflops"], "frac": r["roofline_frac"], "build_ms": r["build_ms"],
                 "speedup_vs_identity": r["speedup_vs_identity"],
                 "lru_ceiling": r.get("lru_model", {}).get("ceiling_frac"),
                 "lru_b_row_misses": r.get("lru_model", {}).get("b_row_misses")}
            m = ncu_metrics(os.path.join(d, f"loc_ncu_{c}_{pol}.csv"))
            if m:
                rd = m.get("dram__bytes_read.sum", 0)
                hit = m.get("lts__t_sectors_srcunit_tex_op_read_lookup_hit.sum", 0)
                miss = m.get("lts__t_sectors_srcunit_tex_op_read_lookup_miss.sum", 0)
                e.update({"ncu_ms": 1e3 * m.get("gpu__time_duration.sum", 0), "dram_read_GB": rd / 1e9,
                          "dram_write_GB": m.get("dram__bytes_write.sum", 0) / 1e9,
                          "l2_hit_pct": m.get("lts__t_sector_hit_rate.pct"),
                          "l2_tex_read_hit_pct": 100.0 * hit / max(hit + miss, 1),
                          "l1_hit_pct": m.get("l1tex__t_sector_hit_rate.pct"),
                          "b_hit_derived": 1.0 - (rd - 8 * nnz - 4 * (M + 1)) / (4.0 * nnz * K)})
            if e.get("lru_ceiling"):
                e["frac_of_ceiling"] = e["frac"] / e["lru_ceiling"]
            res[c]["policies"][pol] = e
    if md:
        for c, v in res.items():
            print(f"\n**{c}** (nnz {v['nnz']:,}, K={v['K']})\n")
            print("| policy | step ms | GFLOP/s | vs identity | HBM frac | LRU ceiling | frac/ceiling | ncu DRAM read GB | L2 hit % | derived B hit | build s |")
            print("|---|---|---|---|---|---|---|---|---|---|---|")
            for pol, e in v["policies"].items():
                f = lambda k, fmt: (fmt % e[k]) if e.get(k) is not None else "—"   # noqa: E731
                print(f"| {pol} | {e['ms']:.3f} | {e['gflops']:,.0f} | {e['speedup_vs_identity']:.2f}× | {e['frac']:.3f} | "
                      f"{f('lru_ceiling', '%.3f')} | {f('frac_of_ceiling', '%.2f')} | {f('dram_read_GB', '%.2f')} | "
                      f"{f('l2_hit_pct', '%.1f')} | {f('b_hit_derived', '%.3f')} | {e['build_ms'] / 1e3:.2f} |")
    else:
        print(json.dumps(res, indent=1))


if __name__ == "__main__":
    main()
