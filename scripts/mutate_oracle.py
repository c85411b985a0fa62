"""Mutation check of the oracle's pins (test infrastructure): apply one plausible mistake at a time to a copy of
oracle/oracle.c (a dropped term, a wrong sign / index / bound, a swapped tie-break, min for max ...), rebuild the
copy's liboracle, run the CPU oracle tests against it, and report which mutations no test catches.

  python scripts/mutate_oracle.py [--only substr] [--out profiles/mutation_oracle.json]

Works in a scratch copy of the repo (the tree is never modified).  Each mutation must change the source exactly
once (checked), so the list stays in step with oracle.c.
"""
import argparse
import json
import os
import shutil
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

# (name, old, new): `old` must occur exactly once in oracle.c
MUTATIONS = [
    ("validate: drop rowidx[0] check", "if (rowidx[0] != 0 || rowidx[M] != nnz) return 2;", "if (rowidx[M] != nnz) return 2;"),
    ("validate: drop rowidx[M] check", "if (rowidx[0] != 0 || rowidx[M] != nnz) return 2;", "if (rowidx[0] != 0) return 2;"),
    ("validate: allow equal columns", "colidx[j] <= colidx[j - 1]) return 5;", "colidx[j] < colidx[j - 1]) return 5;"),
    ("validate: col >= N allowed", "colidx[j] >= N) return 4;", "colidx[j] > N) return 4;"),
    ("spmm: B column index off by one", "B[(int64_t)colidx[j] * K + k]", "B[(int64_t)colidx[j] * K + (k + 1) % K]"),
    ("spmm: B transposed index", "B[(int64_t)colidx[j] * K + k]", "B[(int64_t)k * K + colidx[j] % K]"),
    ("spmm: skip last nnz of a row", "for (int64_t j = rowidx[i]; j < rowidx[i + 1]; ++j) {\n                double a",
     "for (int64_t j = rowidx[i]; j + 1 < rowidx[i + 1]; ++j) {\n                double a"),
    ("spmm: bound without |a|", "bnd += fabs(a) * fabs(b);", "bnd += a * fabs(b);"),
    ("spmm: float accumulation", "double acc = 0.0, bnd = 0.0;", "float acc = 0.0f; double bnd = 0.0;"),
    ("warp load: floor", "return (nnz + nt - 1) / nt; }", "return nnz / nt; }"),
    ("blocks: block = col % bw", "int32_t blk = colidx[j] / bw;", "int32_t blk = colidx[j] % bw;"),
    ("ham: one times common", "- 2 * common;", "- common;"),
    ("sort: ties by descending id", "return (a->id > b->id) - (a->id < b->id);\n}\nstatic int cmp_asc",
     "return (a->id < b->id) - (a->id > b->id);\n}\nstatic int cmp_asc"),
    ("sort: ascending key", "if (a->key != b->key) return a->key > b->key ? -1 : 1;", "if (a->key != b->key) return a->key < b->key ? -1 : 1;"),
    ("minhash: max for min", "if (v < m) m = v;", "if (v > m || m == ~(uint64_t)0) m = v;"),
    ("minhash: seed dropped", "splitmix64((uint64_t)(colidx[j] / bw) ^ seed)", "splitmix64((uint64_t)(colidx[j] / bw))"),
    ("minhash: column instead of block", "splitmix64((uint64_t)(colidx[j] / bw) ^ seed)", "splitmix64((uint64_t)colidx[j] ^ seed)"),
    ("splitmix: wrong shift", "z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;", "z = (z ^ (z >> 26)) * 0x94D049BB133111EBULL;"),
    ("median: upper median", "int64_t want = (nb - 1) / 2, k = -1;", "int64_t want = nb / 2, k = -1;"),
    ("chain CTA: start at max wl", "if (wl[om[a]] < wl[om[best]] || (wl[om[a]] == wl[om[best]] && om[a] < om[best])) best = a;",
     "if (wl[om[a]] > wl[om[best]] || (wl[om[a]] == wl[om[best]] && om[a] < om[best])) best = a;"),
    ("chain: ties to highest id", "(k2 == bk2 && r < om[best])", "(k2 == bk2 && r > om[best])"),
    ("chain: max distance", "if (best < 0 || k1 < bk1 ||", "if (best < 0 || k1 > bk1 ||"),
    ("H21: no wl tie-break", "k1 = ham(bl, r, out[q - 1]); k2 = llabs(wl[r] - wl[out[q - 1]]); break;\n                case M_H22",
     "k1 = ham(bl, r, out[q - 1]); k2 = 0; break;\n                case M_H22"),
    ("H22: reference q-1 for the warp term", "k2 = q >= nw ? ham(bl, r, out[q - nw]) : 0; break;", "k2 = q >= nw ? ham(bl, r, out[q - 1]) : 0; break;"),
    ("WARP: reference previous row", "case M_WARP:\n                    k1 = ham(bl, r, out[q - nw]); break;",
     "case M_WARP:\n                    k1 = ham(bl, r, out[q - 1]); break;"),
    ("H23: wl term against q-nw", "k1 = ham(bl, r, out[q - nw]); k2 = llabs(wl[r] - wl[out[q - 1]]); break;",
     "k1 = ham(bl, r, out[q - nw]); k2 = llabs(wl[r] - wl[out[q - nw]]); break;"),
    ("WARP: seed rows descending", "qsort(t, (size_t)n, sizeof(keyed), cmp_asc_key_asc_id);", "qsort(t, (size_t)n, sizeof(keyed), cmp_desc_key_asc_id);"),
    ("H1: segment start = last row", "out[0] = om[0];\n        placed[0] = 1;", "out[0] = om[n - 1];\n        placed[n - 1] = 1;"),
    ("H1: runs not cut at W", "if (p == run_start || (p - run_start) % W == 0) seg[ns++] = p;", "if (p == run_start) seg[ns++] = p;"),
    ("flipped: even chunks reversed", "perm[p] = (c & 1) ? s[lo + (hi - 1 - p)] : s[p];", "perm[p] = (c & 1) ? s[p] : s[lo + (hi - 1 - p)];"),
    ("LPT: most loaded warp", "if (bw_ < 0 || load[w] < load[bw_]) bw_ = w;", "if (bw_ < 0 || load[w] > load[bw_]) bw_ = w;"),
    ("LPT: no capacity", "if (cnt[w] >= cap[w]) continue;", "if (cnt[w] >= cap[w] + 1) continue;"),
    ("DCSR: empty rows first", "for (int64_t i = 0; i < M; ++i) if (nnz[i] > 0) perm[q++] = (int32_t)i;\n        for (int64_t i = 0; i < M; ++i) if (nnz[i] == 0) perm[q++] = (int32_t)i;",
     "for (int64_t i = 0; i < M; ++i) if (nnz[i] == 0) perm[q++] = (int32_t)i;\n        for (int64_t i = 0; i < M; ++i) if (nnz[i] > 0) perm[q++] = (int32_t)i;"),
    ("permuted csr: values of the position, not the row", "value2[rowidx2[p] + t] = value[rowidx[i] + t];", "value2[rowidx2[p] + t] = value[rowidx[p < M ? p : i] + t];"),
    ("features: density over M*M", "(double)nnz_total / ((double)M * (double)N)", "(double)nnz_total / ((double)M * (double)M)"),
    ("features: mean over n-1", "out3[1] = (double)sum / (double)n;", "out3[1] = (double)sum / (double)(n > 1 ? n - 1 : 1);"),
    ("features: warp of row = p / nw", "tmp[p % nw] += warp_load(", "tmp[(p / nw) % nw] += warp_load("),
    ("features: same-cache-lines counts every nnz", "if (first) { req[b]++; T[p % nw]++; }", "{ req[b]++; T[p % nw]++; (void)first; }"),
    ("features: distinct lines over all rows", "for (int64_t p = w; p < M; p += nw) {\n            int64_t i = perm ? perm[p] : p;\n            for (int64_t t = bl.ptr[i]",
     "for (int64_t p = 0; p < M; p += 1) {\n            int64_t i = perm ? perm[p] : p;\n            for (int64_t t = bl.ptr[i]"),
    ("features: adjacent distance p, p+2", "tmp[p] = ham(&bl, perm ? perm[p] : p, perm ? perm[p + 1] : p + 1);",
     "tmp[p] = ham(&bl, perm ? perm[p] : p, perm ? perm[p + 1 < na ? p + 2 - (p + 2 > na) : p + 1] : (p + 2 < M ? p + 2 : p + 1));"),
    ("features: chunk of nt + 1 nnz", "int64_t c1 = c0 + nt < rowidx[i + 1] ? c0 + nt : rowidx[i + 1];",
     "int64_t c1 = c0 + nt + 1 < rowidx[i + 1] ? c0 + nt + 1 : rowidx[i + 1];"),
    ("b200: g0 groups of 3", "for (int64_t p = 0; p < M; p += 2) u2 += union_count(rowidx, colidx, perm, p, p + 2 < M ? p + 2 : M, mark, touched);",
     "for (int64_t p = 0; p < M; p += 3) u2 += union_count(rowidx, colidx, perm, p, p + 3 < M ? p + 3 : M, mark, touched);"),
    ("b200: window 512", "for (int64_t p = 0; p < M; p += 1024)\n        d += union_count(rowidx, colidx, perm, p, p + 1024 < M ? p + 1024 : M, mark, touched);",
     "for (int64_t p = 0; p < M; p += 512)\n        d += union_count(rowidx, colidx, perm, p, p + 512 < M ? p + 512 : M, mark, touched);"),
    ("b200: g3 without C bytes", "4 * (M + 1) + 8 * nnz + 4 * K * cn + 4 * M * K);", "4 * (M + 1) + 8 * nnz + 4 * K * cn);"),
    ("b200: split at >= 128", "if (len > 128) nsplit += len;", "if (len >= 128) nsplit += len;"),
    ("b200: rpw 4 at K = 32", "int64_t rpw = K <= 32 ? 8 : K <= 256 ? 4 : 2;", "int64_t rpw = K < 32 ? 8 : K <= 256 ? 4 : 2;"),
    ("b200: slots from the group's smallest", "slots += rpw * sl[t];", "slots += rpw * sl[(t + rpw - 1 < w1 ? t + rpw - 1 : w1 - 1)];"),
    ("b200: short rows include 0", "if (len > 0 && len <= 128) sl[ns++] = len;", "if (len <= 128) sl[ns++] = len;"),
    ("partition: floor target", "int64_t target = (p * nnz + P - 1) / P;", "int64_t target = (p * nnz) / P;"),
    ("partition: first row with rowidx > target", "while (r < M && rowidx[r] < target) ++r;", "while (r < M && rowidx[r] <= target) ++r;"),
    ("mlp: no ReLU on layer 1", "h1[o] = s > 0 ? s : 0;\n    }\n    for (int o = 0; o < 32; ++o) {\n        double s = b2[o];\n        for (int i = 0; i < 64; ++i) s += (double)W2[o * 64 + i] * h1[i];\n        h2[o] = s > 0 ? s : 0;\n    }\n    int32_t best = 0;\n    for (int o = 0; o < P; ++o) {\n        double s = b3[o];\n        for (int i = 0; i < 32; ++i) s += (double)W3[o * 32 + i] * h2[i];\n        out[o] = s;\n        if (s < out[best]) best = o;\n    }\n    return best;\n}\n\n/* The",
     "h1[o] = s;\n    }\n    for (int o = 0; o < 32; ++o) {\n        double s = b2[o];\n        for (int i = 0; i < 64; ++i) s += (double)W2[o * 64 + i] * h1[i];\n        h2[o] = s > 0 ? s : 0;\n    }\n    int32_t best = 0;\n    for (int o = 0; o < P; ++o) {\n        double s = b3[o];\n        for (int i = 0; i < 32; ++i) s += (double)W3[o * 32 + i] * h2[i];\n        out[o] = s;\n        if (s < out[best]) best = o;\n    }\n    return best;\n}\n\n/* The"),
    ("mlp: log for log1p", "for (int i = 0; i < 24; ++i) x[i] = (log1p(feat[i])", "for (int i = 0; i < 24; ++i) x[i] = (log(feat[i] + 1e-300)"),
    ("mlp: argmax", "if (s < out[best]) best = o;\n    }\n    return best;\n}\n\n/* The", "if (s > out[best]) best = o;\n    }\n    return best;\n}\n\n/* The"),
    ("mlp_n: sigma not applied", "for (int i = 0; i < F; ++i) x[i] = (log1p(feat[i]) - (double)mu[i]) / (double)sg[i];",
     "for (int i = 0; i < F; ++i) x[i] = (log1p(feat[i]) - (double)mu[i]);"),
]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--only", default="")
    ap.add_argument("--out", default="")
    ap.add_argument("--workers", default="8")
    args = ap.parse_args()
    src0 = open(os.path.join(ROOT, "oracle", "oracle.c")).read()
    work = tempfile.mkdtemp(prefix="mutate_oracle_")
    for d in ("oracle", "tests", "synthetic", "paper_conf_ispass_mehrabilcslo21_b200", "tools", "scripts"):
        shutil.copytree(os.path.join(ROOT, d), os.path.join(work, d),
                        ignore=shutil.ignore_patterns("build", "__pycache__", "*.ncu-rep"))
    for f in ("pytest.ini", "bench.py", "__graft_entry__.py"):
        shutil.copy(os.path.join(ROOT, f), os.path.join(work, f))
    shutil.copytree(os.path.join(ROOT, "include"), os.path.join(work, "include"))
    os.makedirs(os.path.join(work, "profiles"))
    for f in os.listdir(os.path.join(ROOT, "profiles")):
        if f.endswith(".jsonl") or f.endswith(".json"):
            shutil.copy(os.path.join(ROOT, "profiles", f), os.path.join(work, "profiles", f))
    tests = sorted(os.path.join("tests", f) for f in os.listdir(os.path.join(work, "tests"))
                   if f.startswith("test_oracle") or f in ("test_abi.py", "test_sharded_gloo.py"))
    results = []
    for name, old, new in [("(none: the unmutated oracle must pass)", "", "")] + MUTATIONS:
        if old and args.only and args.only not in name:
            continue
        n = src0.count(old) if old else 1
        if n != 1:
            results.append({"mutation": name, "error": f"pattern occurs {n} times"})
            print(f"!! {name}: pattern occurs {n} times", flush=True)
            continue
        with open(os.path.join(work, "oracle", "oracle.c"), "w") as f:
            f.write(src0.replace(old, new) if old else src0)
        lib = os.path.join(work, "oracle", "liboracle.so")
        if os.path.exists(lib):
            os.remove(lib)
        t0 = time.time()
        b = subprocess.run(["gcc", "-O2", "-fopenmp", "-shared", "-fPIC", "-std=gnu11", "oracle/oracle.c", "-o",
                            "oracle/liboracle.so", "-lm"], cwd=work, capture_output=True, text=True)
        if b.returncode != 0:
            results.append({"mutation": name, "error": "does not compile: " + b.stderr[-300:]})
            print(f"!! {name}: compile error", flush=True)
            continue
        r = subprocess.run([sys.executable, "-m", "pytest", "-x", "-q", "-m", "not gpu", "-p", "no:cacheprovider",
                            "-n", args.workers, *tests], cwd=work, capture_output=True, text=True, timeout=1800)
        killed = r.returncode != 0
        tail = [l for l in r.stdout.splitlines() if l.startswith("FAILED") or "passed" in l or "failed" in l][-3:]
        results.append({"mutation": name, "killed": killed, "seconds": round(time.time() - t0, 1), "by": tail})
        print(f"{'killed ' if killed else 'SURVIVED'} {name}  ({time.time() - t0:.0f}s) {tail[:1]}", flush=True)
        if not old and killed:
            raise SystemExit("the unmutated oracle fails its tests in the scratch copy: " + r.stdout[-2000:])
    with open(os.path.join(work, "oracle", "oracle.c"), "w") as f:
        f.write(src0)
    shutil.rmtree(work, ignore_errors=True)
    results = results[1:]
    surv = [r["mutation"] for r in results if r.get("killed") is False]
    summary = {"mutations": len(results), "killed": sum(1 for r in results if r.get("killed")), "survived": surv,
               "errors": [r["mutation"] for r in results if "error" in r], "results": results}
    print(json.dumps({k: summary[k] for k in ("mutations", "killed", "survived", "errors")}))
    if args.out:
        with open(args.out, "w") as f:
            json.dump(summary, f, indent=1)


if __name__ == "__main__":
    main()
