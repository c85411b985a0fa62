"""Train and evaluate the permutation predictor on the C4 corpus (§V.B-E).

  python scripts/train_predictor.py --corpus profiles/corpus_r2.jsonl --out profiles/predictor_r2.json

Per K: a 24-64-32-P MLP with L2 regularisation regresses the execution times of the P policies
(relative to the original order's time, reading A19), loss = mean absolute percentage error, samples
weighted inversely to the population of their best class, 80/20 split; the policy is the
argmin of the predicted times.  Reported like the paper: classification accuracy and confusion
matrix (Fig. 13), predicted-selection speedup vs the exhaustive-timing oracle (the paper's
1.37x vs 1.41x), loss distribution (Fig. 14: within 4% / 10%, mean), regression error CDF (Fig. 12),
the per-policy Table-I analogue, the softmax-classifier variant and the matrix-only-feature
ablation, and (f4) the same regression with the 7 B200 platform features appended.  Weights are written in spmm_predict's flat layout and the library's C inference
(spmm_predict) is checked against the torch forward.
"""
import argparse
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

MATRIX_ONLY = list(range(9))   # n_row, n_col, density, nnz-per-row x3, nnz-blocks-per-row x3 (Tab. II "Matrix")


class MLP(torch.nn.Module):
    def __init__(self, nin, nout, softmax=False):
        super().__init__()
        self.l1 = torch.nn.Linear(nin, 64)
        self.l2 = torch.nn.Linear(64, 32)
        self.l3 = torch.nn.Linear(32, nout)
        self.softmax = softmax

    def forward(self, z):
        return self.l3(torch.relu(self.l2(torch.relu(self.l1(z)))))


def load(path, K, policies, b200=False):
    """X: the 24 Table II features (+ the 7 B200 platform features at this K when b200, f4)."""
    X, T, meta = [], [], []
    for line in open(path):
        r = json.loads(line)
        t = r["times_ms"].get(str(K))
        if not t or any(p not in t for p in policies):
            continue
        if b200 and str(K) not in r.get("features_b200", {}):
            continue
        X.append(r["features"] + (r["features_b200"][str(K)] if b200 else []))
        T.append([t[p] for p in policies])
        meta.append((r["i"], r["family"], r["name"], bool(r.get("params", {}).get("shuffled"))))
    return np.array(X, dtype=np.float64), np.array(T, dtype=np.float64), meta


def train(X, Y, w, feat_idx, softmax=False, epochs=3000, seed=0, lr=3e-3, wd=1e-4):
    torch.manual_seed(seed)
    lx = np.log1p(X[:, feat_idx])
    mu, sg = lx.mean(0), lx.std(0) + 1e-6
    z = torch.tensor((lx - mu) / sg, dtype=torch.float32)
    y = torch.tensor(Y, dtype=torch.float32)
    ww = torch.tensor(w, dtype=torch.float32)
    net = MLP(len(feat_idx), Y.shape[1], softmax)
    opt = torch.optim.Adam(net.parameters(), lr=lr, weight_decay=wd)   # weight decay = L2 regularisation
    for _ in range(epochs):
        opt.zero_grad()
        out = net(z)
        if softmax:
            loss = (torch.nn.functional.cross_entropy(out, y.argmin(1), reduction="none") * ww).mean()
        else:
            loss = ((torch.abs(y - out) / y).mean(1) * ww).mean()      # MAPE
        loss.backward()
        opt.step()
    return net, mu, sg


def predict(net, mu, sg, X, feat_idx):
    z = torch.tensor((np.log1p(X[:, feat_idx]) - mu) / sg, dtype=torch.float32)
    with torch.no_grad():
        return net(z).numpy()


def flat_weights(net, mu, sg):
    parts = [mu, sg] + [t.detach().numpy().ravel() for t in
                        (net.l1.weight, net.l1.bias, net.l2.weight, net.l2.bias, net.l3.weight, net.l3.bias)]
    return np.concatenate([np.asarray(p, dtype=np.float32).ravel() for p in parts])


def evaluate(T, pred_choice, policies):
    best = T.argmin(1)
    t_id = T[:, 0]
    t_best = T[np.arange(len(T)), best]
    t_pred = T[np.arange(len(T)), pred_choice]
    loss = t_pred / t_best - 1.0
    P = len(policies)
    conf = np.zeros((P, P), dtype=int)
    for a, b in zip(best, pred_choice):
        conf[a, b] += 1
    return dict(
        n=len(T), accuracy=float((best == pred_choice).mean()),
        speedup_oracle=float(np.mean(t_id / t_best)), speedup_predicted=float(np.mean(t_id / t_pred)),
        oracle_gain_fraction=float((np.mean(t_id / t_pred) - 1) / max(np.mean(t_id / t_best) - 1, 1e-12)),
        mean_loss=float(loss.mean()), within_4pct=float((loss <= 0.04).mean()), within_10pct=float((loss <= 0.10).mean()),
        confusion={"rows=optimal, cols=predicted": policies, "matrix": conf.tolist()})


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--corpus", default=os.path.join(ROOT, "profiles", "corpus_r2.jsonl"))
    ap.add_argument("--policies", default="identity,nnz_sort,plain_sort,cta_aware,hybrid_1,hybrid_2_1,cta_aware+md")
    ap.add_argument("--table-policies", default=None,
                    help="policies of the Table-I analogue (default: every policy timed in the corpus)")
    ap.add_argument("--K", default="32,64,128,256")
    ap.add_argument("--epochs", type=int, default=3000)
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "predictor_r2.json"))
    ap.add_argument("--weights-dir", default=os.path.join(ROOT, "paper_conf_ispass_mehrabilcslo21_b200", "predictor"))
    args = ap.parse_args()
    policies = args.policies.split(",")
    P = len(policies)
    os.makedirs(args.weights_dir, exist_ok=True)
    import paper_conf_ispass_mehrabilcslo21_b200 as pkg
    report = {"policies": policies, "per_K": {}}
    for K in [int(k) for k in args.K.split(",")]:
        X, T, meta = load(args.corpus, K, policies)
        if len(X) < 10:
            continue
        rng = np.random.default_rng(K)
        idx = rng.permutation(len(X))
        ntr = int(0.8 * len(X))
        tr, te = idx[:ntr], idx[ntr:]
        Y = T / T[:, :1]                                  # times relative to the original order (A19)
        best_tr = T[tr].argmin(1)
        pop = np.bincount(best_tr, minlength=P).astype(np.float64)
        cw = np.where(pop > 0, pop.sum() / np.maximum(pop, 1) / P, 0.0)   # weights ∝ 1/population
        w = cw[best_tr]
        res = {"n_train": int(ntr), "n_test": int(len(te)), "class_population_train": pop.astype(int).tolist(),
               "class_weights": cw.tolist()}
        # Table-I analogue over the whole corpus: per-policy speedup vs the original order, every timed policy
        tab_pols = (args.table_policies.split(",") if args.table_policies else
                    list(json.loads(open(args.corpus).readline())["times_ms"][str(K)].keys()))
        _, TT, _ = load(args.corpus, K, tab_pols)
        sp = TT[:, :1] / TT
        res["table1"] = {p: {"max": float(sp[:, i].max()), "mean": float(sp[:, i].mean()), "min": float(sp[:, i].min())}
                         for i, p in enumerate(tab_pols)}
        res["table1"]["oracle"] = {"max": float((TT[:, 0] / TT.min(1)).max()),
                                   "mean": float((TT[:, 0] / TT.min(1)).mean()), "min": float((TT[:, 0] / TT.min(1)).min())}
        res["table1_best_share"] = dict(zip(tab_pols, (np.bincount(TT.argmin(1), minlength=len(tab_pols)) / len(TT)).tolist()))
        res["best_policy_share"] = dict(zip(policies, (np.bincount(T.argmin(1), minlength=P) / len(T)).tolist()))
        all_feats = list(range(24))
        net, mu, sg = train(X[tr], Y[tr], w, all_feats, epochs=args.epochs, seed=K)
        pr = predict(net, mu, sg, X[te], all_feats)
        choice = pr.argmin(1)
        res["regression"] = evaluate(T[te], choice, policies)
        ape = np.abs(Y[te] - pr) / Y[te] * 100
        res["regression"]["abs_error_pct_cdf"] = {"under_2": float((ape < 2).mean()), "under_10": float((ape < 10).mean()),
                                                  "median": float(np.median(ape))}
        # 5-fold cross-validation: every matrix of the corpus predicted once by a model that did not see it (a test
        # set of the whole corpus instead of one 20 % split)
        folds = np.array_split(rng.permutation(len(X)), 5)
        cv_choice = np.zeros(len(X), dtype=int)
        for f in range(5):
            te_f = folds[f]
            tr_f = np.concatenate([folds[g] for g in range(5) if g != f])
            bt = T[tr_f].argmin(1)
            pp = np.bincount(bt, minlength=P).astype(np.float64)
            cwf = np.where(pp > 0, pp.sum() / np.maximum(pp, 1) / P, 0.0)
            netf, muf, sgf = train(X[tr_f], Y[tr_f], cwf[bt], all_feats, epochs=args.epochs, seed=K + 100 * f)
            cv_choice[te_f] = predict(netf, muf, sgf, X[te_f], all_feats).argmin(1)
        res["cv5_regression"] = evaluate(T, cv_choice, policies)
        shuf = np.array([bool(m[3]) for m in meta])
        if shuf.any() and (~shuf).any():     # rows relabelled (the pre-order's regime) vs the rest
            res["cv5_regression"]["by_subset"] = {
                "shuffled": evaluate(T[shuf], cv_choice[shuf], policies),
                "not_shuffled": evaluate(T[~shuf], cv_choice[~shuf], policies)}
        # C inference through the library must agree with the torch forward
        wflat = flat_weights(net, mu, sg)
        agree = 0
        for f, c in zip(X[te], choice):
            pol, _ = pkg.spmm_predict(f, wflat, P)
            agree += int(pol == c)
        res["c_inference_agreement"] = agree / max(len(te), 1)
        np.save(os.path.join(args.weights_dir, f"mlp_K{K}.npy"), wflat)
        # softmax classifier variant
        netc, muc, sgc = train(X[tr], Y[tr], w, all_feats, softmax=True, epochs=args.epochs, seed=K)
        res["softmax_classifier"] = evaluate(T[te], predict(netc, muc, sgc, X[te], all_feats).argmax(1), policies)
        # matrix-only feature ablation
        netm, mum, sgm = train(X[tr], Y[tr], w, MATRIX_ONLY, epochs=args.epochs, seed=K)
        res["matrix_only_features"] = evaluate(T[te], predict(netm, mum, sgm, X[te], MATRIX_ONLY).argmin(1), policies)
        # f4: the same regression with the 7 B200 platform features appended (F = 31), same split and weights
        Xb, Tb, _ = load(args.corpus, K, policies, b200=True)
        if len(Xb) == len(X):
            feats31 = list(range(31))
            netb, mub, sgb = train(Xb[tr], Y[tr], w, feats31, epochs=args.epochs, seed=K)
            chb = predict(netb, mub, sgb, Xb[te], feats31).argmin(1)
            res["with_b200_features"] = evaluate(T[te], chb, policies)
            wb = flat_weights(netb, mub, sgb)
            agree = sum(int(pkg.spmm_predict_n(f, wb, P)[0] == c) for f, c in zip(Xb[te], chb))
            res["with_b200_features"]["c_inference_agreement"] = agree / max(len(te), 1)
            os.makedirs(args.weights_dir + "_b200", exist_ok=True)
            np.save(os.path.join(args.weights_dir + "_b200", f"mlp_K{K}.npy"), wb)
            rb = res["with_b200_features"]
            print(f"   +B200 features: acc={rb['accuracy']:.2f} predicted {rb['speedup_predicted']:.3f}x "
                  f"gain {rb['oracle_gain_fraction']:.2f} loss {rb['mean_loss']:.3f} C-agree {rb['c_inference_agreement']:.2f}")
        report["per_K"][str(K)] = res
        r = res["regression"]
        print(f"K={K}: n={len(X)} acc={r['accuracy']:.2f} oracle {r['speedup_oracle']:.3f}x predicted "
              f"{r['speedup_predicted']:.3f}x gain {r['oracle_gain_fraction']:.2f} loss {r['mean_loss']:.3f} "
              f"C-agree {res['c_inference_agreement']:.2f}")
        c = res["cv5_regression"]
        print(f"   5-fold CV (n={c['n']}): acc={c['accuracy']:.2f} oracle {c['speedup_oracle']:.3f}x predicted "
              f"{c['speedup_predicted']:.3f}x gain {c['oracle_gain_fraction']:.2f} loss {c['mean_loss']:.3f}")
        for k, v in c.get("by_subset", {}).items():
            print(f"      {k}: n={v['n']} oracle {v['speedup_oracle']:.3f}x gain {v['oracle_gain_fraction']:.2f}")
    with open(args.out, "w") as f:
        json.dump(report, f, indent=1)


if __name__ == "__main__":
    main()
