#!/usr/bin/env python
"""Train the learned schedule selector from the B200 corpus.

PAPER.md:445-469 trains LightGBM on Table 7's features to predict the best parallelization
strategy.  Here: one cost-sensitive regression tree per op class (sklearn, multi-output)
whose targets are the log-slowdowns log(t_s / t_best) of EVERY candidate schedule s; a leaf
stores the mean log-slowdown vector of its training points and predicts the schedule that
minimises it.  Features (the Table 7 graph information plus F, which Fig. 7 shows matters):
    log2 V, log2 E, log2 mean in-degree, CV = std_nnz / mean, log2(max_deg / mean), log2 F.
Validated by leave-graphs-out cross-validation: the slowdown of the predicted schedule versus
the best measured one (the Fig. 12 analogue).  Exports a plain-text tree file that
ug_selector.cpp evaluates (selector_model.txt next to libugraph.so).

    python scripts/train_selector.py gpurun_out/selector_corpus.jsonl \
        --model paper_conf_asplos_0001lslwlgslllw23_b200/selector_model.txt --report profiles/r1/r1_selector_cv.json
"""
import argparse
import json
import math
import sys

import numpy as np

PENALTY = math.log(20.0)          # a schedule that failed / was not timed at a point
FEATURES = ["log2_V", "log2_E", "log2_mean_deg", "cv", "log2_max_over_mean", "log2_F"]


def features(r):
    mean = max(r["mean_deg"], 1e-9)
    return [math.log2(max(r["V"], 1)), math.log2(max(r["E"], 1)), math.log2(mean), r["std_nnz"] / mean,
            math.log2(max(r["max_deg"], 1) / mean), math.log2(r["F"])]


def load(paths):
    rows = []
    for p in paths:
        for line in open(p):
            r = json.loads(line)
            if r.get("times"):
                rows.append(r)
    return rows


def design(rows):
    scheds = sorted({s for r in rows for s in r["times"]})
    idx = {s: i for i, s in enumerate(scheds)}
    X = np.array([features(r) for r in rows])
    Y = np.full((len(rows), len(scheds)), PENALTY)
    T = np.full((len(rows), len(scheds)), np.inf)
    for i, r in enumerate(rows):
        best = min(r["times"].values())
        for s, t in r["times"].items():
            Y[i, idx[s]] = min(PENALTY, math.log(t / best))
            T[i, idx[s]] = t
    groups = np.array([r["graph"] for r in rows])
    return X, Y, T, scheds, groups


def fit(X, Y, depth, leaf):
    from sklearn.tree import DecisionTreeRegressor
    return DecisionTreeRegressor(max_depth=depth, min_samples_leaf=leaf, random_state=0).fit(X, Y)


def cv_eval(X, Y, T, groups, depth, leaf, folds=6):
    """Leave-graphs-out CV: slowdowns of the predicted schedule on held-out graphs."""
    ug = np.unique(groups)
    rng = np.random.default_rng(0)
    rng.shuffle(ug)
    slow = []
    for k in range(folds):
        test_g = set(ug[k::folds].tolist())
        te = np.array([g in test_g for g in groups])
        if te.all() or not te.any():
            continue
        m = fit(X[~te], Y[~te], depth, leaf)
        pred = m.predict(X[te]).argmin(axis=1)
        tt = T[te]
        best = tt.min(axis=1)
        chosen = tt[np.arange(len(pred)), pred]
        chosen = np.where(np.isfinite(chosen), chosen, best * 20.0)
        slow += (chosen / best).tolist()
    return np.array(slow)


def knn_scores(Xtr, Ytr, Xte, k, w):
    """Distance-weighted mean log-slowdown of the k nearest training points (standardised,
    weighted features) -- the rule ug_selector.cpp's knn_rank evaluates."""
    mu, sd = Xtr.mean(axis=0), Xtr.std(axis=0) + 1e-9
    Ztr, Zte = (Xtr - mu) / sd * w, (Xte - mu) / sd * w
    out = np.empty((len(Xte), Ytr.shape[1]))
    for i, z in enumerate(Zte):
        d = np.sqrt(((Ztr - z) ** 2).sum(axis=1))
        nn = np.argsort(d, kind="stable")[:k]
        wt = 1.0 / (d[nn] + 1e-3)
        out[i] = (Ytr[nn] * wt[:, None]).sum(axis=0) / wt.sum()
    return out


def knn_cv_eval(X, Y, T, groups, k, w, folds=6):
    """Leave-graphs-out CV of the nearest-neighbour rule (same folds as cv_eval)."""
    ug = np.unique(groups)
    rng = np.random.default_rng(0)
    rng.shuffle(ug)
    slow = []
    for f in range(folds):
        test_g = set(ug[f::folds].tolist())
        te = np.array([g in test_g for g in groups])
        if te.all() or not te.any():
            continue
        pred = knn_scores(X[~te], Y[~te], X[te], k, w).argmin(axis=1)
        tt = T[te]
        best = tt.min(axis=1)
        chosen = tt[np.arange(len(pred)), pred]
        chosen = np.where(np.isfinite(chosen), chosen, best * 20.0)
        slow += (chosen / best).tolist()
    return np.array(slow)


def export_knn(X, Y, scheds, cls, k, w):
    mu, sd = X.mean(axis=0), X.std(axis=0) + 1e-9
    Z = (X - mu) / sd * w
    lines = [f"knn {cls} {k} {len(X)} {len(scheds)}",
             "w " + " ".join(f"{v:.9g}" for v in w), "mu " + " ".join(f"{v:.9g}" for v in mu),
             "sd " + " ".join(f"{v:.9g}" for v in sd), "s " + " ".join(scheds)]
    for z, y in zip(Z, Y):
        lines.append("p " + " ".join(f"{v:.6g}" for v in z) + " " + " ".join(f"{v:.5g}" for v in y))
    return lines


def export_tree(model, scheds, cls):
    t = model.tree_
    lines = [f"class {cls} {t.node_count}"]
    for n in range(t.node_count):
        if t.children_left[n] < 0:
            best = scheds[int(np.argmin(t.value[n][:, 0]))]
            lines.append(f"{n} -1 0 -1 -1 {best}")
        else:
            lines.append(f"{n} {t.feature[n]} {t.threshold[n]:.9g} {t.children_left[n]} {t.children_right[n]} -")
    return lines


def predict_text(lines, x):
    """Evaluate an exported tree (the same walk ug_selector.cpp does) -- used by the tests."""
    nodes = {}
    for ln in lines[1:]:
        n, f, thr, l, r, s = ln.split()
        nodes[int(n)] = (int(f), float(thr), int(l), int(r), s)
    n = 0
    while nodes[n][0] >= 0:
        f, thr, l, r, _ = nodes[n]
        n = l if x[f] <= thr else r
    return nodes[n][4]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("corpus", nargs="+")
    ap.add_argument("--model", required=True)
    ap.add_argument("--report", default=None)
    ap.add_argument("--depths", nargs="+", type=int, default=[2, 3, 4, 5, 6, 8])
    ap.add_argument("--leaf", type=int, default=3)
    args = ap.parse_args()
    rows = load(args.corpus)
    out = ["# ugraph-b200 learned selector v2 (scripts/train_selector.py): per op class either a regression",
           "# tree over " + " ".join(FEATURES) + "; node: id feature threshold left right schedule",
           "# (x[feature] <= threshold -> left; leaves have feature -1 and name their schedule), or a",
           "# nearest-neighbour block (knn <class> <k> <n> <nsched>; w / mu / sd; s <schedules>; p <z> <log-slowdowns>)",
           "# -- whichever leave-graphs-out CV favours"]
    report = {"features": FEATURES, "classes": {}}
    for cls in sorted({r["class"] for r in rows}):
        rc = [r for r in rows if r["class"] == cls]
        X, Y, T, scheds, groups = design(rc)
        # baseline: the single schedule with the best geometric-mean slowdown over the class
        best_fixed = int(np.argmin(Y.mean(axis=0)))
        fixed = np.exp(Y[:, best_fixed])
        res = {}
        for d in args.depths:
            s = cv_eval(X, Y, T, groups, d, args.leaf)
            res[d] = {"geomean": float(np.exp(np.log(s).mean())), "p90": float(np.quantile(s, 0.9)),
                      "max": float(s.max()), "within_10pct": float((s <= 1.10).mean())}
        d_best = min(res, key=lambda d: res[d]["geomean"])
        # the nearest-neighbour rule over the same folds; the better of the two is exported
        kres = {}
        for k in (3, 5, 8):
            for fw in (1.0, 2.0, 4.0):
                w = np.array([1.0, 1.0, 1.0, 1.0, 1.0, fw])
                sk = knn_cv_eval(X, Y, T, groups, k, w)
                kres[f"k{k}_wF{fw:g}"] = {"k": k, "wF": fw, "geomean": float(np.exp(np.log(sk).mean())),
                                          "p90": float(np.quantile(sk, 0.9)), "max": float(sk.max()),
                                          "within_10pct": float((sk <= 1.10).mean())}
        kb = min(kres, key=lambda key: kres[key]["geomean"])
        use_knn = kres[kb]["geomean"] < res[d_best]["geomean"]
        if use_knn:
            w = np.array([1.0, 1.0, 1.0, 1.0, 1.0, kres[kb]["wF"]])
            out += export_knn(X, Y, scheds, cls, kres[kb]["k"], w)
        else:
            model = fit(X, Y, d_best, args.leaf)
            out += export_tree(model, scheds, cls)
        report["classes"][cls] = {"points": len(rc), "graphs": int(len(np.unique(groups))),
                                  "schedules": len(scheds), "depth": d_best, "cv_by_depth": res,
                                  "knn_cv": kres, "knn_best": kb, "exported": "knn" if use_knn else "tree",
                                  "fixed_best": {"schedule": scheds[best_fixed],
                                                 "geomean": float(np.exp(np.log(fixed).mean())),
                                                 "p90": float(np.quantile(fixed, 0.9))}}
        print(f"{cls:8s} points {len(rc):4d}  tree depth {d_best}: CV geomean slowdown "
              f"{res[d_best]['geomean']:.3f} p90 {res[d_best]['p90']:.3f} within10% "
              f"{res[d_best]['within_10pct']:.2f} | knn {kb}: {kres[kb]['geomean']:.3f} p90 {kres[kb]['p90']:.3f} "
              f"within10% {kres[kb]['within_10pct']:.2f} -> {'knn' if use_knn else 'tree'} | single best "
              f"schedule {scheds[best_fixed]} geomean {report['classes'][cls]['fixed_best']['geomean']:.3f}",
              flush=True)
    with open(args.model, "w") as f:
        f.write("\n".join(out) + "\n")
    if args.report:
        with open(args.report, "w") as f:
            json.dump(report, f, indent=1)
    print("wrote", args.model, file=sys.stderr)


if __name__ == "__main__":
    main()
