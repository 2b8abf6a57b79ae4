#!/usr/bin/env python
"""Fig. 12 analogue: per (config, op, F) of a sweep (scripts/sweep.py), the
schedule the selector picks (AUTO) against the measured best of the whole space, the best of the
paper's own strategies (thread / warp x vertex / edge, Fig. 6) and the worst -- as a markdown table.

    python scripts/fig12.py profiles/r2/sweep_r2.jsonl > profiles/r2/fig12_auto_vs_best.md
"""
import json
import sys
from collections import defaultdict


def main(path):
    runs = defaultdict(list)
    auto = {}
    for line in open(path):
        r = json.loads(line)
        key = (r["config"], r["op"], r["F"])
        if r.get("auto"):
            auto[key] = r
        elif r.get("ms") is not None:
            runs[key].append((r["ms"], r["schedule"]))
    print("| config | op | F | best schedule | best µs | AUTO schedule | AUTO µs | AUTO / best | "
          "best paper strategy (TV/TE/WV/WE) | its µs | paper / best | worst µs |")
    print("|---|---|---|---|---|---|---|---|---|---|---|---|")
    ratios = []
    for key in sorted(runs, key=lambda k: (k[0], k[1], k[2])):
        rs = sorted(runs[key])
        best_ms, best_s = rs[0]
        paper = [x for x in rs if x[1][:2] in ("TV", "TE", "WV", "WE")]
        a = auto.get(key)
        ams = a["ms"] if a else None
        ratio = ams / best_ms if ams else None
        if ratio:
            ratios.append(ratio)
        cells = [key[0], key[1], str(key[2]), best_s, f"{best_ms * 1e3:.1f}"]
        cells += [a["schedule"], f"{ams * 1e3:.1f}", f"{ratio:.2f}"] if a else ["-", "-", "-"]
        cells += [paper[0][1], f"{paper[0][0] * 1e3:.1f}", f"{paper[0][0] / best_ms:.2f}"] if paper else ["-"] * 3
        cells.append(f"{rs[-1][0] * 1e3:.1f}")
        print("| " + " | ".join(cells) + " |")
    if ratios:
        import statistics
        within = sum(1 for r in ratios if r <= 1.10)
        print(f"\nAUTO within 10 % of the measured best on {within} / {len(ratios)} cases; geomean AUTO / best "
              f"{statistics.geometric_mean(ratios):.3f}, max {max(ratios):.2f}.")


if __name__ == "__main__":
    main(sys.argv[1])
