"""Tables of the NEXT-1 sensitivity study from tools/sensitivity.py JSONL output.

  Fig. 6 analogue: geomean over graphs of (per-graph best time / time at this cost), per K;
  default-cost score: geomean of best / time at the default (cost 0), and the worst graph;
  Fig. 7 analogue: geomean GFLOP/s and time at the default cost, per K;
  Fig. 5 analogue: atomic vs regular row writes at K=16, default cost; parity flags.
Usage: python tools/sensitivity_summary.py FILE.jsonl"""
import json
import sys
from collections import defaultdict

import numpy as np


def main(path):
    rows = [json.loads(l) for l in open(path) if l.strip()]
    by = defaultdict(dict)                     # (graph, K) -> cost -> ms
    for r in rows:
        by[(r["graph"], r["K"])][r["cost"]] = r
    Ks = sorted({r["K"] for r in rows})
    costs = sorted({r["cost"] for r in rows if r["cost"] > 0})
    graphs = sorted({r["graph"] for r in rows})
    print("| K | " + " | ".join(str(c) for c in costs) + " | default score | worst graph |")
    print("|---" * (len(costs) + 3) + "|")
    for K in Ks:
        cells = []
        for c in costs:
            v = [by[(g, K)][c_best]["ms"] for g in graphs
                 for c_best in [min(by[(g, K)], key=lambda x: by[(g, K)][x]["ms"])]]
            ratios = [min(x["ms"] for x in by[(g, K)].values()) / by[(g, K)][c]["ms"]
                      for g in graphs if c in by[(g, K)]]
            cells.append("%.3f" % np.exp(np.mean(np.log(ratios))))
        d = [min(x["ms"] for x in by[(g, K)].values()) / by[(g, K)][0]["ms"] for g in graphs]
        print("| %d | %s | %.3f | %.3f |" % (K, " | ".join(cells), np.exp(np.mean(np.log(d))),
                                          min(d)))
    print()
    print("| K | geomean GFLOP/s (default cost) | geomean ms |")
    print("|---|---|---|")
    for K in Ks:
        gf = [by[(g, K)][0]["gflops"] for g in graphs]
        ms = [by[(g, K)][0]["ms"] for g in graphs]
        print("| %d | %.0f | %.4f |" % (K, np.exp(np.mean(np.log(gf))), np.exp(np.mean(np.log(ms)))))
    print()
    ok = [r.get("parity_ok") for r in rows if "parity_ok" in r]
    print("parity ok at K=16, default cost: %d of %d graphs" % (sum(bool(x) for x in ok), len(ok)))


if __name__ == "__main__":
    main(sys.argv[1])
