"""Write full-graph oracle goldens for a BASELINE config: tests/golden/c<cfg>_counts.txt.

Calls only ``oracle/`` (O2, Algorithm 1 + Eq. (1) written out) and the
seeded input generators ``tdfs_inputs`` -- never the CUDA path.  Each query's count is the
size of M(G, Q, C_auto) (R1/R3), which does not depend on the matching order, so
the CUDA path's planner-order count must equal it bit for bit.

Usage: python scripts/golden_counts.py --config 2 [--queries triangle,c4,...] [--threads N]
Appends one line per finished query (so a long run can be resumed / inspected), keeping the
lines of other queries already in the file.
"""
from __future__ import annotations

import argparse
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402
import tdfs_inputs as T  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, required=True)
    ap.add_argument("--queries", default="")
    ap.add_argument("--threads", type=int, default=os.cpu_count() or 1)
    ap.add_argument("--label-count", type=int, default=8)
    a = ap.parse_args()
    names = a.queries.split(",") if a.queries else T.CONFIG_QUERIES[a.config]
    path = os.path.join(ROOT, "tests", "golden", f"c{a.config}_counts.txt")
    have = {}
    if os.path.exists(path):
        for line in open(path):
            if line.strip() and not line.startswith("#"):
                have[line.split(":", 1)[0].strip()] = line
    t0 = time.time()
    g = T.config_graph(a.config)
    og = oracle.OracleGraph(g)
    print(f"config {a.config}: n={g.n} m={g.m} built in {time.time() - t0:.1f}s", flush=True)
    for name in names:
        q = T.labeled_query(name, a.label_count) if a.config == 4 else T.query(name)
        t1 = time.time()
        c = oracle.count(og, q, "auto", threads=a.threads)
        dt = time.time() - t1
        have[name] = (f"{name}: {c}    # oracle O2 (BFS order, C_auto), {a.threads} threads, {dt:.0f} s, "
                      f"{time.strftime('%Y-%m-%d')}\n")
        print(have[name], end="", flush=True)
        with open(path + ".tmp", "w") as f:
            f.write(f"# Full-graph match counts |M(G, Q, C_auto)| of BASELINE config {a.config} "
                    f"({g.name}: n={g.n}, m={g.m}).\n")
            f.write("# Written by scripts/golden_counts.py, which calls only oracle/ (O2: Algorithm 1 + Eq. (1),\n")
            f.write("# PAPER.md:54-82; constraints by the stabilizer chain, DESIGN.md R3) on the seeded generator.\n")
            for v in have.values():
                f.write(v)
        os.replace(path + ".tmp", path)


if __name__ == "__main__":
    main()
