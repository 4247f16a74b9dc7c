"""Write tests/golden/c0_exact_counts.txt: exact embedding counts of the C0 queries
(BASELINE.json configs[0]) computed ONLY by the oracle's exact enumerator (reading A1).
bench.py reads this file for its q-error line; tests check it stays in sync."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402
from workloads import gen  # noqa: E402

g, qs = gen.config_c0()
lines = ["# Exact embedding counts of the C0 queries (workloads/gen.py config_c0), written by",
         "# scripts/make_golden_counts.py with oracle.count_embeddings (plain backtracking, reading A1).",
         "# format: query_index query_name count"]
for i, q in enumerate(qs):
    lines.append(f"{i} {q.name} {oracle.count_embeddings(g, q)}")
path = os.path.join(ROOT, "tests", "golden", "c0_exact_counts.txt")
with open(path, "w") as f:
    f.write("\n".join(lines) + "\n")
print(open(path).read())
