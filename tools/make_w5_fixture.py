"""Writes tests/golden/w5_xshuffle.json: a 16-lane bundle consistent with every fact Fig. 3
prints (P@28428-30196) — lane 0010 reads a1, lane 1010 a5, lane 0000 b0, lane 1000 a4; five
objects a..e; subscripts = chronological order — whose other 12 lanes (not printed: the figure
is absent from PAPER.md) are filled by a seeded search so that the printed outcome holds under
reading R23: only a4 and a5 of object a survive and no object keeps more than mu(4) = 2.
Calls only oracle.prior_art."""
import json
import os
import random
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from oracle import prior_art as pa  # noqa: E402

rng = random.Random(5)
for trial in range(200000):
    row = [None] * 16
    row[0b0010], row[0b1010], row[0b0000], row[0b1000] = ("a", 1), ("a", 5), ("b", 0), ("a", 4)
    pool = [("a", 0), ("a", 2), ("a", 3)] + [(o, t) for o in "bcde" for t in range(8) if (o, t) != ("b", 0)]
    rng.shuffle(pool)
    it = iter(pool[:12])
    row = [r if r is not None else next(it) for r in row]
    fin = pa.x_shuffle_bundle(row, 4)
    if (sorted({m for m in fin if m[0] == "a"}) == [("a", 4), ("a", 5)]
            and all(len({m for m in fin if m[0] == o}) <= 2 for o in "abcde")):
        break
out = {"source": "Fig. 3 X_shuffle on a bundle of 16 threads, P@28428-30196 (partial trace printed; "
                  "lanes 0000, 0010, 1000, 1010 are the paper's, the other 12 are builder-authored by "
                  "tools/make_w5_fixture.py)",
       "eta": 4, "lanes": [[o, t] for o, t in row]}
with open(os.path.join(ROOT, "tests", "golden", "w5_xshuffle.json"), "w") as f:
    json.dump(out, f, indent=1)
print(row)
