"""Summarise TRACE lines of tools/tune.py: per kind, count / total / mean dt and mean N, E."""
import collections
import json
import sys

agg = collections.defaultdict(lambda: [0, 0.0, 0, 0, 0])
rows = []
for line in sys.stdin:
    if not line.startswith("TRACE "):
        continue
    r = json.loads(line[6:])
    rows.append(r)
    a = agg[r["kind"]]
    a[0] += 1; a[1] += r["dt_us"]; a[2] += r["N"]; a[3] += r["E"]; a[4] += r["a"]
tot = sum(a[1] for a in agg.values())
for k, a in agg.items():
    print(f"{k:12s} n={a[0]:6d} total={a[1]/1e3:9.2f} ms ({100*a[1]/max(tot,1e-9):5.1f}%) mean={a[1]/a[0]:8.2f} us "
          f"N={a[2]/a[0]:10.0f} E={a[3]/a[0]:10.0f} a={a[4]/a[0]:10.0f}")
if rows and len(sys.argv) > 1:
    for r in rows[: int(sys.argv[1])]:
        print(r)
