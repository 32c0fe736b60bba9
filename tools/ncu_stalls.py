"""Total warp-stall reasons of an ncu source page (cuda,sass CSV)."""
import re
import sys

lines = open(sys.argv[1]).read().splitlines()
hdr = next(l for l in lines if l.startswith('"Line No"'))
cols = re.findall(r'"([^"]*)"', hdr)
i0 = cols.index("stall_barrier")
names = cols[i0:i0 + 17]
tot = [0] * 17
for l in lines:
    if l.startswith('"",""'):
        f = l.split('","')
        if len(f) == len(cols):
            for k in range(17):
                try:
                    tot[k] += int(f[i0 + k].strip('"'))
                except ValueError:
                    pass
S = sum(tot)
for n, t in sorted(zip(names, tot), key=lambda x: -x[1])[:10]:
    print(f"{n:25s} {t:9d} {100 * t / S:6.2f}%")
