"""Summarise an ncu source page (cuda,sass CSV) by CUDA source line: instructions executed, top N."""
import re
import sys

path = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
lines = open(path).read().splitlines()
hdr = next(l for l in lines if l.startswith('"Line No"'))
cols = re.findall(r'"([^"]*)"', hdr)
ncol = len(cols)
i_ins = cols.index("Instructions Executed")
stats = []
total = 0
for l in lines:
    m = re.match(r'^"(\d+)",', l)
    if not m:
        continue
    tail = l.split('","')
    vals = tail[-(ncol - 2):]
    try:
        ins = int(vals[i_ins - 2].strip('"'))
    except ValueError:
        continue
    total += ins
    src = l[len(m.group(0)):].split('","-","-"')[0].strip('"')[:100]
    stats.append((ins, int(m.group(1)), src))
stats.sort(reverse=True)
print(f"total instructions {total}")
for s, ln, src in stats[:top]:
    print(f"{100.0 * s / total:6.2f}% {s:12d} L{ln:5d} {src}")
