"""Summarise an ncu source page (cuda,sass CSV) by CUDA source line: warp-stall samples, top N."""
import re
import sys

path = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
lines = open(path).read().splitlines()
hdr = next(l for l in lines if l.startswith('"Line No"'))
cols = re.findall(r'"([^"]*)"', hdr)
ncol = len(cols)
i_samp = cols.index("Warp Stall Sampling (All Samples)")
i_ni = cols.index("Warp Stall Sampling (Not-issued Samples)")
stats = []
total = 0
for l in lines:
    m = re.match(r'^"(\d+)",', l)
    if not m:
        continue
    fields = re.findall(r'"((?:[^"]|"")*)"(?:,|$)', l)
    tail = l.split('","')
    vals = tail[-(ncol - 2):]
    try:
        samp = int(vals[i_samp - 2].strip('"'))
    except ValueError:
        continue
    total += samp
    src = l[len(m.group(0)):].split('","-","-"')[0].strip('"')[:110]
    stats.append((samp, int(m.group(1)), src))
stats.sort(reverse=True)
print(f"total samples {total}")
for s, ln, src in stats[:top]:
    print(f"{100.0 * s / total:6.2f}% {s:8d} L{ln:5d} {src}")
