"""Markdown table of bench.py JSON lines: python tools/results_table.py FILE... (no method arithmetic)."""
import json
import sys

print("| config | engine | GTEPS | ms/step | sources | e2e GTEPS | B_min frac | HBM frac (ncu bytes) | workspace GB | SM MHz | file |")
print("|---|---|---|---|---|---|---|---|---|---|---|")
for path in sys.argv[1:]:
    d = None
    for line in open(path):
        if line.startswith("{"):
            d = json.loads(line)
    if d is None or "value" not in d:
        continue
    c, r, st = d.get("config", {}), d.get("roofline") or {}, d.get("setup", {})
    hf = r.get("hbm_frac")
    print(f"| {c.get('workload')} | {(c.get('engine_mode') or '')[:48]} | {d['value']:.2f} | {d['ms_per_step']:.1f} | "
          f"{c.get('sources_per_step')} | {d['e2e']['value']:.2f} | {r.get('frac', 0):.3f} | "
          f"{'%.3f' % hf if hf is not None else 'n/a'} | {st.get('workspace_bytes', 0) / 1e9:.2f} | "
          f"{(d.get('clocks') or {}).get('sm_mhz')} | `{path.split('/')[-1]}` |")
