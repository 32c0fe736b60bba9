"""Print the key fields of a bench.py JSON line (tools; no method arithmetic)."""
import json
import sys

for path in sys.argv[1:]:
    for line in open(path):
        if line.startswith("{"):
            d = json.loads(line)
            r = d.get("roofline") or {}
            c = d.get("config", {})
            print(path, c.get("workload"), "GTEPS %.2f" % d["value"], "ms/step %.1f" % d["ms_per_step"],
                  "| e2e %.2f" % d["e2e"]["value"] if d.get("e2e") else "",
                  "| frac %.3f" % r.get("frac", 0), "|", c.get("engine_mode"), "|", c.get("engine_choice"),
                  "| ws %.2f GB" % (d.get("setup", {}).get("workspace_bytes", 0) / 1e9), "| clocks", d.get("clocks"))
