"""Print the key numbers of a bench.py JSON line: python tools/jq.py file.json"""
import json
import sys

for f in sys.argv[1:]:
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
    except Exception as e:  # noqa: BLE001
        print(f, "unreadable:", e)
        continue
    keys = ["value", "ms_per_step", "step_ms_minmax", "host_ms_per_step", "gpu_launches", "capacity_fallbacks"]
    print(f, {k: d.get(k) for k in keys})
    print("  stages", d.get("stage_ms"))
    r = d.get("roofline") or {}
    print("  roofline", {k: r.get(k) for k in ("kernel", "achieved", "frac", "traffic")}, "clocks", d.get("clocks"))
    if "e2e" in d:
        print("  e2e", d["e2e"])
    if "cpu_baseline" in d:
        print("  cpu", d["cpu_baseline"])
