"""Print the headline fields of a bench.py JSON line (file path args)."""
import json
import sys

for p in sys.argv[1:]:
    try:
        lines = [l for l in open(p) if l.strip().startswith("{")]
        d = json.loads(lines[-1])
    except Exception as e:
        print(p, "unreadable:", e)
        continue
    cfg = d.get("config", {})
    rf = d.get("roofline", {}) or {}
    e2e = d.get("e2e", {}) or {}
    print(f"{p}: {cfg.get('workload')} value={d.get('value', 0):.4g} ms/step={d.get('ms_per_step', 0):.3f} "
          f"e2e={e2e.get('value', 0) or 0:.4g} frac={rf.get('frac')} launch_ms={rf.get('launch_ms')}")
    print("   stages:", cfg.get("stage_ms_per_step"))
