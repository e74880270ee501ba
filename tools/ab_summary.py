"""print one summary line per bench JSON file: ms/step and per-primitive ms (A/B sessions)"""
import json
import sys

for p in sys.argv[1:]:
    try:
        d = json.loads(open(p).read().strip().splitlines()[-1])
    except Exception as e:  # noqa: BLE001
        print(p, "unreadable", e)
        continue
    pp = " ".join(f"{k}={v:.3f}" for k, v in sorted(d.get("per_primitive_ms", {}).items()))
    print(f"{p}: {d['ms_per_step']:.3f} ms/step  {pp}  clocks={d.get('clocks', {}).get('sm_mhz')}")
