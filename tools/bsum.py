"""One-screen summary of a bench.py JSON line: value, step, roofline, per-kind launches, rounds."""
import json
import sys

for p in sys.argv[1:]:
    try:
        d = json.load(open(p))
    except Exception as e:  # noqa: BLE001
        print(p, "unreadable:", e)
        continue
    c = d["config"]
    print(f"== {c['workload']} {d['value']/1e9:.3f} G edges/s  {d['ms_per_step']:.4f} ms/step  "
          f"frac {d['roofline']['frac'] or 0:.3f} ({d['roofline']['kernel']})  {d['parity']}  "
          f"clk {d['clocks']['sm_mhz']} {d['clocks']['reasons']}  launches {d['gpu_launches']}")
    for k, v in d.get("launch_kinds", {}).items():
        print(f"   {k:24s} {v['launches_per_step']:5.1f} x {(v['avg_launch_ms'] or 0)*1e3:8.1f} us = "
              f"{(v['ms_per_step'] or 0)*1e3:8.1f} us/step  frac {v['frac'] or 0:.3f}")
    for r in d.get("rounds", []):
        print(f"   r{r['r']} {r['kind']:9s} n={r['n_r']:>9} A={r['A_r']:>10} comp={r['compacted']} "
              f"{r['filter_ms']*1e3:7.1f} us frac {r['frac'] or 0:.3f}  hook {r.get('hook_ms', 0)*1e3:6.1f} "
              f"jump {r.get('jump_ms', 0)*1e3:6.1f} compose {r.get('compose_ms', 0)*1e3:6.1f} us")
