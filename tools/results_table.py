"""Markdown results table from bench lines: python tools/results_table.py <dir> <prefix>
(e.g. profiles r02s2_bench_) — one row per workload: edges/s, ms/step, dominant kernel frac,
A8 / A2 fracs, light phase, e2e, traffic/algorithmic bytes, oracle."""
import json
import os
import sys

d, pre = sys.argv[1], sys.argv[2]
print("| Config | Bit-exact | Edges/s (device) | ms/step | Dominant kernel (frac of the measured HBM peak) | A2 frac | A8 frac | "
      "DRAM / algorithmic bytes | Light phase | e2e edges/s | Oracle (1 core) | GPU launches |")
print("|---|---|---|---|---|---|---|---|---|---|---|---|")
for w in ["grid64", "uniform", "road", "rmat22", "dense"]:
    p = os.path.join(d, f"{pre}{w}.json")
    if not os.path.exists(p):
        continue
    j = json.load(open(p))
    rf = j["roofline"]
    rk = j.get("roofline_kernels", {})
    a2 = rk.get("A2 min0", {}).get("frac")
    a8 = rk.get("A8 filter", {}).get("frac")
    tr = rf.get("traffic")
    ratio = f"{tr / rf['bytes_per_launch']:.2f}" if tr and rf.get("bytes_per_launch") else "—"
    lp = j.get("light_phase") or {}
    light = f"t = {lp['t']}" if lp.get("t") not in (None, 4294967295) else "off"
    cpu = j.get("cpu_baseline", {})
    e2e = j.get("e2e", {}).get("value")
    val = j["value"]
    vs = f"{val / 1e9:.2f} G" if val >= 1e9 else f"{val / 1e6:.0f} M"
    print(f"| {w} | {j.get('parity')} | **{vs}** | {j['ms_per_step']:.4f} | {rf['kernel'].split(' ')[0]} "
          f"{rf['frac'] * 100:.1f} % | {a2 * 100:.1f} % | " if a2 is not None else
          f"| {w} | {j.get('parity')} | **{vs}** | {j['ms_per_step']:.4f} | {rf['kernel'].split(' ')[0]} "
          f"{rf['frac'] * 100:.1f} % | — | ", end="")
    print(f"{a8 * 100:.1f} % | " if a8 is not None else "— | ", end="")
    print(f"{ratio} | {light} | {e2e / 1e9:.2f} G | {cpu.get('value', 0) / 1e6:.1f} M edges/s | {j.get('gpu_launches')} |")
