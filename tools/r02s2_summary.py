"""profiles/r02s2_ncu_summary.md from the session's final evidence (tools/r02_final2.sh output
copied under profiles/ as r02s2_*): results table, per-workload launch shares and ncu rows."""
import json
import subprocess


def sh(c):
    return subprocess.run(c, shell=True, capture_output=True, text=True).stdout


out = ["# Round 2, session 2 — ncu summaries and bench lines on the final code (1 × B200, `--clock-control none`)", "",
       "Commands: `tools/r02_final2.sh` under `gpurun` (one box): `build()` + `smoke()`, `pytest -m gpu`,",
       "then per workload `tools/profile.sh` (launch list: `ncu --metrics gpu__time_duration.sum`; one `ncu --set full`",
       "capture of the arc passes and member scans of the bench's last `mst_run`; `tools/ncu_traffic.py` → DRAM bytes per",
       "launch → `profiles/ncu_traffic_<wl>.json`, which `bench.py` reports as `roofline.traffic`; raw export",
       "`r02s2_ncu_raw_<wl>.csv.gz`), then `bench.py --workload <wl> --e2e-steps 3` (`r02s2_bench_<wl>.json`) and the",
       "reference arm (`r02s2_reference_rmat22.json`). Bench numbers are never taken under ncu.", "",
       "Launch-list shares are of the summed kernel time of one `mst_run` (build kernels excluded: `tools/launch_share.py",
       "--run-only`); they are cold-cache and serialised, so compare shares with the live per-launch CUDA-event table in",
       "each bench line (`launch_kinds`), not absolute times.", "", sh("python tools/results_table.py profiles r02s2_bench_")]
notes = {
    "rmat22": """* A2 extraction (first row): ~1,083 MB of DRAM for 1,074 MB of records read + the light records written;
  ~161 µs cold = 6.7 TB/s of algorithmic bytes; live 0.98 of the measured 6,551 GB/s. The light minima pass (row 2)
  and the four light FILTER passes (~3 M records each, 44–48 % L2 hit) are bound by the label gathers into the 16.8 MB
  vertex map, not bytes.
* Member scans: ~0.5 M record ends of the small components, then a last one over a few hundred.""",
    "uniform": """* DRAM traffic ≈ the algorithmic bytes on every pass; the passes are bound by L2 operations: 15–16 M read
  requests (two label gathers per record) plus up to 18 M RED requests (two minima per record) while the next round's
  labels do not fit the shared hot table.""",
    "road": """* Traffic = algorithmic bytes on every pass; L1 hit climbs from ~19 % to ~86 % as the graph shrinks (local ids);
  the late passes are latency. Hook + jump of the first two rounds move ≈ 1 GB at 0.6–0.7 of the HBM peak.""",
    "dense": """* The light extraction reads 2,147 MB (all 134 M records) and writes ~1 M light records at ~7 TB/s cold; live
  0.95 of the measured peak.""",
    "grid64": """* `k_small_msf` holds the whole graph in shared memory and runs all 6 rounds in one launch.""",
}
for w in ["rmat22", "uniform", "road", "dense", "grid64"]:
    d = json.load(open(f"profiles/r02s2_bench_{w}.json"))
    out.append(f"\n## {w} ({d['value'] / 1e9:.2f} G edges/s, {d['ms_per_step']:.4f} ms/step)\n")
    out.append(sh(f"python tools/launch_share.py profiles/r02s2_launches_{w}.csv 7 --run-only | head -16"))
    out.append(sh(f"python tools/ncu_summary.py profiles/r02s2_ncu_raw_{w}.csv.gz"))
    out.append(notes[w])
open("profiles/r02s2_ncu_summary.md", "w").write("\n".join(out) + "\n")
