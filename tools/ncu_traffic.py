"""Per-launch DRAM traffic of the A8 passes from an `ncu --set full` capture -> the
profiles/ncu_traffic_<workload>.json that bench.py reports as roofline.traffic.

    python tools/ncu_traffic.py gpurun_out/full.ncu-rep rmat22 "<capture command>"
"""
import csv
import io
import json
import subprocess
import sys

rep, wl = sys.argv[1], sys.argv[2]
cmd = sys.argv[3] if len(sys.argv) > 3 else ""
out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv", "--metrics",
                      "gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum"],
                     capture_output=True, text=True, check=True).stdout
rows = list(csv.reader(io.StringIO(out)))
h = rows[0]
units = rows[1]
i = {k: j for j, k in enumerate(h)}
scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
launches = []
for r in rows[2:]:
    name = r[i["Kernel Name"]]
    b = sum(float(r[i[k]]) * scale[units[i[k]]] for k in ("dram__bytes_read.sum", "dram__bytes_write.sum"))
    launches.append({"kernel": name.split("(")[0], "dram_bytes": b,
                     "us": float(r[i["gpu__time_duration.sum"]])})
filt = [x for x in launches if "k_arc_pass<1" in x["kernel"] or "k_arc_pass<(int)1" in x["kernel"]
        or "k_member_min" in x["kernel"]]
min0 = [x for x in launches if "k_arc_pass<0" in x["kernel"] or "k_arc_pass<(int)0" in x["kernel"]]
small = [x for x in launches if "k_small_msf" in x["kernel"]]
res = {"workload": wl, "kernel": "k_arc_pass<MODE_FILTER> (A8) / <MODE_MIN0> (A2)",
       "source": f"ncu --set full --clock-control none ({cmd})",
       "launches": launches,
       "per_launch_dram_bytes": [x["dram_bytes"] for x in filt],
       "filter_dram_bytes_per_launch": sum(x["dram_bytes"] for x in filt) / max(len(filt), 1),
       "min0_dram_bytes_per_launch": sum(x["dram_bytes"] for x in min0) / max(len(min0), 1),
       "small_dram_bytes_per_launch": sum(x["dram_bytes"] for x in small) / max(len(small), 1)}
json.dump(res, open(f"profiles/ncu_traffic_{wl}.json", "w"), indent=1)
print(json.dumps(res, indent=1))
