"""Per-launch table from an `ncu --page raw --csv` export (gzip): duration, DRAM bytes, L2/L1
hit rates, issue activity, occupancy, L2 throughput and L2 request mix. Usage:
python tools/ncu_summary.py raw_<wl>.csv.gz"""
import csv, gzip, io, sys

COLS = [("us", "gpu__time_duration.sum", 1e-3), ("DRAM MB", None, None),
        ("L2 hit %", "lts__t_sector_hit_rate.pct", 1), ("L1 hit %", "l1tex__t_sector_hit_rate.pct", 1),
        ("issue %", "sm__inst_issued.avg.pct_of_peak_sustained_active", 1),
        ("warps %", "sm__warps_active.avg.pct_of_peak_sustained_active", 1),
        ("L2 thr %", "lts__throughput.avg.pct_of_peak_sustained_elapsed", 1),
        ("L2 rd req M", "lts__t_requests_srcunit_tex_op_read.sum", 1e-6),
        ("L2 red req M", "lts__t_requests_srcunit_tex_op_red.sum", 1e-6),
        ("L2 atom req M", "lts__t_requests_srcunit_tex_op_atom_dot_alu.sum", 1e-6)]


def num(x):
    try:
        return float(x.replace(",", ""))
    except ValueError:
        return float("nan")


def main(path):
    rows = list(csv.reader(io.TextIOWrapper(gzip.open(path))))
    h = rows[0]
    units = rows[1]
    ix = {c: i for i, c in enumerate(h)}
    name = ix["Kernel Name"]
    print("| kernel | " + " | ".join(c[0] for c in COLS) + " |")
    print("|---" * (len(COLS) + 1) + "|")
    for r in rows[2:]:
        out = []
        for lab, col, sc in COLS:
            if lab == "DRAM MB":
                sc = {"byte": 1e-6, "Kbyte": 1e-3, "Mbyte": 1, "Gbyte": 1e3}
                v = sum(num(r[ix[c]]) * sc.get(units[ix[c]], 1e-6)
                        for c in ("dram__bytes_read.sum", "dram__bytes_write.sum"))
                out.append(f"{v:.1f}")
                continue
            v = num(r[ix[col]])
            if lab == "us":
                u = units[ix[col]]
                sc = {"ns": 1e-3, "nsecond": 1e-3, "us": 1, "usecond": 1, "ms": 1e3,
                      "msecond": 1e3}.get(u, 1e-3)
            out.append(f"{v * sc:.1f}")
        k = r[name].split("(")[0].replace("void ", "")
        print(f"| `{k}` | " + " | ".join(out) + " |")


if __name__ == "__main__":
    main(sys.argv[1])
