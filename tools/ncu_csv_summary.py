"""Summarise an `ncu --page raw --csv` export: one line per kernel launch with
duration, DRAM bytes, L2/L1 hit rates and throughputs, tensor-pipe activity."""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
h, units, data = rows[0], rows[1], rows[2:]
cols = [("gpu__time_duration.sum", "us", 1e-3), ("dram__bytes_read.sum", "MB_rd", None),
        ("dram__bytes_write.sum", "MB_wr", None), ("lts__t_sector_hit_rate.pct", "L2hit%", 1),
        ("lts__throughput.avg.pct_of_peak_sustained_elapsed", "L2thr%", 1),
        ("l1tex__throughput.avg.pct_of_peak_sustained_active", "L1thr%", 1),
        ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "SMthr%", 1),
        ("sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active", "TC%", 1),
        ("gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed", "MEM%", 1)]
def val(d, name):
    if name not in h:
        return None
    v = d[h.index(name)].replace(",", "")
    u = units[h.index(name)]
    try:
        x = float(v)
    except ValueError:
        return None
    if name.startswith("dram__bytes"):
        x *= {"byte": 1e-6, "Kbyte": 1e-3, "Mbyte": 1, "Gbyte": 1e3}.get(u, 1)
    if name == "gpu__time_duration.sum":
        x *= {"ns": 1e-3, "us": 1, "usecond": 1, "ms": 1e3, "msecond": 1e3}.get(u, 1)
    return x
print("| kernel | " + " | ".join(c[1] for c in cols) + " |")
print("|---" * (len(cols) + 1) + "|")
for d in data:
    name = d[h.index("Kernel Name")].split("(")[0].replace("rdm::<unnamed>::", "").replace("void ", "")
    vals = [val(d, c[0]) for c in cols]
    print(f"| {name[:40]} | " + " | ".join("" if v is None else f"{v:.1f}" for v in vals) + " |")
