"""Per-call DRAM traffic of the SpMM (all kernels of one rdm_spmm call: tile
colmax/panels, hub tiles, short-row and long-row CSR kernels, heavy-row
reduce) from an `ncu --page raw --csv` export of a capture that starts at the
first SpMM-call kernel of an epoch.  Calls are delimited by the long-row
kernel (`spmm_kernel<`), which every call launches last but the heavy reduce.
Writes/updates profiles/r2_spmm_traffic.json: {workload: {"w<width>": GB}}.
Usage: python tools/spmm_traffic.py <raw.csv> <workload name> <w1,w2,...> <capture description>"""
import csv, json, os, sys
rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 5]
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
if "Metric Name" in rows[0]:
    # long format (ncu --metrics … --csv --log-file): one row per (launch, metric)
    h0 = rows[0]
    ii, ki, mi, ui, vi = (h0.index(x) for x in ("ID", "Kernel Name", "Metric Name", "Metric Unit", "Metric Value"))
    launches = {}
    for r in rows[1:]:
        d = launches.setdefault(r[ii], {"Kernel Name": r[ki]})
        d[r[mi]] = float(r[vi].replace(",", "")) * SCALE.get(r[ui], 1)
    h = ["Kernel Name", "dram__bytes_read.sum", "dram__bytes_write.sum"]
    units = ["", "byte", "byte"]
    data = [[d["Kernel Name"], str(d.get(h[1], 0.0)), str(d.get(h[2], 0.0))]
            for _, d in sorted(launches.items(), key=lambda kv: int(kv[0]))]
else:
    h, units, data = rows[0], rows[1], rows[2:]
def val(d, name):
    v = d[h.index(name)].replace(",", "")
    u = units[h.index(name)]
    x = float(v)
    return x * SCALE.get(u, 1)
widths = [int(x) for x in sys.argv[3].split(",")]
calls, cur = [], 0.0
for d in data:
    name = d[h.index("Kernel Name")]
    cur += val(d, "dram__bytes_read.sum") + val(d, "dram__bytes_write.sum")
    if "spmm_kernel<" in name:
        calls.append(cur)
        cur = 0.0
out_path = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles", "r2_spmm_traffic.json")
js = json.load(open(out_path)) if os.path.exists(out_path) else {}
js[sys.argv[2]] = {"per_width_gb": {f"w{w}": c / 1e9 for w, c in zip(widths, calls)},
                   "source": sys.argv[4]}
json.dump(js, open(out_path, "w"), indent=1)
print(js[sys.argv[2]])
