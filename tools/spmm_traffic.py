"""Per-call DRAM traffic of the SpMM (all kernels of one rdm_spmm call: tile
colmax/panels, hub tiles, short-row and long-row CSR kernels, heavy-row
reduce) from an `ncu --page raw --csv` export of a capture that starts at the
first SpMM-call kernel of an epoch.  Calls are delimited by the long-row
kernel (`spmm_kernel<`), which every call launches last but the heavy reduce.
Writes/updates profiles/r2_spmm_traffic.json: {workload: {"w<width>": GB}}.
Usage: python tools/spmm_traffic.py <raw.csv> <workload name> <w1,w2,...> <capture description>"""
import csv, json, os, sys
rows = list(csv.reader(open(sys.argv[1])))
h, units, data = rows[0], rows[1], rows[2:]
def val(d, name):
    v = d[h.index(name)].replace(",", "")
    u = units[h.index(name)]
    x = float(v)
    return x * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(u, 1)
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
