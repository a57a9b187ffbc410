"""Aggregate an ncu --csv launch list per kernel: share, count, mean µs."""
import collections, subprocess, sys
out = subprocess.run([sys.executable, __file__.replace("agg_launches", "launch_summary"), sys.argv[1]],
                     capture_output=True, text=True).stdout
agg = collections.OrderedDict()
for l in out.splitlines():
    p = l.split()
    us, name = float(p[0]), " ".join(p[2:])
    a = agg.setdefault(name, [0, 0.0])
    a[0] += 1
    a[1] += us
tot = sum(v[1] for v in agg.values())
for k, v in sorted(agg.items(), key=lambda x: -x[1][1])[:int(sys.argv[2]) if len(sys.argv) > 2 else 16]:
    print(f"{v[1] / tot * 100:5.1f}% n={v[0]:4d} avg={v[1] / v[0]:8.1f}us {k}")
