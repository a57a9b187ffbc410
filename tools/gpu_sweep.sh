timeout 1200 python -m pytest tests -m gpu -q -x 2>&1 | tail -2
timeout 900 python bench.py --steps 10 --warmup 3 --sweep --no-e2e --no-cpu-baseline > gpurun_out/sweep_reddit.json 2>gpurun_out/sweep_reddit.err; echo rc=$?
timeout 1200 python bench.py --workload products --steps 10 --warmup 3 --sweep --no-e2e --no-cpu-baseline > gpurun_out/sweep_products.json 2>gpurun_out/sweep_products.err; echo rc=$?
python - <<'PY'
import json
for w in ("reddit", "products"):
    try:
        d = json.loads(open(f"gpurun_out/sweep_{w}.json").read().strip().splitlines()[-1])
    except Exception as e:
        print(w, "failed", e); continue
    c = d["config"]; sw = c["sweep_ms"]
    best = min(sw, key=lambda k: sw[k])
    print(w, "picked", c["config_id"], c["config_name"], "epoch", round(d["value"], 3), "pareto", c["pareto"], "fastest", best, sw[best])
    print("  ", {k: sw[k] for k in sorted(sw, key=lambda k: sw[k])[:8]})
PY
