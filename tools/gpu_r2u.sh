# round 2, call u: int8 tiles with A in shared memory (ss MMAs) vs TMEM (ts) — tests and per-call timing
set -x
mkdir -p gpurun_out
RDM_TILE_ASMEM=1 timeout 900 python -m pytest tests/test_gpu_ops.py tests/test_gpu_fast.py -m gpu -x -q -k "tiles" > gpurun_out/r2u_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/r2u_pytest.txt
cat > /tmp/asm.py <<'PY'
import os, sys, torch
sys.path.insert(0, '.')
import paper_conf_ipps_kurtysps23_b200 as rdm, synth
dev = torch.device('cuda:0')
for wlname, widths in [('reddit', [128, 41, 16]), ('products', [256, 100, 47])]:
    wl = synth.WORKLOADS[wlname]; g = synth.make_graph(wl)
    ctx = rdm.Context(device=0); ctx.set_graph(g.rowptr, g.col, g.val, symmetric=True)
    def timeit(fn, it=10):
        fn(); torch.cuda.synchronize(); s = torch.cuda.Event(enable_timing=True); e = torch.cuda.Event(enable_timing=True)
        s.record(); [fn() for _ in range(it)]; e.record(); torch.cuda.synchronize(); return s.elapsed_time(e) / it
    for prec in ['fp32', 'fast']:
        ctx.set_precision(prec)
        for w in widths:
            X = torch.randn(g.n, (w + 3) // 4 * 4, device=dev)
            res = []; ref = None
            for v in ['0', '1']:
                os.environ['RDM_TILE_ASMEM'] = v
                O = torch.zeros_like(X)
                ms = timeit(lambda: ctx.spmm(0, X, O, w))
                if ref is None: ref = O.clone(); err = 0.0
                else: err = float((O[:, :w] - ref[:, :w]).abs().max() / ref[:, :w].abs().max())
                res.append(f"asmem={v}: {ms:.3f} ms (diff {err:.1e})")
            print(wlname, prec, f"w{w}", " | ".join(res), flush=True)
    del ctx
PY
timeout 900 python /tmp/asm.py > gpurun_out/r2u_asm.txt 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"hub_tile" -c 6 --csv --log-file gpurun_out/r2u_launches.csv env RDM_TILE_ASMEM=1 python bench.py --steps 1 --warmup 1 --no-e2e --no-variants --no-cpu-baseline > gpurun_out/r2u_ncu.log 2>&1
echo done
