# round 2, call m: paired int8 hub tiles — tile tests, per-call timing paired vs single, Reddit bench
set -x
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_ops.py tests/test_gpu_fast.py -m gpu -x -q -k "tiles" > gpurun_out/r2m_pytest_tiles.txt 2>&1; echo "rc=$?" >> gpurun_out/r2m_pytest_tiles.txt
cat > /tmp/pairs.py <<'PY'
import os, sys, torch
sys.path.insert(0, '.')
import paper_conf_ipps_kurtysps23_b200 as rdm, synth
dev = torch.device('cuda:0')
for wlname in ['reddit', 'products']:
    wl = synth.WORKLOADS[wlname]; g = synth.make_graph(wl)
    ctx = rdm.Context(device=0); ctx.set_graph(g.rowptr, g.col, g.val, symmetric=True)
    def timeit(fn, it=5):
        fn(); torch.cuda.synchronize(); s = torch.cuda.Event(enable_timing=True); e = torch.cuda.Event(enable_timing=True)
        s.record(); [fn() for _ in range(it)]; e.record(); torch.cuda.synchronize(); return s.elapsed_time(e) / it
    for prec in ['fp32', 'fast']:
        ctx.set_precision(prec)
        for w in ([128, 41, 16] if wlname == 'reddit' else [256, 100, 47]):
            X = torch.randn(g.n, (w + 3) // 4 * 4, device=dev)
            res = []
            ref = None
            for pr in ['0', '1']:
                os.environ['RDM_TILE_PAIRS'] = pr
                O = torch.zeros_like(X)
                ms = timeit(lambda: ctx.spmm(0, X, O, w))
                if ref is None: ref = O.clone(); err = 0.0
                else: err = float((O[:, :w] - ref[:, :w]).abs().max() / ref[:, :w].abs().max())
                res.append(f"pairs={pr}: {ms:.3f} ms (diff {err:.1e})")
            print(wlname, prec, f"w{w}", " | ".join(res), flush=True)
PY
timeout 900 python /tmp/pairs.py > gpurun_out/r2m_pairs.txt 2>&1
timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/r2m_bench.json 2> gpurun_out/r2m_bench.err
echo done
