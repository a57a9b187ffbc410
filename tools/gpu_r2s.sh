# round 2, call s: evict-first SpMM output stores (RDM_SPMM_STCS) and the GEMM's A prefetch (RDM_PF) on products / Reddit
set -x
mkdir -p gpurun_out
cat > /tmp/stcs.py <<'PY'
import os, sys, torch
sys.path.insert(0, '.')
import paper_conf_ipps_kurtysps23_b200 as rdm, synth
dev = torch.device('cuda:0')
for wlname, widths in [('products', [256, 100, 47]), ('reddit', [128, 41])]:
    wl = synth.WORKLOADS[wlname]; g = synth.make_graph(wl)
    ctx = rdm.Context(device=0); ctx.set_graph(g.rowptr, g.col, g.val, symmetric=True)
    def timeit(fn, it=5):
        fn(); torch.cuda.synchronize(); s = torch.cuda.Event(enable_timing=True); e = torch.cuda.Event(enable_timing=True)
        s.record(); [fn() for _ in range(it)]; e.record(); torch.cuda.synchronize(); return s.elapsed_time(e) / it
    for w in widths:
        X = torch.randn(g.n, (w + 3) // 4 * 4, device=dev)
        res = []
        for v in ['0', '1']:
            os.environ['RDM_SPMM_STCS'] = v
            O = torch.zeros_like(X)
            res.append(f"stcs={v}: {timeit(lambda: ctx.spmm(0, X, O, w)):.3f} ms")
        print(wlname, f"w{w}", " | ".join(res), flush=True)
    del ctx
PY
timeout 900 python /tmp/stcs.py > gpurun_out/r2s_stcs.txt 2>&1
for pf in 0 1; do RDM_PF=$pf timeout 900 python bench.py --workload products --steps 10 --warmup 3 --no-cpu-baseline --no-variants --no-e2e >> gpurun_out/r2s_pf.jsonl 2>> gpurun_out/r2s_pf.err; done
echo done
