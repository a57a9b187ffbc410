"""Short-row SpMM kernel A/B (current build vs lib/librdm_old.so): per-call
time at the workload widths and bitwise equality of the outputs."""
import os, sys, subprocess, json
code = r'''
import os, sys, torch, numpy as np
sys.path.insert(0, '.')
import paper_conf_ipps_kurtysps23_b200 as rdm, synth
dev = torch.device('cuda:0'); out = {}
for wlname, widths in [('reddit', [128, 41]), ('products', [256, 100, 47])]:
    wl = synth.WORKLOADS[wlname]; g = synth.make_graph(wl)
    ctx = rdm.Context(device=0); ctx.set_graph(g.rowptr, g.col, g.val, symmetric=True)
    def timeit(fn, it=10):
        fn(); torch.cuda.synchronize(); s = torch.cuda.Event(enable_timing=True); e = torch.cuda.Event(enable_timing=True)
        s.record(); [fn() for _ in range(it)]; e.record(); torch.cuda.synchronize(); return s.elapsed_time(e) / it
    for w in widths:
        X = torch.randn(g.n, (w + 3) // 4 * 4, device=dev, generator=torch.Generator(device=dev).manual_seed(w)); O = torch.zeros_like(X)
        ms = timeit(lambda: ctx.spmm(0, X, O, w))
        h = int(np.frombuffer(O.cpu().numpy().tobytes(), dtype=np.uint64).sum() % (1 << 61))
        out[f"{wlname} w{w}"] = (ms, h)
        del X, O
    del ctx
print("RESULT", __import__('json').dumps(out))
'''
res = {}
for tag in ['old', 'new', 'old', 'new']:
    env = dict(os.environ)
    if tag == 'old': env['RDM_LIB_VARIANT'] = 'old'
    p = subprocess.run([sys.executable, '-c', code], capture_output=True, text=True, env=env)
    line = [l for l in p.stdout.splitlines() if l.startswith('RESULT')]
    if not line: print(tag, 'FAILED', p.stderr[-2000:]); continue
    r = json.loads(line[0][7:])
    for k, (ms, h) in r.items():
        res.setdefault(k, []).append((tag, round(ms, 3), h))
for k, v in res.items():
    hs = {h for _, _, h in v}
    print(k, ' | '.join(f"{t}: {ms} ms" for t, ms, _ in v), '| bitwise equal' if len(hs) == 1 else '| DIFFERENT')
