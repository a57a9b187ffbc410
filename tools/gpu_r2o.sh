# round 2, call o: int8 tile kernel with the MMAs skipped (RDM_TILE_DBG=1) vs on — is the tensor pipe the bound?
set -x
mkdir -p gpurun_out
cat > /tmp/dbg.py <<'PY'
import os, sys, torch
sys.path.insert(0, '.')
import paper_conf_ipps_kurtysps23_b200 as rdm, synth
dev = torch.device('cuda:0')
wl = synth.WORKLOADS['reddit']; g = synth.make_graph(wl)
os.environ['RDM_TILE_MIN_NNZ'] = '400'
ctx = rdm.Context(device=0); ctx.set_graph(g.rowptr, g.col, g.val, symmetric=True)
def timeit(fn, it=10):
    fn(); torch.cuda.synchronize(); s = torch.cuda.Event(enable_timing=True); e = torch.cuda.Event(enable_timing=True)
    s.record(); [fn() for _ in range(it)]; e.record(); torch.cuda.synchronize(); return s.elapsed_time(e) / it
for w in [128, 41]:
    X = torch.randn(g.n, (w + 3) // 4 * 4, device=dev)
    for dbg in ['0', '1']:
        os.environ['RDM_TILE_DBG'] = dbg
        O = torch.zeros_like(X)
        print(f"w{w} dbg={dbg}: {timeit(lambda: ctx.spmm(0, X, O, w)):.3f} ms", flush=True)
    os.environ['RDM_TILE_DBG'] = '0'
    os.environ['RDM_NO_TILES_CALL'] = '1'
PY
timeout 600 python /tmp/dbg.py > gpurun_out/r2o_dbg.txt 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"hub_tile" -c 8 --csv --log-file gpurun_out/r2o_launches.csv env RDM_TILE_DBG=1 python /tmp/dbg.py > gpurun_out/r2o_ncu.log 2>&1
echo done
