"""Hub-tile kernel decomposition: SpMM calls on the Reddit-shaped graph with
parts of hub_tile_i8_kernel switched off (RDM_TILE_DBG: 1 = MMAs, 2 = bit
expansion, 4 = epilogue stores); run under an ncu launch list to read the tile
kernel's own duration per setting (results are wrong by design)."""
import os, sys, torch
sys.path.insert(0, '.')
import paper_conf_ipps_kurtysps23_b200 as rdm, synth
dev = torch.device('cuda:0')
wl = synth.WORKLOADS['reddit']; g = synth.make_graph(wl)
ctx = rdm.Context(device=0); ctx.set_graph(g.rowptr, g.col, g.val, symmetric=True)
for w in (128, 41):
    X = torch.randn(g.n, (w + 3) // 4 * 4, device=dev); O = torch.zeros_like(X)
    for dbg in (sys.argv[1].split(',') if len(sys.argv) > 1 else ['0', '1', '2', '3', '4', '6', '7']):
        os.environ['RDM_TILE_DBG'] = dbg
        for _ in range(2):
            ctx.spmm(0, X, O, w)
        ctx.sync()
        print(f"w{w} dbg{dbg}", flush=True)
