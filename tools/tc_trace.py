"""Timeline of CTA 0 of the tcgen05 GEMM (lib/librdm_trace.so, built with
-DRDM_TC_TRACE): per k-block the producer's issue (after its empty wait), the
converter's full-wait return and conv arrive, the MMA issuer's conv-wait return;
per tile the commit, the epilogue's tfull-wait return and tempty arrive.
Prints per-interval medians in SM cycles."""
import os, sys, ctypes, numpy as np, torch
os.environ['RDM_LIB_VARIANT'] = 'trace'
sys.path.insert(0, '.')
import paper_conf_ipps_kurtysps23_b200 as rdm
lib = rdm._lib
lib.rdm_debug_tc_trace.argtypes = [ctypes.c_void_p, ctypes.c_int]
dev = torch.device('cuda:0'); ctx = rdm.Context(device=0)
rows = 232965
def run(name, op, k, m, env):
    for kk, vv in env.items(): os.environ[kk] = vv
    ldk, ldm = (k + 3) // 4 * 4, (m + 3) // 4 * 4
    if op == rdm.GEMM_NN:
        X = torch.randn(rows, ldk, device=dev); C = torch.zeros(rows, ldm, device=dev)
    else:
        X = torch.randn(rows, ldm, device=dev); C = torch.zeros(rows, ldk, device=dev)
    W = torch.randn(k, m, device=dev)
    for _ in range(3): ctx.gemm(op, X, W, C, rows, k, m)
    ctx.sync()
    buf = np.zeros(8 * 4096, dtype=np.int64)
    n = lib.rdm_debug_tc_trace(buf.ctypes.data, buf.size)
    t = buf.reshape(8, 4096)
    for kk in env: os.environ.pop(kk)
    nk = int((t[0] > 0).sum()); nt = int((t[4] > 0).sum())
    base = t[0][0]
    ev = [t[i][:nk] - base for i in range(4)]
    tiles = [t[i][:nt] - base for i in (4, 5, 6)]
    med = lambda a: float(np.median(a)) if len(a) else float('nan')
    print(f"== {name}: {nk} k-blocks, {nt} tiles on CTA 0, span {int(max(ev[3].max(), tiles[2].max() if nt else 0))} cycles")
    print(f"   producer issue cadence      {med(np.diff(ev[0])):8.0f}   (empty-wait bound when > converter cadence)")
    print(f"   TMA latency (issue->full)   {med(ev[1]-ev[0]):8.0f}")
    print(f"   convert (full->conv arrive) {med(ev[2]-ev[1]):8.0f}")
    print(f"   conv arrive -> MMA wakes    {med(ev[3]-ev[2]):8.0f}")
    print(f"   MMA issue cadence           {med(np.diff(ev[3])):8.0f}")
    print(f"   converter cadence           {med(np.diff(ev[1])):8.0f}")
    if nt > 1:
        print(f"   tile cadence (commit)       {med(np.diff(tiles[0])):8.0f}")
        print(f"   commit -> epilogue wakes    {med(tiles[1]-tiles[0]):8.0f}")
        print(f"   epilogue (tfull->tempty)    {med(tiles[2]-tiles[1]):8.0f}")
    print("   first 12 k-blocks [issue, full, conv, mma]:")
    for i in range(min(12, nk)):
        print("    ", [int(ev[j][i]) for j in range(4)])
for name, op, k, m, env in [
        ('NN 602->128 pair ASM', rdm.GEMM_NN, 602, 128, {}),
        ('NN 602->128 single', rdm.GEMM_NN, 602, 128, {'RDM_PAIR': '0'}),
        ('NN 128->41 pair ASM', rdm.GEMM_NN, 128, 41, {}),
        ('NN 128->41 single', rdm.GEMM_NN, 128, 41, {'RDM_PAIR': '0'}),
        ('NT 41->128 single', rdm.GEMM_NT, 128, 41, {}),
        ('NT 128->602 single', rdm.GEMM_NT, 602, 128, {})]:
    run(name, op, k, m, env)
