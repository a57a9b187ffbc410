"""One Reddit-shaped 602-wide NN GEMM call (for ncu captures of a single launch)."""
import sys, torch
sys.path.insert(0, '.')
import paper_conf_ipps_kurtysps23_b200 as rdm
dev = torch.device('cuda:0'); ctx = rdm.Context(device=0)
rows = 232965
X = torch.randn(rows, 604, device=dev); C = torch.zeros(rows, 128, device=dev); W = torch.randn(602, 128, device=dev)
for _ in range(2):
    ctx.gemm(rdm.GEMM_NN, X, W, C, rows, 602, 128)
ctx.sync()
