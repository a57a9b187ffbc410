import sys, torch
sys.path.insert(0, '.')
import paper_conf_ipps_kurtysps23_b200 as rdm
dev = torch.device('cuda:0'); ctx = rdm.Context(device=0)
K, w = 16384, int(sys.argv[1]) if len(sys.argv) > 1 else 48
A = torch.randn(K, K, device=dev); B = torch.randn(K, w, device=dev); C = torch.zeros(K, w, device=dev)
for _ in range(3):
    ctx.gemm(rdm.GEMM_NN, A, B, C, K, K, w)
ctx.sync()
