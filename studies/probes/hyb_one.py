"""One update launch per scheme (F16X3, F16I8) at M = Nc = N, K (for ncu captures)."""
import os, sys
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", ".."))
import torch
import paper_conf_cluster_zhongrl12_b200 as pkg
N = int(sys.argv[1]) if len(sys.argv) > 1 else 16384
K = int(sys.argv[2]) if len(sys.argv) > 2 else 2048
dev = "cuda"
srcA = torch.empty((N, K), dtype=torch.float32, device=dev); pkg.k_fill_synthetic(srcA, pkg.FPM_F32, K, 5, N, 0, 0, N, K)
srcB = torch.empty((K, N), dtype=torch.float32, device=dev); pkg.k_fill_synthetic(srcB, pkg.FPM_F32, N, 6, N, 0, 0, K, N)
ah = torch.empty((N, K), dtype=torch.float16, device=dev); al = torch.empty_like(ah)
bh = torch.empty((N, K), dtype=torch.float16, device=dev); bl = torch.empty_like(bh)
sa = torch.empty(N, device=dev); sb = torch.empty(N, device=dev)
C = torch.zeros((N, N), dtype=torch.float32, device=dev)
for scheme in (pkg.SCHEME_F16X3, pkg.SCHEME_F16I8):
    pkg.k_split_f32(srcA, K, N, K, scheme, ah, al, sa)
    pkg.k_split_cols_f32(srcB, N, K, N, scheme, bh, bl, sb)
    for _ in range(2):
        pkg.k_update_f32(ah, al, bh, bl, sa, sb, C, N, N, K, N, scheme=scheme)
torch.cuda.synchronize()
print("done")
