"""ncu target: one FP64 update launch, L = 8192, K = 512."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import torch
import paper_conf_cluster_zhongrl12_b200 as pkg
L, K = 8192, 512
A = torch.empty((L, K), dtype=torch.float64, device="cuda")
Bt = torch.empty((L, K), dtype=torch.float64, device="cuda")
pkg.k_fill_synthetic(A, pkg.FPM_F64, K, 1, 1 << 20, 0, 0, L, K)
pkg.k_fill_synthetic(Bt, pkg.FPM_F64, K, 2, 1 << 20, 0, 0, L, K)
C = torch.zeros((L, L), dtype=torch.float64, device="cuda")
for _ in range(3):
    pkg.k_update_f64(A, K, Bt, C, L, L, K, L)
torch.cuda.synchronize()
