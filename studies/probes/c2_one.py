"""Config 2 profiling helper: one update launch C (L x L) += A (L x K) B (K x L)
per L given, after the staging (for ncu -k regex:update_kernel)."""
import os
import sys

sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", ".."))
import torch  # noqa: E402

import paper_conf_cluster_zhongrl12_b200 as pkg  # noqa: E402

K = int(os.environ.get("K", "512"))
for L in [int(x) for x in sys.argv[1:]] or [8192, 16384]:
    A = torch.empty((L, K), device="cuda")
    B = torch.empty((K, L), device="cuda")
    pkg.k_fill_synthetic(A, pkg.FPM_F32, K, 1, 1 << 20, 0, 0, L, K)
    pkg.k_fill_synthetic(B, pkg.FPM_F32, L, 2, 1 << 20, 0, 0, K, L)
    ah = torch.empty((L, K), dtype=torch.float16, device="cuda")
    al, bh, bl = torch.empty_like(ah), torch.empty_like(ah), torch.empty_like(ah)
    sa, sb = torch.empty(L, device="cuda"), torch.empty(L, device="cuda")
    pkg.k_split_f32(A, K, L, K, pkg.SCHEME_F16X3, ah, al, sa)
    pkg.k_split_cols_f32(B, L, K, L, pkg.SCHEME_F16X3, bh, bl, sb)
    C = torch.zeros((L, L), device="cuda")
    pkg.k_update_f32(ah, al, bh, bl, sa, sb, C, L, L, K, L)
    torch.cuda.synchronize()
    print(f"L={L} K={K} done", flush=True)
