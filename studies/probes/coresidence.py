"""Probe: which staging kernels co-run under the persistent c5 update?  The
update (M = Nc = 49152, K = 2048, F16X3, default variant) on stream 1; each
candidate on stream 2 right after it starts; prints when the candidate ended
relative to the update's end (negative = it ran under the update)."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", ".."))
import torch  # noqa: E402

import paper_conf_cluster_zhongrl12_b200 as pkg  # noqa: E402

N, K = 49152, 2048
dev = "cuda"
src = torch.empty((K, N), dtype=torch.float32, device=dev)
pkg.k_fill_synthetic(src, pkg.FPM_F32, N, 6, N, 0, 0, K, N)
srcA = torch.empty((N, K), dtype=torch.float32, device=dev)
pkg.k_fill_synthetic(srcA, pkg.FPM_F32, K, 5, N, 0, 0, N, K)
ah = torch.empty((N, K), dtype=torch.float16, device=dev)
al, bh, bl = torch.empty_like(ah), torch.empty_like(ah), torch.empty_like(ah)
ah2, al2, bh2, bl2 = (torch.empty_like(ah) for _ in range(4))
sa, sb, sa2, sb2 = (torch.empty(N, dtype=torch.float32, device=dev) for _ in range(4))
C = torch.zeros((N, N), dtype=torch.float32, device=dev)
pkg.k_split_f32(srcA, K, N, K, pkg.SCHEME_F16X3, ah, al, sa)
pkg.k_split_cols_f32(src, N, K, N, pkg.SCHEME_F16X3, bh, bl, sb)
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
small = torch.empty(1 << 20, dtype=torch.float32, device=dev)
cands = {
    "split_rows": lambda st: pkg.k_split_f32(srcA, K, N, K, pkg.SCHEME_F16X3, ah2, al2, sa2, stream=st),
    "split_cols(memset+colmax+split+scale)": lambda st: pkg.k_split_cols_f32(src, N, K, N, pkg.SCHEME_F16X3, bh2,
                                                                           bl2, sb2, stream=st),
    "torch fill (1M floats)": None,
}
out = {}
for name, fn in cands.items():
    for rep in range(3):
        torch.cuda.synchronize()
        e = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
        e[0].record(s1)
        pkg.k_update_f32(ah, al, bh, bl, sa, sb, C, N, N, K, N, stream=s1.cuda_stream)
        e[1].record(s1)
        time.sleep(0.002)     # the update is resident on every SM by now
        e[2].record(s2)
        if fn is None:
            with torch.cuda.stream(s2):
                small.fill_(1.0)
        else:
            fn(s2.cuda_stream)
        e[3].record(s2)
        torch.cuda.synchronize()
        out.setdefault(name, []).append({"update_ms": e[0].elapsed_time(e[1]),
                                         "cand_ms": e[2].elapsed_time(e[3]),
                                         "cand_end_minus_update_end_ms": e[1].elapsed_time(e[3])})
print(json.dumps(out, indent=1))
