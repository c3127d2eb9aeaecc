"""Probe: the c5 update launch (M = Nc = 49152, K = 2048, F16X3) back to back
on one stream, alone, vs inside the k-loop (staging co-running); and the
staging kernels alone.  Prints ms per launch."""
import os
import sys

sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", ".."))
import torch  # noqa: E402

import paper_conf_cluster_zhongrl12_b200 as pkg  # noqa: E402

N, K = 49152, 2048
dev = "cuda"
src = torch.empty((K, N), dtype=torch.float32, device=dev)     # B block-rows (K x W)
pkg.k_fill_synthetic(src, pkg.FPM_F32, N, 6, N, 0, 0, K, N)
srcA = torch.empty((N, K), dtype=torch.float32, device=dev)    # A panel (H x K)
pkg.k_fill_synthetic(srcA, pkg.FPM_F32, K, 5, N, 0, 0, N, K)
ah = torch.empty((N, K), dtype=torch.float16, device=dev)
al = torch.empty_like(ah)
bh = torch.empty((N, K), dtype=torch.float16, device=dev)
bl = torch.empty_like(bh)
sa = torch.empty(N, dtype=torch.float32, device=dev)
sb = torch.empty(N, dtype=torch.float32, device=dev)
C = torch.zeros((N, N), dtype=torch.float32, device=dev)
s = torch.cuda.current_stream()


def timeit(fn, reps):
    for _ in range(2):
        fn()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record(s)
    for _ in range(reps):
        fn()
    e1.record(s)
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


t_rows = timeit(lambda: pkg.k_split_f32(srcA, K, N, K, pkg.SCHEME_F16X3, ah, al, sa, stream=s.cuda_stream), 10)
t_cols = timeit(lambda: pkg.k_split_cols_f32(src, N, K, N, pkg.SCHEME_F16X3, bh, bl, sb, stream=s.cuda_stream), 10)
print(f"split_rows (H x 2048 -> halves): {t_rows:.3f} ms = {2 * N * K * 4 / t_rows / 1e6:.0f} GB/s", flush=True)
print(f"split_cols (2048 x W -> transposed halves): {t_cols:.3f} ms = {2 * N * K * 4 / t_cols / 1e6:.0f} GB/s",
      flush=True)
for v in (-1, 2):
    t_upd = timeit(lambda: pkg.k_update_f32(ah, al, bh, bl, sa, sb, C, N, N, K, N, variant=v, stream=s.cuda_stream), 24)
    print(f"update alone variant {v}: {t_upd:.3f} ms/launch = {2 * N * N * K / t_upd / 1e9:.1f} TFLOP/s", flush=True)

# co-residence: the update on one stream, the staging kernels on another
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
for v in (-1, 2):
    torch.cuda.synchronize()
    e = [torch.cuda.Event(enable_timing=True) for _ in range(5)]
    e[0].record(s1)
    pkg.k_update_f32(ah, al, bh, bl, sa, sb, C, N, N, K, N, variant=v, stream=s1.cuda_stream)
    e[1].record(s1)
    e[2].record(s2)
    pkg.k_split_cols_f32(src, N, K, N, pkg.SCHEME_F16X3, bh, bl, sb, stream=s2.cuda_stream)
    e[3].record(s2)
    pkg.k_split_f32(srcA, K, N, K, pkg.SCHEME_F16X3, ah, al, sa, stream=s2.cuda_stream)
    e[4].record(s2)
    torch.cuda.synchronize()
    print(f"variant {v}: update {e[0].elapsed_time(e[1]):.3f} ms; co-running split_cols {e[2].elapsed_time(e[3]):.3f} ms, "
          f"split_rows {e[3].elapsed_time(e[4]):.3f} ms; split_cols started {e[0].elapsed_time(e[2]):.3f} ms after the update",
          flush=True)
