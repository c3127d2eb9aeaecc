"""Probe: co-residence under the persistent c5 update as a function of the
co-running kernel's CTA size and registers (coprobe.cu: a float4 copy of
256 MB).  Prints, per (registers, CTA size), when the copy ended relative to
the update's end (negative = it ran under the update) and its duration."""
import ctypes
import json
import os
import sys
import time

HERE = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, os.path.join(HERE, "..", ".."))
import torch  # noqa: E402

import paper_conf_cluster_zhongrl12_b200 as pkg  # noqa: E402

lib = ctypes.CDLL(os.path.join(HERE, "libcoprobe.so"))
lib.coprobe_launch.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p,
                               ctypes.c_int64, ctypes.c_void_p, ctypes.c_int]
N, K = 49152, 2048
dev = "cuda"
ah = torch.zeros((N, K), dtype=torch.float16, device=dev)
al, bh, bl = torch.zeros_like(ah), torch.zeros_like(ah), torch.zeros_like(ah)
sa, sb = (torch.ones(N, dtype=torch.float32, device=dev) for _ in range(2))
C = torch.zeros((N, N), dtype=torch.float32, device=dev)
src = torch.ones(1 << 26, dtype=torch.float32, device=dev)
dst = torch.empty_like(src)
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
variant = int(os.environ.get("VARIANT", "-1"))
carveout = int(os.environ.get("CARVEOUT", "-1"))
pads = [int(x) for x in os.environ.get("PADS", "1,24,48").split(",")]
blocks = [int(x) for x in os.environ.get("BLOCKS", "32,64,128,256").split(",")]
out = []
for pad in pads:
    for block in blocks:
        rows = []
        for rep in range(2):
            torch.cuda.synchronize()
            e = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
            e[0].record(s1)
            pkg.k_update_f32(ah, al, bh, bl, sa, sb, C, N, N, K, N, variant=variant, stream=s1.cuda_stream)
            e[1].record(s1)
            time.sleep(0.003)
            e[2].record(s2)
            rc = lib.coprobe_launch(pad, block, 148 * 4, src.data_ptr(), dst.data_ptr(), src.numel() // 4,
                                    ctypes.c_void_p(s2.cuda_stream), carveout)
            e[3].record(s2)
            torch.cuda.synchronize()
            rows.append((e[1].elapsed_time(e[3]), e[2].elapsed_time(e[3]), e[0].elapsed_time(e[1]), rc))
        out.append({"variant": variant, "carveout": carveout, "pad": pad, "block": block, "end_minus_update_end_ms": [r[0] for r in rows],
                    "copy_ms": [r[1] for r in rows], "update_ms": [r[2] for r in rows], "rc": rows[-1][3]})
        print(out[-1], file=sys.stderr, flush=True)
print(json.dumps(out))
