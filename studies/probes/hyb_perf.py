"""Update kernel alone, sustained (power-capped): F16X3 vs F16I8 at the c5
launch shape (M = Nc = N, K = 2048), clocks and power sampled; checks the
F16I8 result against F16X3 on the same operands (rel-Fro of the difference)."""
import json, os, statistics, subprocess, sys, threading, time
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", ".."))
import torch
import paper_conf_cluster_zhongrl12_b200 as pkg

def sampler(stop, rows):
    p = subprocess.Popen(["nvidia-smi", "--query-gpu=clocks.sm,power.draw", "--format=csv,noheader,nounits", "-lms", "100"],
                         stdout=subprocess.PIPE, text=True)
    while not stop.is_set():
        line = p.stdout.readline()
        if line:
            rows.append([float(x) for x in line.split(",")])
    p.kill()

def run(name, fn, flops, secs=4.0):
    s = torch.cuda.current_stream()
    for _ in range(2): fn()
    torch.cuda.synchronize()
    rows, stop = [], threading.Event()
    th = threading.Thread(target=sampler, args=(stop, rows)); th.start(); time.sleep(0.3)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    n = 0; t0 = time.time(); e0.record(s)
    while time.time() - t0 < secs:
        for _ in range(3): fn()
        n += 3; torch.cuda.synchronize()
    e1.record(s); torch.cuda.synchronize(); stop.set(); th.join()
    ms = e0.elapsed_time(e1) / n
    load = [r for r in rows if r[1] > 300]
    out = {"name": name, "ms": ms, "tflops": flops / ms / 1e9, "sm_mhz": statistics.median([r[0] for r in load]) if load else None,
           "power_w": statistics.median([r[1] for r in load]) if load else None}
    print(json.dumps(out), flush=True)
    return out

N = int(sys.argv[1]) if len(sys.argv) > 1 else 49152
K = int(sys.argv[2]) if len(sys.argv) > 2 else 2048
dev = "cuda"
srcA = torch.empty((N, K), dtype=torch.float32, device=dev); pkg.k_fill_synthetic(srcA, pkg.FPM_F32, K, 5, N, 0, 0, N, K)
srcB = torch.empty((K, N), dtype=torch.float32, device=dev); pkg.k_fill_synthetic(srcB, pkg.FPM_F32, N, 6, N, 0, 0, K, N)
ah = torch.empty((N, K), dtype=torch.float16, device=dev); al = torch.empty_like(ah)
bh = torch.empty((N, K), dtype=torch.float16, device=dev); bl = torch.empty_like(bh)
sa = torch.empty(N, device=dev); sb = torch.empty(N, device=dev)
C = torch.zeros((N, N), dtype=torch.float32, device=dev)
res = []
for scheme, name in ((pkg.SCHEME_F16X3, "F16X3"), (pkg.SCHEME_F16I8, "F16I8"), (pkg.SCHEME_F16X3, "F16X3"), (pkg.SCHEME_F16I8, "F16I8")):
    pkg.k_split_f32(srcA, K, N, K, scheme, ah, al, sa)
    pkg.k_split_cols_f32(srcB, N, K, N, scheme, bh, bl, sb)
    for v in ((6, 9, 10, 11) if scheme == pkg.SCHEME_F16I8 else (-1,)):
        res.append(run(f"{name} v{v}", lambda: pkg.k_update_f32(ah, al, bh, bl, sa, sb, C, N, N, K, N, scheme=scheme, variant=v),
                       2 * N * N * K))
# parity of the two schemes on one launch (overwrite mode)
M2 = min(N, 8192)
outs = []
for scheme in (pkg.SCHEME_F16X3, pkg.SCHEME_F16I8):
    pkg.k_split_f32(srcA, K, N, K, scheme, ah, al, sa)
    pkg.k_split_cols_f32(srcB, N, K, N, scheme, bh, bl, sb)
    pkg.k_update_f32(ah, al, bh, bl, sa, sb, C, N, N, K, N, scheme=scheme, accumulate=False)
    outs.append(C[:M2, :M2].double().clone())
ref = srcA[:M2].double() @ srcB[:, :M2].double()
for o, nm in zip(outs, ("F16X3", "F16I8")):
    print(nm, "rel-Fro vs fp64 (first 8192^2 block):", float(torch.linalg.norm(o - ref) / torch.linalg.norm(ref)))
os.makedirs("gpurun_out", exist_ok=True)
json.dump(res, open("gpurun_out/hyb_perf.json", "w"), indent=1)

# MMA-issuer wait counters (fpm_k_prof) over 5 launches of the default F16I8 kernel
pkg.k_split_f32(srcA, K, N, K, pkg.SCHEME_F16I8, ah, al, sa)
pkg.k_split_cols_f32(srcB, N, K, N, pkg.SCHEME_F16I8, bh, bl, sb)
for v in (0, 6):
    torch.cuda.synchronize(); pkg.k_prof(1)
    for _ in range(5):
        pkg.k_update_f32(ah, al, bh, bl, sa, sb, C, N, N, K, N, scheme=pkg.SCHEME_F16I8, variant=v)
    torch.cuda.synchronize(); pr = pkg.k_prof(2); pkg.k_prof(0)
    print(f"variant {v}: issuer waits TMEM {pr['tmem_wait'] / pr['issuer']:.3f}, operands {pr['operand_wait'] / pr['issuer']:.3f}"
          f" of its loop; {pr['tiles']} tiles", flush=True)
