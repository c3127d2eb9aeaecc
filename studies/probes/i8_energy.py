"""Go/no-go probe: sustained (power-capped) rate of the tcgen05 update kernel
with kind::i8 operands (3 MMAs per k-step, s32 accumulator) vs kind::f16
(F16X3), same structure, same operand bytes per row, clocks and power sampled."""
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

def run(name, fn, ops, secs=4.0):
    s = torch.cuda.current_stream()
    for _ in range(3): fn()
    torch.cuda.synchronize()
    rows, stop = [], threading.Event()
    th = threading.Thread(target=sampler, args=(stop, rows)); th.start(); time.sleep(0.3)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    n = 0; t0 = time.time(); e0.record(s)
    while time.time() - t0 < secs:
        for _ in range(5): fn()
        n += 5; torch.cuda.synchronize()
    e1.record(s); torch.cuda.synchronize(); stop.set(); th.join()
    ms = e0.elapsed_time(e1) / n
    load = [r for r in rows if r[1] > 300]
    out = {"name": name, "ms": ms, "tops": ops / ms / 1e9, "sm_mhz": statistics.median([r[0] for r in load]) if load else None,
           "power_w": statistics.median([r[1] for r in load]) if load else None}
    print(json.dumps(out), flush=True)
    return out

M = N = int(sys.argv[1]) if len(sys.argv) > 1 else 16384
K = 2048
dev = "cuda"
g = torch.Generator(device=dev).manual_seed(0)
C = torch.zeros((M, N), dtype=torch.float32, device=dev)
sa = torch.ones(M, device=dev); sb = torch.ones(N, device=dev)
h = lambda r: ((torch.rand(r, K, device=dev, generator=g) * 2 - 1) * 2**14).half()
ah, al, bh, bl = h(M), h(M), h(N), h(N)
res = []
res.append(run("f16x3 K=2048", lambda: pkg.k_update_f32(ah, al, bh, bl, sa, sb, C, M, N, K, N, scheme=0), 3 * 2 * M * N * K))
q = lambda r, lim: torch.randint(-lim, lim + 1, (r, 2 * K), device=dev, dtype=torch.int8, generator=g)
qa, qla, qb, qlb = q(M, 127), q(M, 64), q(N, 127), q(N, 64)
res.append(run("i8x3 K=4096 (same bytes)", lambda: pkg.k_update_f32(qa, qla, qb, qlb, sa, sb, C, M, N, 2 * K, N, scheme=2),
               3 * 2 * M * N * 2 * K))
res.append(run("i8x6 K=4096 (same bytes, twice the MMAs)", lambda: pkg.k_update_f32(qa, qla, qb, qlb, sa, sb, C, M, N, 2 * K, N, scheme=2, variant=1),
               6 * 2 * M * N * 2 * K))
res.append(run("f16x3 K=2048 again", lambda: pkg.k_update_f32(ah, al, bh, bl, sa, sb, C, M, N, K, N, scheme=0), 3 * 2 * M * N * K))
os.makedirs("gpurun_out", exist_ok=True)
json.dump(res, open("gpurun_out/i8_energy.json", "w"), indent=1)
