"""Sustained (power-capped) tensor throughput of library GEMMs by operand type:
bf16 / fp16 (randn and U[-1,1) scaled like the F16X3 halves) and int8 (torch._int_mm),
8192^3 back to back for ~4 s each, with nvidia-smi clocks and power sampled."""
import json, subprocess, sys, time, threading, statistics
import torch

def sample(stop, rows):
    p = subprocess.Popen(["nvidia-smi", "--query-gpu=clocks.sm,power.draw", "--format=csv,noheader,nounits", "-lms", "100"],
                         stdout=subprocess.PIPE, text=True)
    while not stop.is_set():
        line = p.stdout.readline()
        if line:
            rows.append([float(x) for x in line.split(",")])
    p.kill()

def run(name, fn, flops, secs=4.0):
    for _ in range(3): fn()
    torch.cuda.synchronize()
    rows, stop = [], threading.Event()
    th = threading.Thread(target=sample, args=(stop, rows)); th.start()
    time.sleep(0.3)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    n = 0; t0 = time.time(); e0.record()
    while time.time() - t0 < secs:
        for _ in range(10): fn()
        n += 10
        torch.cuda.synchronize()
    e1.record(); torch.cuda.synchronize()
    stop.set(); th.join()
    ms = e0.elapsed_time(e1)
    load = [r for r in rows if r[1] > 300]
    out = {"name": name, "tops": flops * n / ms / 1e9, "sm_mhz": statistics.median([r[0] for r in load]) if load else None,
           "power_w": statistics.median([r[1] for r in load]) if load else None}
    print(json.dumps(out), flush=True)
    return out

L = 8192
dev = "cuda"
g = torch.Generator(device=dev).manual_seed(0)
res = []
a = torch.randn(L, L, device=dev, generator=g, dtype=torch.bfloat16); b = torch.randn(L, L, device=dev, generator=g, dtype=torch.bfloat16)
res.append(run("bf16 randn", lambda: a @ b, 2 * L**3))
a16 = (torch.rand(L, L, device=dev, generator=g) * 2 - 1).mul(2**14).half(); b16 = (torch.rand(L, L, device=dev, generator=g) * 2 - 1).mul(2**14).half()
res.append(run("fp16 U[-1,1)*2^14 (h0-like)", lambda: a16 @ b16, 2 * L**3))
ab = a16.bfloat16(); bb = b16.bfloat16()
res.append(run("bf16 U[-1,1)*2^14", lambda: ab @ bb, 2 * L**3))
ai = torch.randint(-127, 128, (L, L), device=dev, dtype=torch.int8, generator=g)
bi = torch.randint(-127, 128, (L, L), device=dev, dtype=torch.int8, generator=g)
try:
    res.append(run("int8 uniform", lambda: torch._int_mm(ai, bi.t().contiguous().t()), 2 * L**3))
except Exception as ex:
    print("int8 failed", ex)
a8 = a16.to(torch.float8_e4m3fn) if hasattr(torch, "float8_e4m3fn") else None
try:
    s = torch.tensor(1.0, device=dev)
    a8 = (torch.rand(L, L, device=dev, generator=g) * 2 - 1).to(torch.float8_e4m3fn)
    b8 = (torch.rand(L, L, device=dev, generator=g) * 2 - 1).to(torch.float8_e4m3fn).t().contiguous().t()
    res.append(run("fp8 e4m3 U[-1,1)", lambda: torch._scaled_mm(a8, b8, s, s, out_dtype=torch.bfloat16), 2 * L**3))
except Exception as ex:
    print("fp8 failed", ex)
res.append(run("fp16 U[-1,1)*2^14 again", lambda: a16 @ b16, 2 * L**3))
json.dump(res, open("gpurun_out/power_dtypes.json", "w"), indent=1)
