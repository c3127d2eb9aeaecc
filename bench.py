#!/usr/bin/env python
"""Benchmark of the FPM-partitioned column-based parallel matrix multiplication.

    python bench.py --gpus N --steps K --warmup W [--impl ours|reference] [--config c5|c3|c4]

One process per GPU (torchrun for N > 1: RANK / WORLD_SIZE / LOCAL_RANK); the
pivot exchange inside libfpmpmm -- one-sided pulls from the peers' memory over
NVLink fused into the staging kernels (IPC, default) or NCCL send/recv +
column broadcasts (--transport nccl); torch.distributed (gloo) only for the
control plane (IPC handles, unique id, barriers, max-over-ranks of device times).

Workload (BASELINE.json config 5, default): N = 49152, b = 1024,
FP32, square U[-1,1) matrices from the shared counter-based generator, p = N
GPUs, strong scaling.  --config c3: N = 16384, b = 512 homogeneous; --config c4:
N = 32768, b = 512, rank i capped to {144, 128, 112, 96, 80, 64, 48, 32}[i] SMs
in a green-context partition (one GPU: eight partitions of it), plus the CPM and
homogeneous partitions.  A step = fpm_partition + colpart_arrange + pmm_compute
(the N/b iterations of pivot exchange, staging and rank-b update) on inputs
resident in HBM; `value` = 2 N^3 K / sum of per-step device times (max over
ranks).  `e2e` = the same through the public API on pinned host buffers (H2D
and D2H inside the timed region).  `--impl reference` times the CPU oracle
(plain triple loop) on a bounded sample of the same workload (rank 0 only).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

# the arithmetic the FP32 path computes in (inputs, outputs and accumulation FP32)
DTYPE = {"f16x3": "f32 (F16X3: 3 fp16 tcgen05 products per FP32 MAC, FP32 accumulate)",
         "tf32x3": "f32 (TF32X3: 3 tf32 tcgen05 products per FP32 MAC, FP32 accumulate)",
         "f16i8": "f32-emulated-f16i8 (fp16 + int8 products, row-max fixed point: NOT FP32-class)"}
METRIC = "partitioned GEMM GFLOPS & % tensor peak at 1/2/4/8 B200; FPM load imbalance %"
UNIT = "GFLOP/s"
ORACLE_ROWS, ORACLE_COLS = 2048, 1024   # bounded sample for the CPU oracle (~206 GFLOP at c5, ~5 s on 16 cores)


def log(*a):
    print(*a, file=sys.stderr, flush=True)


# ----------------------------------------------------------------- clocks
class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""
    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu: int):
        self.gpu = gpu
        self.rows = []
        self.proc = None

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.gpu), f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits",
                 "-lms", "200"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.thread = threading.Thread(target=self._read, daemon=True)
            self.thread.start()
        except Exception as e:  # pragma: no cover
            log("clock sampler unavailable:", e)
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            parts = [p.strip() for p in line.split(",")]
            if len(parts) == 7:
                self.rows.append(parts)

    def stop(self) -> dict:
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        sms, mx, reasons, power = [], None, set(), []
        for r in self.rows:
            try:
                sms.append(float(r[0]))
                mx = float(r[1])
                power.append(float(r[2]))
            except ValueError:
                continue
            for nm, v in zip(names, r[3:]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        loaded = [s for s, p in zip(sms, power) if p > 200.0] or sms
        watts = [p for p in power if p > 200.0]
        return {"sm_mhz": statistics.median(loaded) if loaded else None, "sm_max_mhz": mx,
                "reasons": sorted(reasons), "samples": len(sms),
                "power_w_median": statistics.median(watts) if watts else None}


# ----------------------------------------------------------------- peaks
def measured_peaks() -> dict:
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(path):
        with open(path) as f:
            d = json.load(f)
        return {"bf16_burst": d.get("bf16_tflops", 1590.0), "bf16_sustained": d.get("bf16_tflops_sustained", 1400.0),
                "hbm_gbs": d.get("hbm_gbs", 6650.0), "source": "measured"}
    return {"bf16_burst": 1590.0, "bf16_sustained": 1400.0, "hbm_gbs": 6650.0, "source": "fallback"}


def committed_traffic(N: int, b: int, args):
    """DRAM bytes per update launch from the committed ncu capture of the same
    configuration (profiles/ncu_traffic.json), else None."""
    path = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    variant = (6 if args.scheme == "f16i8" else 8) if args.kernel_variant < 0 else args.kernel_variant
    fuse = args.fuse if args.fuse > 0 else max(1, min(8, 2048 // b))
    G = args.raster_group if args.raster_group > 0 else (12 if args.scheme == "f16i8" else 16)
    fs = getattr(args, "fused_staging", 0) and args.scheme == "f16x3" and variant in (7, 8)
    key = (f"{N}_{b}_{args.scheme}_v{variant}" + ("" if fuse == 1 else f"_f{fuse}") + ("" if G == 16 else f"_r{G}")
           + ("_fs" if fs else ""))
    if args.gpus != 1 or not os.path.exists(path):
        return None
    entry = json.load(open(path)).get(key)
    return entry["dram_bytes_per_launch"] if entry else None


# ----------------------------------------------------------------- oracle
def oracle_sample(N: int, reps: int = 1, want_c: bool = False, seed_cfg: int = 4):
    """Time the CPU oracle (plain triple loop, FP64 accumulation) on the block
    C[0:R, 0:S] = A[0:R, :] B[:, 0:S] of the workload; returns (GFLOP/s, cores,
    desc, seconds[, C block])."""
    import synth
    from oracle import gemm as og
    R, S = min(ORACLE_ROWS, N), min(ORACLE_COLS, N)
    sa, sb = synth.seeds_for_config(seed_cfg)
    A = synth.rect(sa, N, 0, 0, R, N)
    B = synth.rect(sb, N, 0, 0, N, S)
    og.gemm(A[:2, :64], B[:64, :8])  # build / load outside the timing
    ts = []
    for _ in range(reps):
        t0 = time.perf_counter()
        Cs = og.gemm(A, B)
        ts.append(time.perf_counter() - t0)
    t = min(ts)
    flops = 2.0 * R * S * N
    desc = (f"C[0:{R},0:{S}] = A[0:{R},:] B[:,0:{S}] of the N={N} workload (K={N}); "
            f"{flops / 1e9:.2f} GFLOP per step, oracle triple loop (gcc -O2, OpenMP, FP64 accumulation)")
    if want_c:
        return flops / t / 1e9, og.num_threads(), desc, t, Cs
    return flops / t / 1e9, og.num_threads(), desc, t


def e2e_parity(N: int, hC, oracle_block, seeds) -> dict:
    """Parity of the timed e2e output (pmm_run, default options) against the
    oracle on sampled blocks (exact oracle on a sample of C):
    the top-left block the CPU baseline computes anyway, plus the bottom-right
    corner and an interior block computed here.  Tolerance 1e-5 rel-Fro (FP32)."""
    import numpy as np

    import synth
    from oracle import gemm as og
    sa, sb = seeds
    C = hC.numpy() if hasattr(hC, "numpy") else np.asarray(hC)
    R, S = oracle_block.shape
    blocks = [("top-left", 0, 0, R, S, oracle_block)]
    for name, r0, c0, h, w in (("bottom-right", N - 256, N - 256, 256, 256),
                               ("interior", N // 2 - 100, N // 3 - 60, 200, 120)):
        A = synth.rect(sa, N, r0, 0, h, N)
        B = synth.rect(sb, N, 0, c0, N, w)
        blocks.append((name, r0, c0, h, w, og.gemm(A, B)))
    out = []
    for name, r0, c0, h, w, ref in blocks:
        out.append({"block": name, "rows": [r0, r0 + h], "cols": [c0, c0 + w],
                    "rel_fro": float(og.rel_fro(C[r0:r0 + h, c0:c0 + w], ref))})
    worst = max(b["rel_fro"] for b in out)
    return {"what": "e2e output C (host, pmm_run) vs the CPU oracle on sampled blocks", "tol": 1e-5,
            "blocks": out, "max_rel_fro": worst, "ok": bool(worst <= 1e-5)}


def e2e_parity_rank(N: int, hC, window, seeds, rank: int) -> list:
    """N > 1: sampled 64 x 64 blocks (corners and centre) of this rank's
    rectangle of the e2e output against the oracle; the operands' full rows and
    columns come from the same counter-based generator the device filled them
    with (synth)."""
    import numpy as np

    import synth
    from oracle import gemm as og
    R0, C0, H, W = window
    sa, sb = seeds
    C = hC.numpy() if hasattr(hC, "numpy") else np.asarray(hC)
    h, w = min(64, H), min(64, W)
    out = []
    for name, r, c in (("top-left", 0, 0), ("bottom-right", H - h, W - w), ("centre", (H - h) // 2, (W - w) // 2)):
        A = synth.rect(sa, N, R0 + r, 0, h, N)
        B = synth.rect(sb, N, 0, C0 + c, N, w)
        ref = og.gemm(A, B)
        out.append({"rank": rank, "block": name, "rows": [R0 + r, R0 + r + h], "cols": [C0 + c, C0 + c + w],
                    "rel_fro": float(og.rel_fro(C[r:r + h, c:c + w], ref))})
    return out


# ----------------------------------------------------------------- main arms
def run_reference(args, rank: int):
    if rank != 0:
        return
    # rank 0 alone runs: give the oracle every host core (torchrun exports OMP_NUM_THREADS=1)
    from oracle import gemm as og
    og.set_num_threads(len(os.sched_getaffinity(0)))
    cfg = CONFIGS[args.config]
    N, b = args.N or cfg["N"], args.b or cfg["b"]
    vals, times = [], []
    for i in range(args.warmup + args.steps):
        g, cores, desc, t = oracle_sample(N, seed_cfg=cfg["seed_cfg"])
        if i >= args.warmup:
            vals.append(g)
            times.append(t)
    value = statistics.median(vals)
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * statistics.median(times),
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64",
        "data": "synthetic",
        "config": {"workload": f"{args.config}: N={N}, b={b}, FP32 inputs (oracle accumulates in FP64)",
                   "N": N, "b": b, "sample": desc},
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": cores, "kind": "oracle", "sample": desc},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


# BASELINE.json configs bench.py can run; seeds = synth.seeds_for_config(index)
CONFIGS = {
    "c3": {"N": 16384, "b": 512, "caps": None, "seed_cfg": 2,
           "desc": "c3: N=16384, b=512, FP32, p={p} homogeneous B200, FPM partition + column arrangement"},
    "c4": {"N": 32768, "b": 512, "caps": [144, 128, 112, 96, 80, 64, 48, 32], "seed_cfg": 3,
           "desc": "c4: N=32768, b=512, FP32, p={p} B200 with SM caps {caps} (green-context partitions), "
                   "FPM vs constant-model vs homogeneous partition"},
    "c5": {"N": 49152, "b": 1024, "caps": None, "seed_cfg": 4,
           "desc": "c5: N=49152, b=1024, FP32, p={p} homogeneous B200, FPM partition + column arrangement"},
}
# c4 on ONE GPU: the eight caps scaled to fit its 148 SMs (studies/hetero.py)
C4_ONE_GPU_CAPS = [30, 26, 24, 20, 16, 14, 10, 6]


def imbalance(ts) -> float:
    """max / mean - 1 over devices with work (reading Q18)."""
    live = [t for t in ts if t > 0]
    return max(live) / (sum(live) / len(live)) - 1.0 if live else 0.0


def build_line(*, world, steps, warmup, step_times, workload, cfg, scheme, roofline, per_dev, e2e, cpu, parity,
               launches, clocks, extra_config=None) -> dict:
    """The bench JSON line from per-step device times (max over ranks) and
    per-device records (pure: tested without a GPU, tests/test_bench_contract.py).
    per_dev: one dict per device of the arrangement with keys rank, device, rect,
    compute_s, update_s, predicted_s."""
    total_t = sum(step_times)
    N = cfg["N"]
    value = 2.0 * N ** 3 * steps / total_t / 1e9
    live = [d for d in per_dev if d["rect"][3] * d["rect"][4] > 0]
    meas = [d.get("span_s", 0.0) for d in live]          # when each device finished (P:9)
    comp = [d["compute_s"] for d in live]                # sum of its staging + update event times
    pred = [d["predicted_s"] for d in live]
    peak = roofline["peak"]
    config = {
        "workload": workload, "N": N, "b": cfg["b"], "p": len(per_dev),
        "partition": [d["area"] for d in per_dev], "rects": [d["rect"] for d in per_dev],
        "f32_scheme": scheme,
        "l2": (f"inputs larger than L2 (A, B, C {N * N * 4 / 1e9:.2f} GB each)" if N * N * 4 > 126e6
               else "inputs fit in L2 (no flush between steps)"),
        "pct_tensor_peak": 100.0 * value / 1e3 / (peak * world) if peak else None,
        # load imbalance (reading Q18): max / mean - 1 of the devices' finish times -- the
        # k-loop span of each device, start to its last update's end (P:9: "all processors
        # complete their work within the same time"); also over the sums of each device's
        # staging + update event times (round 1's measure, which counts staging that runs
        # under the device's own updates a second time) and as the FPMs predict it
        "imbalance_pct_measured": 100.0 * imbalance(meas),
        "imbalance_pct_compute_sum": 100.0 * imbalance(comp),
        "imbalance_pct_predicted": 100.0 * imbalance(pred),
        "per_device": per_dev,
    }
    config.update(extra_config or {})
    return {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": steps, "warmup": warmup,
        "ms_per_step": 1e3 * total_t / steps, "higher_is_better": True, "scaling": "strong",
        "vs_baseline": None, "dtype": DTYPE[scheme], "data": "synthetic", "config": config,
        "roofline": roofline, "cpu_baseline": cpu, "parity": parity, "e2e": e2e, "gpu_launches": launches,
        "clocks": clocks,
    }


def run_ours(args, rank: int, world: int, local_rank: int, dist, emit: bool = True) -> dict | None:
    """One bench run of args.config; rank 0 returns (and, with `emit`, prints) the
    JSON line, the other ranks return None."""
    import torch

    import paper_conf_cluster_zhongrl12_b200 as pkg
    import synth

    torch.cuda.set_device(local_rank)
    cfg = dict(CONFIGS[args.config])
    if args.N:
        cfg["N"] = args.N
    if args.b:
        cfg["b"] = args.b
    N, b = cfg["N"], cfg["b"]
    n = N // b
    T = n * n
    # devices of the arrangement: one per rank; c4 on one GPU emulates eight in
    # disjoint green-context SM partitions of it
    if world == 1 and cfg["caps"]:
        caps = list(C4_ONE_GPU_CAPS)
    elif cfg["caps"]:
        caps = [cfg["caps"][r % len(cfg["caps"])] for r in range(world)]
    else:
        caps = None
    p = world if world > 1 else (len(caps) if caps else 1)
    mine = [rank] if world > 1 else list(range(p))   # devices this process drives

    def make_ctx(transport: str):
        if transport.startswith("nccl") and not (world == 1 and caps):
            obj = [pkg.Context.nccl_unique_id() if rank == 0 else None]
            if world > 1:
                dist.broadcast_object_list(obj, src=0)
            c = pkg.Context.nccl(rank, world, local_rank, obj[0], sm_cap=caps[rank] if caps else 0)
        elif world > 1:
            c = pkg.Context.ipc(rank, world, local_rank, sm_cap=caps[rank] if caps else 0)
        else:
            c = pkg.Context.local([local_rank] * p, sm_caps=caps)
        c.set_option("f32_scheme", {"f16i8": pkg.SCHEME_F16I8, "f16x3": pkg.SCHEME_F16X3,
                                    "tf32x3": pkg.SCHEME_TF32X3}[args.scheme])
        c.set_option("cta_group", args.cta_group)
        c.set_option("raster_group", args.raster_group)
        c.set_option("l2_hint_b", args.l2_hint_b)
        c.set_option("kernel_variant", args.kernel_variant)
        c.set_option("chunk_k", args.chunk_k)
        c.set_option("raster_snake", args.raster_snake)
        c.set_option("share_b", args.share_b)
        c.set_option("fused_staging", args.fused_staging)
        c.set_option("fuse", args.fuse)
        c.set_option("tail_stream", args.tail_stream)
        c.set_option("e2e_tail", args.e2e_tail)
        if args.tail_band:
            c.set_option("tail_band", args.tail_band)
        if caps:
            c.set_option("sm_partition", 1)   # every kernel of a device inside its SM partition
        return c

    transport = args.transport if (world > 1 or args.transport == "nccl") else "none (one process)"
    ctx = make_ctx(transport)

    # ---- FPMs (offline): each device's speed function sampled once,
    # gathered so every rank partitions identically
    sizes = [m * m for m in ((1, 2, 4, 8, 12, 16, 20, 24, 28, 32) if caps else (1, 2, 4, 8, 12, 16))]
    t0 = time.perf_counter()
    fpm_source = "sampled"
    if args.no_sample:  # profiling runs: identical constant models, predictable launch order
        mine_models = [(sizes, [1.0] * len(sizes)) for _ in mine]
        fpm_source = "constant (profiling)"
    else:
        from paper_conf_cluster_zhongrl12_b200 import fpm_store
        meta = [{"device": torch.cuda.get_device_name(local_rank), "kind": "gpu",
                 "sm_cap": caps[dev] if caps else 0, "cores": None, "dtype": "f32", "b": b,
                 "scheme": args.scheme, "fuse": args.fuse} for dev in mine]
        cache = (f"{args.fpm_cache}.rank{rank}" if world > 1 else args.fpm_cache) if args.fpm_cache else None
        mine_models = None
        if cache and os.path.exists(cache):   # FPMs built in advance, reused if measured alike
            try:
                recs = fpm_store.load(cache, expect=meta)
                if all(r["x"] == sizes for r in recs):
                    mine_models = fpm_store.models(recs)
                    fpm_source = f"loaded from {cache}"
            except ValueError as ex:
                log(f"rank {rank}: FPM cache not used: {ex}")
        if mine_models is None:
            recs = []
            for dev, m in zip(mine, meta):
                sp, ci, reps = ctx.sample(dev, b, sizes, pkg.FPM_F32)
                recs.append(fpm_store.record(sizes, sp, ci, reps, **m))
            mine_models = fpm_store.models(recs)
            if cache:
                fpm_store.save(cache, recs)
    t_sample = time.perf_counter() - t0
    if world > 1:
        models = [None] * world
        dist.all_gather_object(models, mine_models[0])
    else:
        models = mine_models

    def barrier():
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()

    def max_over_ranks(x: float) -> float:
        if world == 1:
            return x
        t = torch.tensor([x], dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    seeds = synth.seeds_for_config(cfg["seed_cfg"])

    def install(rects):
        """Set up the arrangement on every rank (IPC: exchange the mappings), fill
        the synthetic inputs, and barrier so every rank's inputs are resident."""
        nonlocal ctx, transport
        ctx.setup(N, b, rects, pkg.FPM_F32)
        if transport == "ipc":
            ok = 1
            blobs = [None] * world
            dist.all_gather_object(blobs, ctx.ipc_export())
            try:
                ctx.ipc_import(blobs)
            except pkg.FpmError as ex:  # e.g. no peer access between these GPUs
                log(f"rank {rank}: IPC import failed ({ex}); falling back to NCCL")
                ok = 0
            flag = torch.tensor([ok], dtype=torch.int32)
            dist.all_reduce(flag, op=dist.ReduceOp.MIN)
            if int(flag.item()) == 0:
                dist.barrier()
                ctx.close()
                transport = "nccl (ipc unavailable)"
                ctx = make_ctx("nccl")
                ctx.setup(N, b, rects, pkg.FPM_F32)
        ctx.fill_synthetic(seeds[0], seeds[1], pkg.FPM_DIST_PM1)
        barrier()

    # devices sharing one GPU (c4 on one GPU): the FPM-chosen integer arrangement (Q25)
    arrange_fpm = world == 1 and bool(caps)

    def plan(part_models):
        d = pkg.fpm_partition(T, part_models)
        return d, (pkg.colpart_arrange_fpm(n, d, part_models) if arrange_fpm else pkg.colpart_arrange(n, d))

    def per_device(comp, upd, span, rects, part_models):
        """Per-device records (Fig. 6 metric): this process's devices (comp /
        upd indexed by device, as pmm_stats), gathered over the ranks."""
        recs = []
        for dev in mine:
            r = rects[dev]
            a = r[3] * r[4]
            recs.append({"rank": rank, "device": dev, "rect": list(r), "area": a,
                         "sm_cap": caps[dev] if caps else None,
                         "compute_s": comp[dev], "update_s": upd[dev], "span_s": span[dev],
                         "predicted_s": (2.0 * a * b * b * N / pkg.fpm_model_speed(part_models[dev], a)
                                         if a > 0 else 0.0)})
        if world > 1:
            allr = [None] * world
            dist.all_gather_object(allr, recs)
            recs = [x for rr in allr for x in rr]
        return recs

    refine_hist = None
    if arrange_fpm and not args.no_sample:
        # devices that share one GPU share its power budget: models measured alone take the
        # level the devices reach when all run (synchronised level correction, Q26)
        from studies import refine as rf
        models, refine_hist, _, _ = rf.refine(ctx, n, b, models, 3, arrange="fpm", ci_permille=10)
        fpm_source += " + synchronised level correction (Q26)"
    d, rects = plan(models)
    install(rects)

    # ---- device-resident steps: fpm_partition + colpart_arrange + the k-loop
    for _ in range(args.warmup):
        d, rects = plan(models)
        ctx.compute(zero_c=True)
    barrier()
    clocks = ClockSampler(local_rank)
    clocks.start()
    step_times, recs_steps, own_times, launches, comm = [], [], [], 0, 0
    wall0 = time.perf_counter()
    for _ in range(args.steps):
        d, rects = plan(models)
        st = ctx.compute(zero_c=True)
        own_times.append(st.t_compute_s)
        step_times.append(max_over_ranks(st.t_compute_s))
        recs_steps.append([(st.per_dev_compute_s[i], st.per_dev_update_s[i], st.per_dev_span_s[i]) for i in range(16)])
        launches += st.kernel_launches
        comm += st.comm_bytes
    barrier()
    wall = time.perf_counter() - wall0
    clk = clocks.stop()
    # the median step's per-device record
    med = sorted(range(args.steps), key=lambda i: own_times[i])[args.steps // 2]
    per_dev = per_device([x[0] for x in recs_steps[med]], [x[1] for x in recs_steps[med]],
                         [x[2] for x in recs_steps[med]], rects, models)
    mine_recs = [x for x in per_dev if x["rank"] == rank]
    upd_med = max(x["update_s"] for x in mine_recs)
    comp_med = max(x["compute_s"] for x in mine_recs)
    stage = comp_med - upd_med
    exposed = max(0.0, own_times[med] - upd_med)   # k-loop time with no update running
    # with in-kernel staging the later groups' staging runs inside the updates
    # (their staging intervals are empty), so a ratio over staging intervals
    # would mean nothing: the exposed time per step is reported instead
    fused = bool(args.fused_staging) and args.scheme == "f16x3"
    overlap = (1.0 - exposed / stage) if (stage > 0 and not fused) else None
    overlaps, exposeds = [overlap], [exposed]
    if world > 1:
        overlaps, exposeds = [None] * world, [None] * world
        dist.all_gather_object(overlaps, overlap)
        dist.all_gather_object(exposeds, exposed)

    # ---- the exchange against NVLink ("NVLink bandwidth for the
    # broadcasts"): pivot bytes this rank pulled per step over its staging time (the
    # pulls are fused into the staging kernels, so this is a lower bound of the link rate)
    ex = None
    if world > 1:
        mine_bytes = comm / max(1, args.steps)
        rate = mine_bytes / stage / 1e9 if stage > 0 and mine_bytes > 0 else None
        rates = [None] * world
        dist.all_gather_object(rates, rate)
        peer = "same GPU (--same-gpu): HBM, not NVLink" if args.same_gpu else "NVLink 5, 900 GB/s per direction"
        valid = [r for r in rates if r]
        ex = {"bound": "nvlink", "unit": "GB/s", "peak": 900.0, "peak_basis": "B200 NVLink 5 nominal per direction "
              "(/opt/skills/guides/B200_PROFILING.md)", "achieved_per_rank": rates,
              "achieved": max(valid) if valid else None, "frac": (max(valid) / 900.0) if valid else None,
              "path": peer, "what": "pivot bytes pulled per step / the rank's staging time (pull fused into the split)"}

    # ---- roofline of the dominant kernel (rank-(f b) update): algorithmic flops
    # 2 H W b n of the busiest device over its summed update time (CUDA events on its stream)
    peaks = measured_peaks()
    busiest = max(mine_recs, key=lambda x: x["update_s"])
    rb = busiest["rect"]
    H, W = rb[3] * b, rb[4] * b
    achieved = 2.0 * H * W * b * n / busiest["update_s"] / 1e12 if busiest["update_s"] > 0 else 0.0
    dense_peak = peaks["bf16_sustained"] if args.scheme != "tf32x3" else peaks["bf16_sustained"] / 2.0
    mma_per_mac = 2.0 if args.scheme == "f16i8" else 3.0
    peak = dense_peak / mma_per_mac
    if caps:  # one device's share of the GPU
        peak *= caps[busiest["device"]] / torch.cuda.get_device_properties(local_rank).multi_processor_count
    basis = {"f16i8": "fp16 dense tensor peak ({src} {p:.1f} TFLOP/s sustained) / 2 (one fp16 product + one "
                      "int8 product of 2K at 2x the fp16 rate per FP32 MAC)",
             "f16x3": "fp16 dense tensor peak ({src} {p:.1f} TFLOP/s sustained) / 3 MMAs per FP32 MAC",
             "tf32x3": "tf32 dense tensor peak ({src} {p:.1f} TFLOP/s sustained) / 3 MMAs per FP32 MAC"}[args.scheme]
    if caps:
        basis += " x the device's SM share"
    roofline = {"bound": "tensor", "achieved": achieved, "peak": peak, "unit": "TFLOP/s",
                "frac": achieved / peak if peak else None,
                "traffic": (args.traffic if args.traffic is not None else
                            (committed_traffic(N, b, args) if not caps else None)),
                "peak_basis": basis.format(src=peaks["source"], p=dense_peak),
                "tensor_pipe_frac": achieved * mma_per_mac / dense_peak if dense_peak else None,
                "kernel": ("rank-(f b) update (update_acc_kernel: F16X3 chunked accumulation"
                           + (", staging the next group in its staging warp)" if args.fused_staging else ")"))
                if args.scheme == "f16x3" else "rank-(f b) update",
                "device": busiest["device"]}

    # ---- c4: the same multiply under the constant-model and homogeneous partitions
    partitions = None
    if caps and not args.no_partitions:
        x_cal = max(1, (8192 // b) ** 2 // p)   # CPM constants at the even share of N_cal = 8192 (Q9)
        alt = {"cpm_ncal": [([1], [pkg.fpm_model_speed(m, x_cal)]) for m in models],
               "homogeneous": [([1], [1.0])] * p}
        partitions = {"fpm": {"t_s": statistics.median(step_times), "d": list(d),
                              "imbalance_pct_measured": 100.0 * imbalance([x["span_s"] for x in per_dev]),
                              "imbalance_pct_compute_sum": 100.0 * imbalance([x["compute_s"] for x in per_dev]),
                              "imbalance_pct_predicted": 100.0 * imbalance([x["predicted_s"] for x in per_dev])}}
        for name, pm in alt.items():
            dd, rr = plan(pm)
            install(rr)
            ctx.compute()
            best, t_best = None, None
            for _ in range(2):
                s2 = ctx.compute()
                t2 = max_over_ranks(s2.t_compute_s)
                if t_best is None or t2 < t_best:
                    best, t_best = s2, t2
            recs = per_device(list(best.per_dev_compute_s), list(best.per_dev_update_s), list(best.per_dev_span_s),
                              rr, models)
            partitions[name] = {"t_s": t_best, "d": list(dd),
                                "imbalance_pct_measured": 100.0 * imbalance([x["span_s"] for x in recs]),
                                "imbalance_pct_compute_sum": 100.0 * imbalance([x["compute_s"] for x in recs]),
                                "imbalance_pct_predicted": 100.0 * imbalance([x["predicted_s"] for x in recs])}
        for v in partitions.values():
            v["gflops"] = 2.0 * N ** 3 / v["t_s"] / 1e9
        partitions["fpm_vs_cpm_time_delta_pct"] = 100.0 * (partitions["fpm"]["t_s"] / partitions["cpm_ncal"]["t_s"] - 1)
        partitions["fpm_vs_homogeneous_time_delta_pct"] = 100.0 * (
            partitions["fpm"]["t_s"] / partitions["homogeneous"]["t_s"] - 1)
        install(rects)   # back to the FPM arrangement for e2e

    # ---- end to end through pmm_run with pinned host buffers
    e2e, hC, window = None, None, None
    if args.e2e_steps > 0:
        try:
            e2e, hC, window = run_e2e(args, ctx, rects, rank, world, max_over_ranks, barrier, transport == "ipc",
                                      N, b, seeds)
        except Exception as ex:  # report, do not hide
            log("e2e failed:", repr(ex))
            e2e = {"value": None, "unit": UNIT, "error": repr(ex)[:200]}

    # the oracle leg, after every timed region: at N = 1 rank 0 times the oracle
    # (cpu_baseline; N > 1 lines carry null) and checks the e2e output with it;
    # at N > 1 every rank checks sampled blocks of its own rectangle
    cpu, parity = None, None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        g, cores, desc, _, c_block = oracle_sample(N, want_c=True, seed_cfg=cfg["seed_cfg"])
        cpu = {"value": g, "unit": UNIT, "cores": cores, "kind": "oracle", "sample": desc}
        if hC is not None:
            parity = e2e_parity(N, hC, c_block, seeds)
            if not parity["ok"]:
                log("PARITY FAILURE of the e2e output:", json.dumps(parity))
    elif world > 1 and not args.no_cpu_baseline and args.e2e_steps > 0:
        # every rank checks sampled blocks of its own rectangle of the e2e output
        # against the oracle; rank 0 reports them all (every rank joins the gather)
        ok_here = hC is not None and e2e is not None and e2e.get("value") is not None
        mine = e2e_parity_rank(N, hC, window, seeds, rank) if ok_here else []
        allb = [None] * world
        dist.all_gather_object(allb, mine)
        blocks = [blk for r in allb for blk in r]
        worst = max((blk["rel_fro"] for blk in blocks), default=0.0)
        parity = {"what": "e2e output C (each rank's host window, pmm_run) vs the CPU oracle on sampled blocks "
                          "of every rank's rectangle", "tol": 1e-5, "blocks": blocks, "max_rel_fro": worst,
                  "ok": bool(blocks) and worst <= 1e-5}
        if rank == 0 and not parity["ok"]:
            log("PARITY FAILURE of the e2e output:", json.dumps(parity))

    line = None
    if rank == 0:
        line = build_line(
            world=world, steps=args.steps, warmup=args.warmup, step_times=step_times,
            workload=cfg["desc"].format(p=p, caps=caps), cfg=cfg, scheme=args.scheme, roofline=roofline,
            per_dev=per_dev, e2e=e2e, cpu=cpu, parity=parity, launches=launches, clocks=clk,
            extra_config={
                "config": args.config, "cta_group": args.cta_group, "raster_group": args.raster_group,
                "kernel_variant": args.kernel_variant, "chunk_k": args.chunk_k, "raster_snake": args.raster_snake,
                "fused_staging": args.fused_staging,
                "fuse": args.fuse,
                "update_launches_per_step": st.updates, "transport": transport,
                "fpm_sample_s": t_sample, "fpm_sizes": sizes, "fpm_models": fpm_source,
                "fpm_refine_rounds": len(refine_hist) if refine_hist else None,
                "comm_bytes_per_step": comm // max(1, args.steps),
                # share of the exchange + staging time hidden under the updates, per rank (CUDA
                # events of each rank's streams; SURVEY §8(d) c5 "broadcast/update overlap")
                "exchange_staging_overlap": overlaps[0] if world == 1 else overlaps,
                # per step: k-loop time during which no update kernel ran (the first group's
                # staging, launch gaps, and any staging between updates), per rank
                "exposed_between_updates_ms": (1e3 * exposeds[0]) if world == 1 else [1e3 * x for x in exposeds],
                "exchange_roofline": ex,
                "wall_s_timed_region": wall,
                "partitions": partitions,
            })
    barrier()  # no rank frees buffers a peer may still read (IPC)
    ctx.close()
    if rank == 0:
        if world == 1 and not caps and not args.no_hetero:
            try:
                line["hetero"] = run_hetero(peak, args.share_b, args.hetero_fused_staging)
            except Exception as ex:  # report, do not hide
                log("hetero failed:", repr(ex))
                line["hetero"] = {"error": repr(ex)[:200]}
        if world == 1:
            line["fig7"] = fig7_summary()
        if parity is not None and not parity["ok"]:
            print(json.dumps(line), flush=True)
            sys.exit(3)
        if emit:
            print(json.dumps(line), flush=True)
    return line


def run_hetero_multi(args, rank: int, world: int, local_rank: int, dist) -> dict | None:
    """N > 1: the heterogeneity measurement on the job's own GPUs -- config 4
    (N = 32768, b = 512, rank i capped to {144, 128, ..., 32}[i] SMs in a green
    partition of its GPU) run through the same code path as
    `--config c4`: FPMs sampled per rank, FPM / CPM(N_cal) / homogeneous
    partitions, max-over-ranks device times.  Rank 0 returns the summary."""
    import copy

    import torch
    h = copy.copy(args)
    h.config, h.N, h.b = "c4", args.hetero_N, 0
    h.steps, h.warmup, h.e2e_steps = 3, 3, 0
    h.no_cpu_baseline, h.no_partitions, h.fpm_cache = True, False, ""
    h.traffic = None
    t0 = time.perf_counter()
    hl = run_ours(h, rank, world, local_rank, dist, emit=False)
    if rank != 0:
        return None
    c = hl["config"]
    sms = torch.cuda.get_device_properties(local_rank).multi_processor_count
    caps = [x["sm_cap"] for x in c["per_device"]]
    mma_per_mac = 2.0 if args.scheme == "f16i8" else 3.0
    peaks = measured_peaks()
    dense = peaks["bf16_sustained"] if args.scheme != "tf32x3" else peaks["bf16_sustained"] / 2.0
    capped_peak = dense / mma_per_mac * sum(caps) / sms
    out = {"workload": c["workload"], "N": c["N"], "b": c["b"], "sm_caps": caps,
           "source": "bench.py --config c4 path run inside this job across its ranks (one GPU each, "
                     "green-context partitions)",
           "method": "fpm: each rank's FPM sampled on its own capped GPU (P:18), gathered, fpm_partition + "
                     "colpart_arrange (P:9, P:15)",
           "capped_aggregate_peak_tflops": capped_peak, "value_gflops": hl["value"],
           "roofline_frac_busiest": hl["roofline"]["frac"], "transport": c["transport"]}
    for name, r in (c["partitions"] or {}).items():
        if not isinstance(r, dict):
            continue
        out[name] = dict(r, pct_of_capped_peak=100.0 * r["gflops"] / 1e3 / capped_peak)
    for k in ("fpm_vs_cpm_time_delta_pct", "fpm_vs_homogeneous_time_delta_pct"):
        out[k] = (c["partitions"] or {}).get(k)
    out["wall_s"] = time.perf_counter() - t0
    return out


def fig7_summary() -> dict | None:
    """The memory-cliff study (Table III / Fig. 7 analogue, NEXT-2) summarised
    from its committed records (`studies/memcap.py`, several minutes of GPU
    time: not re-run inside the bench): per layout and n, the time of each
    partition and FPM's delta against CPM and the homogeneous split."""
    out = {"source": "committed study records, not re-measured in this run", "layouts": {}}
    for layout in ("sockets", "cores"):
        path = os.path.join(ROOT, "profiles", f"memcap_fig7_r02_{layout}.json")
        if not os.path.exists(path):
            continue
        d = json.load(open(path))
        rows, ok_cpm, ok_hom = [], True, True
        for r in d["table"]:
            f = r.get("fpm_refined", r["fpm"])
            row = {"n": r["n"], "fpm_s": f["t_total_s"], "fpm_static_s": r["fpm"]["t_total_s"],
                   "cpm_s": r["cpm"]["t_total_s"], "homogeneous_s": r["homogeneous"]["t_total_s"]}
            row["fpm_vs_cpm_pct"] = 100.0 * (row["fpm_s"] / row["cpm_s"] - 1)
            row["fpm_vs_homogeneous_pct"] = 100.0 * (row["fpm_s"] / row["homogeneous_s"] - 1)
            ok_cpm = ok_cpm and row["fpm_vs_cpm_pct"] <= 1.0     # within 1 % counts as a tie
            ok_hom = ok_hom and row["fpm_vs_homogeneous_pct"] <= 1.0
            rows.append(row)
        out["layouts"][layout] = {
            "file": os.path.relpath(path, ROOT), "devices": d["config"]["names"],
            "sm_caps": d["config"]["sm_caps"], "c_cap_bytes": d["config"]["c_cap_bytes"],
            "fpm": "cliff-bracketed FPMs with synchronised level correction (DESIGN Q26)",
            "fpm_no_slower_than_cpm_every_n": ok_cpm, "fpm_no_slower_than_homogeneous_every_n": ok_hom,
            "tie_tolerance_pct": 1.0,
            "rows": rows}
    return out if out["layouts"] else None


def run_hetero(peak_tflops: float, share_b: int = 1, fused_staging: int = 1) -> dict:
    """The metric's 'FPM load imbalance %' under emulated heterogeneity (SURVEY
    §8(d) c4 analogue, studies/hetero.py): 8 devices on this GPU in disjoint
    green-context SM partitions, FPMs sampled per device, the multiply under
    FPM / CPM / homogeneous / in-situ corrected FPM partitions."""
    import torch

    from studies import hetero
    caps = [30, 26, 24, 20, 16, 14, 10, 6]   # config 4's {144 .. 32} scaled to fit 148 SMs
    t0 = time.perf_counter()
    res = hetero.c4_study(caps, N=32768, b=512, reps=3, insitu=1, graph=0, sm_partition=1, log=log, refine_rounds=3,
                          refine_arrange=("fpm",), refine_ci_permille=10,
                          options={"share_b": share_b, "fused_staging": fused_staging})
    sms = torch.cuda.get_device_properties(0).multi_processor_count
    capped_peak = peak_tflops * sum(caps) / sms
    out = {"workload": ("c4 analogue: N=32768, b=512, FP32, p=8 devices emulated on one B200 by green-context "
                        f"SM partitions {caps}; FPMs sampled per device alone (P:11), "
                        f"{len(res['config']['sizes'])} sizes"),
           "method": ("fpm: the FPM partition of models built by the paper's protocol -- size sweep of each "
                      "device alone (P:18, P:11), level from the synchronised run of all devices at their "
                      "operating points (P:10 (ii); DESIGN Q26) -- with FPM-chosen integers (Q25)"),
           "partitions": {"fpm": "FPM, synchronised level correction (Q26), FPM-chosen integer arrangement (Q25)",
                          "fpm_exclusive": "FPM of the exclusive size-sweep models alone, paper arrangement",
                          "fpm_exclusive_arr": "the same, FPM-chosen integer arrangement (Q25)",
                          "cpm_ncal": "constant models at the even share of N_cal = 8192 (Q9)",
                          "cpm_self": "constant models at this run's even share",
                          "homogeneous": "equal areas",
                          "fpm_insitu1": "exclusive models rescaled by one FPM run's own per-device times "
                                         "(side study, not the method)"},
           "capped_aggregate_peak_tflops": capped_peak, "fpm_sample_s": res["fpm_sample_s"]}
    rename = {"fpm_refined_arr": "fpm", "fpm": "fpm_exclusive", "fpm_arr": "fpm_exclusive_arr"}
    for name, r in res["partitions"].items():
        out[rename.get(name, name)] = {
            "t_s": r["t_total_s"], "gflops": r["gflops"], "d": r["d"],
            "refine_rounds": len(r.get("refine_history", [])) or None,
            "imbalance_pct_measured": 100.0 * r.get("imbalance_span", 0.0),
            "imbalance_pct_compute_sum": 100.0 * r["imbalance_measured"],
            "imbalance_pct_predicted": 100.0 * r["imbalance_predicted"],
            "pct_of_capped_peak": 100.0 * r["gflops"] / 1e3 / capped_peak}
    if "fpm" in out and "cpm_ncal" in out:
        out["fpm_vs_cpm_time_delta_pct"] = 100.0 * (out["fpm"]["t_s"] / out["cpm_ncal"]["t_s"] - 1)
        out["fpm_vs_homogeneous_time_delta_pct"] = 100.0 * (out["fpm"]["t_s"] / out["homogeneous"]["t_s"] - 1)
        out["fpm_exclusive_vs_cpm_time_delta_pct"] = 100.0 * res["fpm_vs_cpm_ncal_time_delta"]
    out["wall_s"] = time.perf_counter() - t0
    return out


def run_e2e(args, ctx, rects, rank, world, max_over_ranks, barrier, ipc, N, b, seeds):
    """e2e through the public API with pinned host buffers: pmm_run (host panels
    streamed in under the k-loop, C streamed out; under IPC every rank streams
    its own window and peers' pulls wait on its progress flag); median of
    args.e2e_steps calls after one warm-up call, max over ranks.  Returns the
    record and, in one process, the host C (all of it) for the parity check."""
    import torch

    import paper_conf_cluster_zhongrl12_b200 as pkg
    # host windows: this rank's rectangle (IPC / NCCL) or all of A, B, C (one process)
    if world > 1:
        r = rects[rank]
        H, W, R0, C0 = r[3] * b, r[4] * b, r[1] * b, r[2] * b
    else:
        H = W = N
        R0 = C0 = 0
    live = H * W > 0
    if live:   # generated on the device by the shared generator once, untimed
        hA = torch.empty((H, W), dtype=torch.float32, pin_memory=True)
        hB = torch.empty((H, W), dtype=torch.float32, pin_memory=True)
        hC = torch.empty((H, W), dtype=torch.float32, pin_memory=True)
        tmp = torch.empty((H, W), dtype=torch.float32, device="cuda")
        pkg.k_fill_synthetic(tmp, pkg.FPM_F32, W, seeds[0], N, R0, C0, H, W)
        hA.copy_(tmp)
        pkg.k_fill_synthetic(tmp, pkg.FPM_F32, W, seeds[1], N, R0, C0, H, W)
        hB.copy_(tmp)
        del tmp
        torch.cuda.empty_cache()
    barrier()
    ts, st = [], None
    streamed = True   # IPC: streamed pmm_run (peer progress flags); fallback: upload + barrier + compute_into

    def ipc_resident_call():
        if live:
            ctx.upload(hA, hB, W, R0, C0)
        barrier()
        return ctx.compute_into(hC, W, R0, C0) if live else ctx.compute()

    for i in range(args.e2e_steps + 1):
        barrier()
        t0 = time.perf_counter()
        if ipc and not live:
            st = ctx.compute()   # takes part in the exchange only
        elif ipc and not streamed:
            st = ipc_resident_call()
        elif live:
            # blocking call: H2D streamed under the updates, k-loop, D2H of C
            try:
                st = ctx.run(hA, hB, hC, N, b, rects, pkg.FPM_F32, ld=W, row_base=R0, col_base=C0)
            except pkg.FpmError as ex:
                if not ipc or i > 0:
                    raise
                log(f"rank {rank}: streamed IPC pmm_run failed ({ex}); using upload + barrier + compute_into")
                streamed = False
        if ipc and i == 0:   # every rank takes the same path from here on
            flag = torch.tensor([1 if streamed else 0], dtype=torch.int32)
            import torch.distributed as dist
            dist.all_reduce(flag, op=dist.ReduceOp.MIN)
            if int(flag.item()) == 0 and streamed:
                streamed = False
            if not streamed:
                barrier()
                st = ipc_resident_call()
        t_host = time.perf_counter() - t0
        t_all = max_over_ranks(t_host)
        if i > 0:  # first call is a warm-up
            ts.append(t_all)
    t = statistics.median(ts)
    rec = {"value": 2.0 * N ** 3 / t / 1e9, "unit": UNIT, "h2d_bytes_per_step": 2 * H * W * 4,
           "d2h_bytes_per_step": H * W * 4, "steps": len(ts), "ms_per_step": 1e3 * t,
           "device_kloop_s": st.t_compute_s if st else None, "download_s": st.t_download_s if st else None,
           "timing": (("host wall clock around the blocking pmm_run call (IPC: each rank's window streamed in, "
                       "peers' pulls ordered by its progress flag), max over ranks") if (ipc and streamed) else
                      "host wall clock: pmm_upload + barrier + pmm_compute_into (IPC), max over ranks" if ipc else
                      "host wall clock around the blocking pmm_run call, max over ranks")}
    if world > 1:
        rec["h2d_bytes_per_step_rank0"] = rec["h2d_bytes_per_step"]
        tot = torch.tensor([2 * H * W * 4, H * W * 4], dtype=torch.float64)
        import torch.distributed as dist
        dist.all_reduce(tot)
        rec["h2d_bytes_per_step"], rec["d2h_bytes_per_step"] = int(tot[0].item()), int(tot[1].item())
    return rec, (hC if live else None), (R0, C0, H, W)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--config", choices=sorted(CONFIGS), default="c5",
                    help="BASELINE config: c5 (default; N=49152, b=1024), c3 (N=16384, b=512), c4 (N=32768, "
                         "b=512, SM caps {144..32} per rank; one GPU: 8 green partitions)")
    ap.add_argument("--N", type=int, default=0, help="override the config's N")
    ap.add_argument("--b", type=int, default=0, help="override the config's b")
    ap.add_argument("--no-partitions", action="store_true", help="c4: skip the CPM / homogeneous runs")
    ap.add_argument("--scheme", choices=["f16i8", "f16x3", "tf32x3"], default="f16x3",
                    help="FP32 arithmetic: f16x3 (default, FP32-class), tf32x3, or f16i8 (opt-in, "
                         "fixed point relative to the row maximum: not FP32-class, DESIGN Q15b)")
    ap.add_argument("--transport", choices=["ipc", "nccl"], default="ipc",
                    help="N > 1: pull pivots from peers' memory (ipc) or exchange them with NCCL")
    ap.add_argument("--cta-group", type=int, default=2)
    ap.add_argument("--raster-group", type=int, default=0, help="0 = auto (12 for F16I8, 16 otherwise)")
    ap.add_argument("--l2-hint-b", type=int, default=0, help="0 evict_normal, 1 evict_first, 2 evict_last")
    ap.add_argument("--kernel-variant", type=int, default=-1, help="update kernel smem split (-1 auto, 0..3)")
    ap.add_argument("--raster-snake", type=int, default=0, help="serpentine raster over groups (0/1)")
    ap.add_argument("--fused-staging", type=int, default=1,
                    help="resident k-loop: the update kernel's staging warp stages the next group (0/1)")
    ap.add_argument("--share-b", type=int, default=1,
                    help="column members on the B owner's GPU read its staged B operand (0/1; local contexts)")
    ap.add_argument("--chunk-k", type=int, default=0, help="K per TMEM accumulation (variants 7/8; 0 auto = 512)")
    ap.add_argument("--fuse", type=int, default=0, help="pivots fused per update (0 auto = K of about 2048)")
    ap.add_argument("--e2e-steps", type=int, default=5)
    ap.add_argument("--tail-stream", type=int, default=1, help="pmm_run option tail_stream (e2e, one device)")
    ap.add_argument("--e2e-tail", type=int, default=-1, help="pmm_run option e2e_tail (-1 auto)")
    ap.add_argument("--tail-band", type=int, default=0, help="pmm_run option tail_band (rows, multiple of 256; 0 default)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--hetero-fused-staging", type=int, default=1,
                    help="hetero block: option fused_staging of its contexts (1 auto: off for devices sharing a GPU; 2 forced)")
    ap.add_argument("--no-hetero", action="store_true",
                    help="skip the heterogeneity measurement added to the line: N = 1 the c4 analogue on "
                         "eight green partitions of the GPU, N > 1 config 4 across the job's GPUs")
    ap.add_argument("--hetero-N", type=int, default=32768,
                    help="N > 1: matrix size of the config-4 heterogeneity run (b = 512)")
    ap.add_argument("--no-sample", action="store_true", help="skip fpm_sample (profiling runs)")
    ap.add_argument("--fpm-cache", default="",
                    help="FPM model file: reused when it was measured on the same device / cap / b / scheme, "
                         "else sampled and written (per rank under torchrun: PATH.rankR)")
    ap.add_argument("--same-gpu", action="store_true",
                    help="testing only: put every rank on cuda:0 (IPC transport works within one GPU)")
    ap.add_argument("--traffic", type=float, default=None,
                    help="dram bytes per update launch from an ncu --set full capture")
    args = ap.parse_args()
    if (args.N or CONFIGS[args.config]["N"]) % (args.b or CONFIGS[args.config]["b"]):
        ap.error("b must divide N")

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if args.same_gpu:
        local_rank = 0
    dist = None
    if world > 1:
        import torch.distributed as dist
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        if args.transport == "nccl":   # communicator set-up in the log (ranks per communicator)
            os.environ.setdefault("NCCL_DEBUG", "INFO")
            os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
        import datetime
        # a rank that fails between collectives surfaces as an error on the others
        # after this long instead of hanging the job
        dist.init_process_group("gloo", rank=rank, world_size=world, timeout=datetime.timedelta(minutes=10))
    if args.impl == "reference":
        run_reference(args, rank)
    else:
        line = run_ours(args, rank, world, local_rank, dist, emit=False)
        if world > 1 and args.config != "c4" and not args.no_hetero:
            # every rank takes part; a failure is reported in the line, not hidden
            try:
                het = run_hetero_multi(args, rank, world, local_rank, dist)
            except Exception as ex:  # pragma: no cover (GPU only)
                log(f"rank {rank}: multi-GPU hetero failed:", repr(ex))
                het = {"error": repr(ex)[:200]}
            if rank == 0:
                line["hetero"] = het
        if rank == 0:
            print(json.dumps(line), flush=True)
    if dist is not None:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
