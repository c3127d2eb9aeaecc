"""The one-process-per-device runtime path for real, on ONE GPU: world-size 2
and 3 processes, each with a pmm_create_ipc context on cuda:0, control plane
over gloo (handle all-gather, barrier), pivots pulled from the peers' resident
buffers through CUDA IPC by the staging kernels.  Each rank downloads its
rectangle of C and checks it against the oracle (integer inputs: bit-exact;
U[-1,1): rel-Fro <= 1e-5)."""
import os
import socket

import numpy as np
import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
import torch.multiprocessing as mp  # noqa: E402


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, rects, N, b, dist_kind, q, opts=None):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import torch.distributed as dist

    import paper_conf_cluster_zhongrl12_b200 as pkg
    import synth
    from oracle import gemm as og
    try:
        torch.cuda.set_device(0)
        dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
        with pkg.Context.ipc(rank, world, 0) as ctx:
            for k, v in (opts or {}).items():
                ctx.set_option(k, v)
            ctx.setup(N, b, rects, pkg.FPM_F32)
            blobs = [None] * world
            dist.all_gather_object(blobs, ctx.ipc_export())
            ctx.ipc_import(blobs)
            ctx.fill_synthetic(1, 2, dist_kind)
            torch.cuda.synchronize()
            dist.barrier()                       # every rank's inputs are resident
            for _ in range(2):                   # repeated: the staging barrier re-arms
                st = ctx.compute()
            col, r0, c0, h, w = rects[rank]
            ok, err = True, 0.0
            if h * w:
                got = ctx.download_block(r0 * b, c0 * b, h * b, w * b)
                A_rows = synth.rect(1, N, r0 * b, 0, h * b, N, dist_kind)
                B_cols = synth.rect(2, N, 0, c0 * b, N, w * b, dist_kind)
                ref = og.gemm(A_rows, B_cols)
                if dist_kind == synth.DIST_INT:
                    ok = bool(np.array_equal(got.astype(np.float64), ref))
                else:
                    err = og.rel_fro(got, ref)
                    ok = err <= 1e-5
            dist.barrier()                       # peers stop reading before anyone frees
        q.put((rank, ok, err, st.comm_bytes))
        dist.destroy_process_group()
    except Exception as e:  # pragma: no cover
        q.put((rank, repr(e), -1.0, -1))


def _run(world, rects, N, b, dist_kind, opts=None):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, rects, N, b, dist_kind, q, opts))
             for r in range(world)]
    for p in procs:
        p.start()
    out = sorted(q.get(timeout=300) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
    return out


@pytest.fixture(autouse=True)
def _cuda():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


@pytest.mark.parametrize("dist_kind", [0, 1])
def test_ipc_two_ranks_two_columns(dist_kind):
    N, b = 1024, 128
    n = N // b
    rects = [(0, 0, 0, n, 3), (1, 0, 3, n, n - 3)]          # A slices move every iteration
    out = _run(2, rects, N, b, dist_kind)
    assert all(ok is True for (_, ok, _, _) in out), out
    assert all(by > 0 for (*_, by) in out)


def test_ipc_three_ranks_mixed_columns():
    import paper_conf_cluster_zhongrl12_b200 as pkg
    N, b = 1536, 128
    n = N // b
    rects = pkg.colpart_arrange(n, [70, 44, 30])             # one 2-device column, one 1-device column
    assert len({r[0] for r in rects}) == 2
    out = _run(3, rects, N, b, 1)
    assert all(ok is True for (_, ok, _, _) in out), out


@pytest.mark.parametrize("fused", [2, 0])
def test_ipc_fused_staging_pulls_peer_pieces(fused):
    """In-kernel staging on IPC contexts (the driver's N > 1 bench path): the
    staging warp of update g pulls group g + 1's A slices from the holders'
    and B from the owner's resident memory (several pieces per job); integer
    inputs bit-exact, with the option on and off."""
    import paper_conf_cluster_zhongrl12_b200 as pkg
    N, b = 4096, 256
    n = N // b
    rects = pkg.colpart_arrange(n, [120, 80, 56])            # a two-device column and a one-device column
    assert len({r[0] for r in rects}) == 2
    out = _run(3, rects, N, b, 1, {"fused_staging": fused})
    assert all(ok is True for (_, ok, _, _) in out), out


def _worker_run(rank, world, port, rects, N, b, reps, q, opts=None):
    """pmm_run on an IPC context: each rank streams its own host window in (k
    order, its progress flag written after each pivot's panels) while peers
    wait on that flag in their streams before pulling; C streamed out."""
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import torch.distributed as dist

    import paper_conf_cluster_zhongrl12_b200 as pkg
    import synth
    try:
        torch.cuda.set_device(0)
        dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
        col, r0, c0, h, w = rects[rank]
        H, W = h * b, w * b
        A = synth.rect(11, N, r0 * b, c0 * b, H, W, synth.DIST_INT)
        B = synth.rect(12, N, r0 * b, c0 * b, H, W, synth.DIST_INT)
        results = []
        with pkg.Context.ipc(rank, world, 0) as ctx:
            for k, v in (opts or {}).items():
                ctx.set_option(k, v)
            ctx.setup(N, b, rects, pkg.FPM_F32)
            blobs = [None] * world
            dist.all_gather_object(blobs, ctx.ipc_export())
            ctx.ipc_import(blobs)
            for it in range(reps):           # repeated runs: the flag epochs must not confuse the waits
                C = np.full((H, W), np.nan, np.float32)
                dist.barrier()
                ctx.run(A, B, C, N, b, rects, pkg.FPM_F32, ld=W, row_base=r0 * b, col_base=c0 * b)
                results.append(C)
            dist.barrier()
        from oracle import gemm as og
        ref = og.gemm(synth.rect(11, N, r0 * b, 0, H, N, synth.DIST_INT),
                      synth.rect(12, N, 0, c0 * b, N, W, synth.DIST_INT))
        ok = all(np.array_equal(C.astype(np.float64), ref) for C in results)
        q.put((rank, ok, 0.0, 0))
        dist.destroy_process_group()
    except Exception as e:  # pragma: no cover
        q.put((rank, repr(e), -1.0, -1))


@pytest.mark.parametrize("world,d", [(2, [40, 24]), (3, [70, 44, 30])])
def test_ipc_streamed_pmm_run(world, d):
    """pmm_run on IPC contexts (the bench's e2e at N > 1): host windows streamed
    in under the k-loop, integer inputs bit-exact, three repeated runs."""
    import paper_conf_cluster_zhongrl12_b200 as pkg
    N, b = 1536 if world == 3 else 1024, 128
    n = N // b
    rects = pkg.colpart_arrange(n, d if world == 2 else d)
    if world == 2:
        rects = pkg.colpart_arrange(n, [40, 24])
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker_run, args=(r, world, port, rects, N, b, 3, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = sorted(q.get(timeout=300) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
    assert all(ok is True for (_, ok, _, _) in out), out


@pytest.mark.parametrize("fused", [2, 0])
def test_ipc_streamed_fused_staging(fused):
    """pmm_run on IPC contexts at a size where the update's staging warp stages
    the next group: it waits in-kernel for the holders' upload-progress flags
    (own and peers') before pulling; integer inputs bit-exact over repeated runs."""
    import paper_conf_cluster_zhongrl12_b200 as pkg
    N, b = 4096, 256
    n = N // b
    rects = pkg.colpart_arrange(n, [120, 80, 56])
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker_run, args=(r, 3, port, rects, N, b, 2, q, {"fused_staging": fused}))
             for r in range(3)]
    for p in procs:
        p.start()
    out = sorted(q.get(timeout=300) for _ in range(3))
    for p in procs:
        p.join(timeout=60)
    assert all(ok is True for (_, ok, _, _) in out), out
