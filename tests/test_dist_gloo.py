"""N > 1 path on CPU: one process per rank over gloo (127.0.0.1), exchanging the
pivots exactly as the NCCL mode of the runtime does (runtime.cu issue_comm):
per iteration k one grouped point-to-point set for the A slices (plan from the
library's colpart_plan_step) and one broadcast of the B block-row inside each
column group from its owner.  Each rank then applies the rank-b update to its
C_i (numpy, float64, integer inputs -> exact) and compares with the oracle.
"""
import os
import socket

import numpy as np
import pytest

torch = pytest.importorskip("torch")
import torch.multiprocessing as mp  # noqa: E402


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, rects, N, b, q):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import torch.distributed as dist

    import paper_conf_cluster_zhongrl12_b200 as pkg
    import synth
    from oracle import gemm as og

    try:
        dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
        n = N // b
        col, r0, c0, h, w = rects[rank]
        live = h * w > 0
        A_loc = synth.rect(1, N, r0 * b, c0 * b, h * b, w * b, synth.DIST_INT, np.float64)
        B_loc = synth.rect(2, N, r0 * b, c0 * b, h * b, w * b, synth.DIST_INT, np.float64)
        C = np.zeros((h * b, w * b))
        # per-column groups (the ncclCommSplit of the runtime); created by all ranks in the same order
        members = {}
        for qi, rr in enumerate(rects):
            if rr[3] * rr[4] > 0:
                members.setdefault(rr[0], []).append(qi)
        groups = {c: dist.new_group(m) for c, m in sorted(members.items())}
        recv_bytes = 0
        for k in range(n):
            a_moves, b_moves = pkg.colpart_plan_step(n, rects, k)
            a_panel = np.full((h * b, b), np.nan)
            reqs, pending = [], []
            for (src, dst, lo, hi) in a_moves:       # grouped send/recv (horizontal)
                if src == dst == rank:
                    a_panel[(lo - r0) * b:(hi - r0) * b] = A_loc[(lo - r0) * b:(hi - r0) * b,
                                                                 (k - c0) * b:(k - c0 + 1) * b]
                elif src == rank:
                    piece = A_loc[(lo - r0) * b:(hi - r0) * b, (k - c0) * b:(k - c0 + 1) * b].copy()
                    reqs.append(dist.isend(torch.from_numpy(piece), dst))
                elif dst == rank:
                    buf = torch.empty(((hi - lo) * b, b), dtype=torch.float64)
                    reqs.append(dist.irecv(buf, src))
                    pending.append((lo, hi, buf))
            for rq in reqs:
                rq.wait()
            for lo, hi, buf in pending:
                a_panel[(lo - r0) * b:(hi - r0) * b] = buf.numpy()
                recv_bytes += buf.numel() * 8
            if not live:
                continue
            owner = [s for (s, d, _, _) in b_moves if d == rank][0]
            if owner == rank:
                b_row = torch.from_numpy(B_loc[(k - r0) * b:(k - r0 + 1) * b].copy())
            else:
                b_row = torch.empty((b, w * b), dtype=torch.float64)
            if len(members[col]) > 1:                  # vertical broadcast in the column
                dist.broadcast(b_row, src=owner, group=groups[col])
                if owner != rank:
                    recv_bytes += b_row.numel() * 8
            assert not np.isnan(a_panel).any()
            C += a_panel @ b_row.numpy()            # C_i += A(b) B(b)
        ok = True
        if live:
            A_rows = synth.rect(1, N, r0 * b, 0, h * b, N, synth.DIST_INT, np.float64)
            B_cols = synth.rect(2, N, 0, c0 * b, N, w * b, synth.DIST_INT, np.float64)
            ok = bool(np.array_equal(C, og.gemm(A_rows, B_cols)))
        q.put((rank, ok, recv_bytes))
        dist.barrier()
        dist.destroy_process_group()
    except Exception as e:  # pragma: no cover
        q.put((rank, repr(e), -1))


def _run(world, rects, N, b):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, rects, N, b, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = [q.get(timeout=240) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    return sorted(out)


def test_two_ranks_canonical_arrangement():
    """p = 2: the canonical arrangement is one column (B moves vertically only)."""
    import paper_conf_cluster_zhongrl12_b200 as pkg
    N, b = 96, 8
    n = N // b
    d = pkg.fpm_partition(n * n, [([1], [3.0]), ([1], [1.0])])
    rects = pkg.colpart_arrange(n, d)
    out = _run(2, rects, N, b)
    assert all(ok is True for (_, ok, _) in out), out
    assert sum(by for (_, _, by) in out) > 0


def test_two_ranks_two_columns():
    """A forced side-by-side arrangement: A slices move horizontally every iteration."""
    N, b = 96, 8
    n = N // b
    rects = [(0, 0, 0, n, 5), (1, 0, 5, n, n - 5)]
    out = _run(2, rects, N, b)
    assert all(ok is True for (_, ok, _) in out), out
    assert all(by > 0 for (_, _, by) in out)


def test_three_ranks_mixed():
    import paper_conf_cluster_zhongrl12_b200 as pkg
    N, b = 120, 8
    n = N // b
    rects = pkg.colpart_arrange(n, [100, 70, 55])
    assert len({r[0] for r in rects}) == 2            # a 2-device column and a 1-device column
    out = _run(3, rects, N, b)
    assert all(ok is True for (_, ok, _) in out), out
