import sys, os
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", ".."))
import numpy as np, torch
import synth
import paper_conf_cluster_zhongrl12_b200 as pkg
N, b = 1024, 128
n = N // b
for devs, d in (([0, 0], [40, 24]), ([0], [64])):
    rects = pkg.colpart_arrange(n, d)
    A = synth.rect(1, N, 0, 0, N, N); B = synth.rect(2, N, 0, 0, N, N)
    hA = torch.from_numpy(A).pin_memory(); hB = torch.from_numpy(B).pin_memory()
    hC = torch.full((N, N), float("nan")).pin_memory()
    for tail in (-1, 0, 1, 2, 3, 4):
        with pkg.Context.local(devs) as ctx:
            ctx.set_option("e2e_tail", tail)
            for _ in range(2):
                st = ctx.run(hA, hB, hC, N, b, rects, pkg.FPM_F32)
            print(devs, tail, "updates", st.updates, "t_compute", st.t_compute_s, "t_up", st.t_upload_s, "t_down", st.t_download_s, flush=True)
