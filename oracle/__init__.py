"""CPU oracle for the FPM-partitioned column-based parallel matrix multiplication.

TEST INFRASTRUCTURE ONLY.  Nothing in the product path
(``paper_conf_cluster_zhongrl12_b200``) may import, call, link or execute
anything under ``oracle/``.  The only permitted users are ``tests/``,
``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` leg.  The oracle shares no code with the CUDA path; its
inputs come from :mod:`synth` (a generator module that holds none of the
method's arithmetic).

Source: Zhong, Rychkov, Lastovetsky, Cluster 2012 -- ``PAPER.md`` line numbers
are cited as ``P:<line>``.

Contents
--------
``oracle.fpm``    O1 model evaluation, O2 canonical partition, O4 column-based
                  arrangement, O6 pivot delivery plan (pure Python, plain loops).
``oracle.gemm``   O5 plain triple-loop GEMM in C (``gemm.c``, FP64 accumulation,
                  OpenMP over rows, no BLAS) loaded through ctypes.

Parity status (also in DESIGN.md §"Oracle pins"):
    model eval, partition, arrangement, plan, GEMM -- pinned by tests/test_oracle_*.py
    speed functions measured by fpm_sample -- parity unpinned (hardware timing)
"""
