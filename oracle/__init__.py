"""CPU oracle for the Tacker hot path — TEST INFRASTRUCTURE ONLY.

Plain, slow, obviously-correct fp64 reference implementations of what the B200 path
computes, written from the paper (/root/reference/PAPER.md, cited as P:a-b) and, where
the paper is silent, from the readings recorded in DESIGN.md §2 (= SURVEY.md §8(c)).

Rules:
  * Only `tests/`, `__graft_entry__.smoke()` and `bench.py`'s cpu_baseline / --impl
    reference legs may import anything under `oracle/`.  The product package never does.
  * The oracle shares no code with the CUDA path (no kernels, headers, tables or helpers);
    the only common module is `synth` (seeded input generators, no method arithmetic).
  * Every function is pinned by `-m "not gpu"` tests in tests/test_oracle_*.py against
    something other than itself (closed forms, brute force on tiny inputs, invariants,
    worked examples from the paper).  Functions without such a pin say "parity unpinned".

Modules:
  lc         LC tensor-core work: fp16 GEMM D = A.B^T, implicit-GEMM convolution (c1, c2)
  be         BE CUDA-core kernels: sgemm, stencil, mri-q, cutcp, lbm, spmv(JDS), histo,
             bfs, fma_burn (c3-c10)
  fusion     Fused-kernel index mapping (Fig. 5/6), PTB coverage (Fig. 7), budget (§V-C)
  predictor  Per-kernel LR and two-stage fused-duration model (§VI, Eqs. 1-6)
  manager_ref  Discrete-event reference of the QoS-aware manager (§VII, Eqs. 7-9)
  metrics    Eq. 10 throughput improvement, Eq. 11 overlap rate, parity error metric
"""
