"""FLEP oracle — TEST INFRASTRUCTURE ONLY.

A plain, slow, obviously correct CPU implementation of what the FLEP hot path computes
(Wu, Liu, Zhou, Jiang, "FLEP: Enabling Flexible and Efficient Preemption on GPUs", ASPLOS'17;
`P:N` = line N of the paper text). Only `tests/`, `__graft_entry__.smoke()` and `bench.py`'s
`cpu_baseline` / `--impl reference` legs may import anything from here. The product path
(`paper_conf_asplos_wulzj17_b200/`) never imports it and shares no code with it; the only
common dependency is `synth/` (seeded input generators, no method arithmetic).

Modules
  workloads  — plain definitions of the original block bodies (SAXPY, SpMV-CSR, stencil5, GEMM)
  coverage   — step-by-step model of the persistent-CTA wrapper protocol (Fig. 4) with an
               exhaustive interleaving explorer
  des        — discrete-event simulation of the runtime policies (Fig. 6, §5): FIFO, HPF(+SRPT),
               kernel slicing; simulate and replay modes
  estimates  — ridge-regression duration model (§4.2) and the preemption-overhead mean
  intile     — k-step model of in-tile preemption of the contraction body (R21)
  clc        — step model of the CLC task fetch (R25) with an exhaustive explorer
  metrics    — NTT / ANTT / STP / speedup / spatial-overhead definitions (§6.1)

Parity status: every function is pinned by `tests/test_oracle_*.py`
except absolute timings, which are reported, not checked ("parity unpinned": none of the
oracle's *functions*; the timing model constants of `des.simulate` are inputs, not results).
"""
