"""ORACLE -- test infrastructure only.

A plain, slow, obviously-correct CPU implementation of what gLLM's per-stage
hot path computes (Guo et al., SC'25; /root/reference/PAPER.md):

  * `oracle.scheduler` -- Token Throttling (§3.1 Eq.1-3, §3.2 Eq.4)
    plus the paged-KV block manager, under the canonical readings R1-R18
    (DESIGN.md §3 / SURVEY.md §8(c) O1-O2).
  * `oracle.weights`   -- the counter-based weight generator O4.
  * `oracle.model`     -- fp32 (or fp64) decoder-only transformer forward with
    its own paged cache (§2.1; O3).

Only `tests/`, `__graft_entry__.smoke()` and `bench.py`'s cpu_baseline /
`--impl reference` legs may import anything under `oracle/`.  The product
path (`paper_conf_sc_00090d00l25_b200`) never imports it and the oracle never
imports the product path; the two share only the seeded input generators in
`workloads/`.

Parity status per function is listed in each module header.
"""
