"""FlashPS oracle: a plain, slow, obviously-correct CPU implementation of the hot path.

TEST INFRASTRUCTURE ONLY. Only `tests/`, `__graft_entry__.smoke()` and `bench.py`'s
`cpu_baseline` / `--impl reference` legs may import or execute anything under `oracle/`.
The product path (`paper_conf_eurosys_jianglyfdlzllyl26_b200/`) never imports it, shares no code
with it, and fails loudly when its CUDA library is missing.

Precision: float64 numpy over inputs that are already rounded to their storage precision by
`synth` (bf16 or fp32). Library primitives used as single steps: `numpy.matmul`, `numpy.exp`,
`numpy.tanh`. No blocking, fusion or reordering beyond what the paper's definitions state.

Citations: `Lnnn` = /root/reference/PAPER.md line nnn (section / figure / table / algorithm
named beside it). Readings of silent or garbled passages are numbered R1.. in DESIGN.md.

Modules
  index     a1, a2, a9   mask -> sorted token ids; gather/scatter of rows
  block     a4-a8        dense block B(x); mask-aware block in KV- and Y-cache modes
  stack     a3, a9, a10  template run (cache producer), masked denoising step over N blocks
  counters  Table 1      FLOP / cache-byte closed forms per mode
  pipeline  Alg. 1       pipeline-latency simulator, brute-force and DP planners
  sched     Alg. 2, §4.4 least-squares latency models, greedy mask-aware routing, DES

Parity pins for every function are in tests/test_oracle_*.py; nothing here is "parity unpinned"
except the end-to-end speedups quoted from the paper (context only).
"""
