"""ORACLE -- TEST INFRASTRUCTURE ONLY.

A plain, slow, obviously-correct CPU implementation of what the TGOpt hot
path computes, written from /root/reference/PAPER.md (TGOpt, PPoPP'23) and the
readings listed in DESIGN.md ("Readings of the paper").

  oracle.tgat   -- the baseline TGAT forward (no dedup, no memoization, no
                   precomputed time encoding): the *definition* the optimised
                   path must reproduce.
  oracle.tgopt  -- Alg. 1/2/3 followed step by step (DedupFilter, ComputeKeys,
                   CacheLookup, CacheStore with FIFO eviction, precomputed
                   time-encoding window), used for the invariance pin and for
                   the exact integer counters (dedup / hit / miss / eviction).

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / reference
leg may import this package. The product path (paper_conf_ppopp_wangm23_b200)
never imports it and shares no code with it.

Parity-pin status (see tests/test_oracle_*.py and DESIGN.md):
  sampler, dedup, keys, time encoding, attention M, merge FFN, recursion,
  Alg.1 simulator, counters  -- pinned;
  link-prediction score      -- pinned to torch float64 Linear/ReLU/sigmoid
                                only (no printed value in the paper).
"""
