"""CPU float64 oracle of E.T.'s hot path (PAPER.md = dblp/paper_conf_sc_chenhplg0d021).

THIS PACKAGE IS TEST INFRASTRUCTURE.  Only `tests/`, `__graft_entry__.smoke()`
and `bench.py`'s `cpu_baseline` / `--impl reference` legs may import it.  The
product path (`paper_conf_sc_chenhplg0d021_b200`, `libet.so`) never imports,
links or calls anything here, and this package shares no code with it; the
only common module is `et_synth` (seeded input generators, no method
arithmetic).

Modules:
  prune     -- tile / row / column pruning, masks, CSR index
  encoder   -- the pruned encoder forward, literally (Eq. 3-4, lines 68-75)
  variants  -- independent formulations used only as pins (Fig. 3(a) per-row OTF,
               Eq. 5 pre-computed operator, scalar brute force)

Every function is pinned by a `-m "not gpu"` test in tests/test_oracle_*.py
against closed forms, torch float64 library routines at ratio 0, brute force
on tiny inputs and hand-computed fixtures (tests/golden/).  No function is
"parity unpinned".
"""
from oracle import prune, encoder, variants  # noqa: F401
