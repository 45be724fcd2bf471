"""Oracle for the Souffle B200 hot path — TEST INFRASTRUCTURE ONLY.

A plain, slow, obviously-correct CPU implementation (fp64 numpy / pure Python) of what the
fused-subprogram path computes, written from PAPER.md.  It shares no code with the CUDA path
(`paper_conf_asplos_xiazswwyfc24_b200/`), and neither imports the other.  Only tests/,
__graft_entry__.smoke() and bench.py (cpu_baseline leg and --impl reference) may import it.

Modules:
  te.py        unfused TE interpreter (vectorised + brute force), oracle-own bf16 rounding
  analysis.py  classification, reuse sets, BFS order, partition, index maps, horizontal groups
  graphs.py    the oracle's own TE-program builders (Fig. 2/3/4, BERT layer, MMoE, LSTM)
  models.py    direct formulas of the evaluated models (plain definitions)

Parity status: every function is pinned by tests in tests/test_oracle_*.py; see DESIGN.md
"Oracle pins".  MMoE sizes are a reading ("parity unpinned" for the sizes only).
"""
