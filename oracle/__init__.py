"""ORACLE — plain, slow, obviously-correct CPU implementation of the paper's
two-dimensional weighted-checksum ABFT (Chen et al., SC'18; reference
`PAPER.md`, cited as L<line> + section).

THIS PACKAGE IS TEST INFRASTRUCTURE.  Only `tests/`, `__graft_entry__.smoke()`
and `bench.py`'s `cpu_baseline` / `--impl reference` legs may import it.  It
shares no code with the CUDA path (`paper_conf_sc_chenlllwtolzgc18_b200/`):
neither imports the other; the only common dependency is `synth_inputs`
(seeded input generators, no method arithmetic).

Precision: float64 throughout (the paper's experiments are double precision,
L536).  fp32 GPU data is checked by promoting it and using the fp32 unit
round-off in the thresholds.

Modules
  checksum  — encode / verify / locate / classify+correct   (§8 rows a1–a3)
  updates   — PD/PU/TMU checksum-maintenance rules          (§8 rows a4–a6)
  drivers   — ft_potrf / ft_getrf / ft_geqrf, Alg. 2 order  (§8 row a7)

Parity status of every function is stated in its docstring; functions with
no independent pin say "parity unpinned" (also listed in DESIGN.md §4).
"""
