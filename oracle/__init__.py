"""CPU oracle -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline``
/ ``--impl reference`` legs may import, call, link or execute anything in this
package.  The product path (``paper_conf_icppw_matzdf20_b200``) never imports it
and fails loudly when its CUDA extension is missing.

Contents (each function cites the PAPER.md passage it follows; P:Lnnn = line):
  kernels.c / kernels.py  single-device kernel semantics in fp64
  grid.py                 the grid-partition rule (Eq. 8-10; reading Q1)
  regions.py              brute-force address enumeration per partition (c2;
                          P:L451-466 §4.1, §6)
  polyhedral.py           Eq. 1-4 integer sets and the row-wise first/last
                          enumeration of P:L763-775 §6.1 (brute force)
  shadow.py               shadow-memory tracker replaying the Fig. 4 launch
                          sequence (c3)
  closed_forms.py         analytic stale-byte minima and numeric closed forms (c5)

It shares no code with the CUDA path: the only common module is ``synth`` (seeded
random inputs, no method arithmetic).
"""
