"""DySel oracle — TEST INFRASTRUCTURE ONLY.

A plain, slow, obviously-correct CPU model of what DySel's hot path computes,
written from PAPER.md (cited as ``P:L<a>-<b>``, PAPER.md line numbers, with the
section / figure / table).  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import it.  It
shares no code with the CUDA path (``paper_conf_asplos_changkh16_b200``) and
never imports it; the only shared module is ``workloads`` (seeded inputs).

Halves:
  * numerics   — fp64 SpMV / SGEMM and their |A||x| error denominators
                 (``spmv``, ``sgemm``), the ELL / block-JDS layouts
                 (``formats``);
  * the method — slice planning, ticket order, mode semantics (``slice_plan``),
                 selection by packed argmin and exhaustive best-pure-variant
                 (``selection``).
  * ``c/oracle_ref.c`` — the same fp64 SpMV / GEMM as plain C loops (OpenMP),
                 used for the CPU baseline timing; pinned against ``spmv`` /
                 ``sgemm`` and scipy in tests.

Pins: tests/test_oracle_*.py (``-m "not gpu"``).  Functions without an
independent pin say "parity unpinned" in their docstring.
"""
