"""ORACLE package — TEST INFRASTRUCTURE ONLY.

Plain, slow, obviously-correct CPU implementations written from PAPER.md
(encoder forward of a per-length runtime: ``encoder``; Arlo's Request and
Runtime Schedulers: ``scheduler``).  Only ``tests/``, ``__graft_entry__.smoke()``
and ``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import it.
The product path never routes through it.
"""
