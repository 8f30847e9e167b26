"""CPU oracle of the LFD step (TEST INFRASTRUCTURE ONLY).

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline / ``--impl reference``
leg may import this package. The product path (``paper_conf_ipps_razakhllknvn24_b200``) never does.
"""
