"""CPU ORACLE package -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
--impl reference legs may import this package.  The product path
(paper_conf_ipps_madougouvln16_b200/) never imports it.
"""
