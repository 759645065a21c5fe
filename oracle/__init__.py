"""TagMatch ORACLE (TEST INFRASTRUCTURE ONLY).

o1: the plain definition in Python (sec. 2-3).
o2: the paper's CPU method in plain C (oracle/o2.c), loaded through ctypes.

Only tests/, __graft_entry__.smoke() and bench.py (cpu_baseline leg and
--impl reference) may import this package.  The product path never does.
"""
