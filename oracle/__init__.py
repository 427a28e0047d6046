"""TEST INFRASTRUCTURE ONLY: the CPU oracle for the Menos server segment.

Importable only from tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / --impl reference legs.  The product path never imports it.
"""
