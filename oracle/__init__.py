"""CPU oracle for the GSAP hot path — TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
reference leg may import this package.  See oracle/gsap_oracle.c.
"""
