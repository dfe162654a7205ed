"""TEST INFRASTRUCTURE: the independent fp64 CPU oracle (see oracle.py, bvh_oracle.cpp).

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
reference legs may import this package.
"""
