"""TEST INFRASTRUCTURE ONLY: the CPU oracle (unfused executor + reference planner).

May be imported only by tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / --impl reference legs.  Never imported by the product package.
"""
