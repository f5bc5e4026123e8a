"""KTILER oracle — TEST INFRASTRUCTURE ONLY (see oracle.py / ktiler_oracle.c headers).

Only tests/, __graft_entry__.smoke() and bench.py (cpu_baseline, --impl reference) may import this.
"""
