"""CPU oracle for the Aho-Corasick scan -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
``--impl reference`` legs may import this package.
"""
from .oracle import Oracle, build_oracle  # noqa: F401
