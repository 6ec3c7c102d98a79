"""CPU oracle — TEST INFRASTRUCTURE ONLY (see occu_oracle.py header).

May be imported only by tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / --impl reference legs.  Never by the product package.
"""
from .occu_oracle import *  # noqa: F401,F403
from . import occu_oracle  # noqa: F401
