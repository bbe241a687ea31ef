"""ORACLE — TEST INFRASTRUCTURE ONLY (see oracle/oracle.c).  Importable only from tests/,
__graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs."""
from .oracle import *  # noqa: F401,F403
