"""CPU oracle -- TEST INFRASTRUCTURE ONLY (see oracle/oracle.py header).

Importable only by tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / --impl reference legs; never by the product package."""
