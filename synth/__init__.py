"""Seeded synthetic protein workloads shared by tests/ and bench.py.

Holds none of the method's arithmetic: no scoring matrix, no words, no hits.
It only draws residues (Robinson-Robinson background), lengths and planted
query copies, as stated in DESIGN.md ("Input recipe").
"""
from .generate import (CONFIGS, RR_FREQ, SyntheticDB, gen_db, gen_query, gen_queries, config_offsets,
                       config_workload)

__all__ = ["CONFIGS", "RR_FREQ", "SyntheticDB", "gen_db", "gen_query", "gen_queries", "config_offsets",
           "config_workload"]
