"""Seeded synthetic read generator -- shared by tests, bench and smoke.

Holds none of the method's arithmetic (no encoding, minimizers, hashing or
counting): it only draws a genome and reads from it, as ASCII bytes plus
read offsets.  Both the CUDA path (after its own host encoder) and the oracle
(with its own decoder) consume this output.  The recipe per configuration is
in DESIGN.md "Inputs" and follows SURVEY.md Sec. 8(d).
"""
from .reads import CONFIGS, ReadSet, genome, make_reads, make_config, random_reads

__all__ = ["CONFIGS", "ReadSet", "genome", "make_reads", "make_config", "random_reads"]
