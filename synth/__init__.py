"""Seeded synthetic inputs (genome pairs + seed lists).  Holds none of the method's arithmetic; the only
module shared by the oracle tests and the CUDA path (see synth.genome)."""
