"""Seeded synthetic input generators shared by the CUDA path tests/bench and the oracle."""
