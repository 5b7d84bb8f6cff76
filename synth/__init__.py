"""Seeded synthetic inputs shared by the oracle (tests) and the CUDA path. Holds none of the
method's arithmetic: only random draws with fixed seeds (DESIGN.md §5 input recipe)."""
