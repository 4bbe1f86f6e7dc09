"""Seeded input generators (no method arithmetic); shared by oracle-side and CUDA-side tests."""
