"""Measurement harnesses (sweep, multi-GPU runner, report) built on the public binding."""
