"""Seeded synthetic input generators shared by the oracle side and the CUDA side.

This package holds NO arithmetic of the EATSS method or of any kernel; it only
draws the input arrays (see SURVEY.md §8(d) "Input generators" and DESIGN.md §3).
"""
from .inputs import *  # noqa: F401,F403
