"""Seeded synthetic input generators (no method arithmetic); see generators.py."""
from .generators import CONFIGS, NAMES, generate

__all__ = ["CONFIGS", "NAMES", "generate"]
