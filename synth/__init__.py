"""Seeded synthetic input generators (no method arithmetic). See DESIGN.md §4."""
from . import gen  # noqa: F401
