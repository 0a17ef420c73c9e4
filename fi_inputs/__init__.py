"""Seeded synthetic input generators shared by the oracle tests and the CUDA
path.  Holds the program *format* and generators only — none of the method's
arithmetic (counting, selection, injection, classification)."""
from . import isa, program, programs  # noqa: F401
from .program import Program  # noqa: F401
