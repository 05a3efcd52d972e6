"""Seeded synthetic inputs (designs + stimuli) shared by the oracle tests and
the CUDA path. Input plumbing only: nothing here evaluates the design."""
from . import ir, builder, designs, stim, shaped  # noqa: F401
from .ir import IR, OPCODES  # noqa: F401
