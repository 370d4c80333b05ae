"""Seeded workload descriptions and input generators shared by oracle/ and the CUDA path.

Holds no arithmetic of the method: only program *descriptions* (kernels as RPN)
and seeded input arrays.  See program.py for the encoding."""
from . import program, programs, data  # noqa: F401
