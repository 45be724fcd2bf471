"""souffle-b200: Souffle's (ASPLOS'24) fused-subprogram execution path, B200-native.

libsouffle.so (C ABI, include/souffle.h) builds a tensor-expression program, analyses and
partitions it (§5) and runs every subprogram as one persistent sm_100a kernel (§6).
This package holds the thin ctypes binding (`_lib`), the model builders (`models`) and the torch
device-memory plumbing (`session`)."""
from . import _lib  # noqa: F401
