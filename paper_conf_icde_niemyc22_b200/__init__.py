"""B200-native TSPLIT: micro-tensor split execution of a training step under a
hard HBM budget (Nie et al., ICDE'22).  The compute path lives in libtsplit.so
(C ABI, include/ts.h); `tsplit` is its thin ctypes binding."""

from .tsplit import Graph, Plan, Profile, TsError, lib  # noqa: F401
