"""Neutral input module shared by the oracle and the product: DFG descriptions
(`graphs`) and seeded synthetic data (`gen`).  Holds none of the method's
arithmetic (no scheduling, planning, simulation or op maths)."""

from . import gen, graphs  # noqa: F401
