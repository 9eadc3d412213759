"""CPU oracle for the Stokes-FO cell evaluator -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import anything from here.
The product path (``paper_conf_sc_antepara0cw24_b200``) never imports it and
shares no code with it; the two meet only through the seeded input
generators in ``paper_conf_sc_antepara0cw24_b200/synth.py``.

Contents:
  oracle.c      plain C fp64: reference elements, geometry, residual (both
                Fig. 2 loop orders), forward-AD Jacobian, closed-form tangent,
                gather, scatter, CSR scatter.
  basal.py      numpy basal-friction side-set term (NEXT-4, reading Z18)
  lateral.py    numpy lateral (calving-front) pressure side-set term and the
                footprint boundary-side set (NEXT-4, reading Z19)
  ref.py        ctypes wrapper of oracle.c + numpy O1 extrusion, O9 CSR
                pattern / partition / halo lists, and a numpy complex-step
                residual used as an independent derivative pin.

Parity status per function is listed in DESIGN.md ("Oracle and pins").
"""
from .ref import *  # noqa: F401,F403
