"""Seeded synthetic-input generators shared by the oracle, the tests and bench.py.

This package holds NONE of the method's arithmetic (no progress order, no squad
generation, no predictors, no quota apportionment, no layer maths).  It only
draws seeded random inputs and reads/writes the three shared file formats:

* ``trace.jsonl``   -- request arrivals ``(arrival_ns:int64, tenant:int)``
* ``profile.txt``   -- the kernel x SM-count duration table ``t[j][k][s]``
* ``params.json``   -- scheduler parameters

Everything is generated once, in Python, with numpy PCG64 and recorded seeds,
and stored as integers so that the C++ scheduler and the Python oracle read
byte-identical inputs.
"""
from . import trace, profile, tensors  # noqa: F401
