"""BLESS oracle -- TEST INFRASTRUCTURE ONLY.

A plain, slow, obviously-correct CPU implementation of what the B200 hot path
computes, written from the paper (PAPER.md = Zhang et al., "Improving GPU
Sharing Performance through Adaptive Bubbleless Spatial-Temporal Sharing",
EuroSys '25) and the readings recorded in DESIGN.md §3:

* ``sched_ref``  -- quota apportionment, request-progress order, kernel-squad
  generation, the two squad-duration predictors (Eq. 1, Eq. 2), the argmin
  over the execution-configuration space by plain enumeration, and the
  Semi-SP range plan (§4.3-§4.5).
* ``des``        -- a discrete-event model that drives ``decide_ref`` on a
  virtual clock, plus ISO/STATIC and TEMPORAL latency models.
* ``layers_ref`` -- float64 numpy reference of the tenants' layers.
* ``metrics_ref``-- latency statistics, quota attainment, latency deviation.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline /
``--impl reference`` legs may import this package.  It shares no code with the
product (``paper_conf_eurosys_zhangcc0xz0g25_b200``) and never imports it; the
only common module is ``synth`` (seeded input generators and file formats,
which contain none of the method's arithmetic).
"""
