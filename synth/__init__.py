"""Seeded synthetic inputs shared by the oracle tests and the CUDA path tests.

This package holds NO arithmetic of the method (no routing, splitting,
scheduling or eviction).  It only produces inputs:

* ``payload``  -- SplitMix64 counter-mode byte streams,
* ``calib``    -- synthetic calibration (topology) descriptions,
* ``traces``   -- request traces for configs 1-5 and random
                  fuzz traces.

Both ``oracle/`` and the library-side test runner consume these; neither
imports the other.
"""
