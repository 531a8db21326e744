"""Seeded synthetic inputs shared by the oracle tests and the CUDA path.

This package holds ONLY input generators: IR kernel texts and seeded buffer
contents for the BASELINE.json configs (C1-C5) and random IR programs for
property tests.  It contains none of the method's arithmetic (no liveness,
no flashback analysis, no save/restore, no interpreter) and imports neither
``oracle`` nor ``paper_conf_ipps_jiw21_b200``.  Input recipes are described in
DESIGN.md "Inputs".
"""
