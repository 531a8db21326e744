"""CTXBack oracle -- TEST INFRASTRUCTURE ONLY.

A plain, slow, obviously-correct CPU implementation of what the CTXBack hot
path computes (Ji & Wang, "CTXBack: Enabling Low Latency GPU Context Switching
via Context Flashback", IPDPS 2021; `P:n` = line n of the paper text):

* ``oracle.ir``        -- the oracle's own parser of the IR text format
                          (DESIGN.md "IR v1"); shares no code with the C++ one.
* ``oracle.fp32``      -- exact IEEE binary32 arithmetic (RN, no FTZ), incl. a
                          correctly rounded fused multiply-add.
* ``oracle.interp``    -- SIMT interpreter of the IR (warps of 32 lanes,
                          uniform branches) with preempt / poison / restore /
                          replay of a flashback plan.
* ``oracle.analysis``  -- liveness, windows, the flashback-point
                          search of Alg. 1 / Alg. 2 / OSRB in the
                          normative sweep reading CTXB-R1,
                          plan selection and context accounting.
* ``oracle.brute``     -- brute-force enumeration (BF1-BF3) for tiny kernels.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline /
``--impl reference`` leg may import this package.  The product path
(``paper_conf_ipps_jiw21_b200``) never imports it, and this package never
imports the product.  Every function names the passage it follows.

Parity status: every function is pinned by ``tests/test_oracle_*.py`` against
the paper's worked examples (Figs 2-6), closed forms, textbook routines or
brute force, except where its docstring says "parity unpinned".
"""
