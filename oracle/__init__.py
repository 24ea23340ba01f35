"""Split-CNN ORACLE -- test infrastructure, NOT the product path.

A plain, slow, obviously-correct CPU statement of what the split window
operators compute (Jin & Hong, ASPLOS'19, /root/reference/PAPER.md, cited as
P:<line>):

* ``oracle.plan``    -- O1: the split plan, Eq. 1-5, chaining,
                         even (R3) and stochastic (R5) boundaries.
* ``oracle.ops``     -- O2-O8: split (Eq. 4), per-patch conv / max-pool forward and
                         backward (Eq. 6) as fp64 direct loops in C, merge (Eq. 7).
* ``oracle.offload`` -- Algorithm 1 and its reverse pass.
                         PARITY UNPINNED: the paper gives no worked example; only
                         invariants pin it.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  The CUDA path
(``paper_conf_asplos_jinh19_b200``) never imports it and shares no code with it;
the only common module is ``synth`` (seeded input generators, no arithmetic of
the method).
"""
