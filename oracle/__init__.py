"""CPU oracle for the state-vector hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import or execute anything in
this package.  The product library (``paper_conf_sc_markidis23_b200``) never
imports it and shares no code, header, table or constant with it; the only
common module is ``workloads/`` (seeded inputs, no method arithmetic).

Contents, each a plain and slow transcription of the paper / SURVEY.md §8c:

* ``sv``      -- S0 simulator: psi' = G psi applied gate by gate, matrix-free
                 (§2.2 Fig. 3/4), complex128; plus the
                 brute-force full 2^n x 2^n unitary for n <= 10.
* ``fuse``    -- S3 greedy fuser (§2.2 Fig. 5).
* ``plan``    -- S4 global/local qubit-map planner and a virtual-shard
                 emulator of its exchanges (north star).
* ``sample``  -- S5 fixed-point sampler.
* ``sv_ref.c``-- the S0 loop in plain C + OpenMP (complex128, unfused), used
                 for large n and as the timed CPU baseline.

Parity status of every function is listed in DESIGN.md §Oracle; all are
pinned by tests under ``tests/oracle`` against closed forms, brute force,
identities or the SURVEY.md Appendix C regression vectors.
"""
