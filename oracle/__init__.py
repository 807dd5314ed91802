"""CPU oracle for the Strings scheduler hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import, call or execute
anything in this package.  The product path (``paper_conf_sc_senguptagsp14_b200``)
never imports it and fails loudly when its CUDA library is missing.

Modules:
  des         deterministic discrete-event model of the two-level scheduler
  kernels     plain CPU VSCALE / GEMM / XFER (closed-form tenant results)
  metrics     Jain (Eq. 3), weighted speedup (Eq. 2), overlapped roofline T*_d
  bruteforce  optimal static vector-load placement for tiny job sets
  invariants  I1-I5 checker for any decision trace

Pins (tests/test_oracle_*.py, all ``-m "not gpu"``) tie every function to
something other than itself: the paper's rules as worked cases, closed forms
(M/M/1, Eq. (1) geometric decay, Jain limits), published MurmurHash3 test
vectors, exact integer GEMM, brute-force optimal placements and Graham's
list-scheduling bound.  Functions without such a pin are listed in DESIGN.md
§6 as "parity unpinned":  the trace record format, the weighted-LAS
cross-multiplication, the quantum/epoch boundary convention, the admission
cap, the SFT EWMA and the arbiter trigger (paper silent; readings R-5, R-7,
R-12, R-14, R-15, R-20).
"""
