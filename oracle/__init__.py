"""ORACLE — test infrastructure only.

A plain, slow, obviously-correct CPU (fp64 / exact-rational) implementation of what
the hot path computes, written from the paper text
(/root/reference/PAPER.md, Sojoodi et al., SC-W '25; cited as ``P:<line>``).

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import, call or execute anything in this package.
The product path (``paper_conf_sc_sojoodiasfga25_b200``) never imports it, and this
package never imports the product path.  The two share no code; the only common
module is ``synth`` (seeded input generators, no model arithmetic).

Modules
-------
model      Eq 1-24 (§3), the O2 evaluator and the O3 selector (Alg 1, §4).
optimize   Exact optimisers (rational water-filling, continuous-k / integer-k level
           bisection, active-set LP) and brute-force grids — used only to pin
           ``model``.
pipeline   Discrete-event simulation of a two-stage staged path (pins Eq 13).
transfer   The memcpy reference transfer replayed through a chosen split (O1).
calibration  The Step-1 Hockney fit (reading C12).
flows      Concurrent-flow (MaxRate-style) selection, NEXT f1 (reading C19).
bands      Size bands of the Step-1 parameters, NEXT f4 (reading C20).
collectives  MPI Alltoall / Allreduce definitions and a plain plan executor, NEXT f3.
"""
