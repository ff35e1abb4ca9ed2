"""ORACLE (test infrastructure only; see oracle/__init__.py).  NEXT f1: concurrent flows.

SURVEY §8(f) f1 / PAPER.md P:97 ("if the communication pattern … can be known ahead
of time, unused paths can be extracted and utilized for multi-path communication more
effectively") and P:410 (future work: "MaxRate when considering contention on shared
links").  Reading C19: a MaxRate-style fair share — every link used by
k of the known concurrent flows gives each of them 1/k of its bandwidth — applied to
the per-pair model, after which each flow is selected on its own (O3):

* the source NVLink egress / destination ingress (the B200 shared port, and the
  direct path's β) are shared by the flows leaving the source / entering the
  destination: both scaled by 1 / max(k_out(src), k_in(dst));
* a relay GPU that is itself an endpoint of a flow has no spare NVLink capacity and
  is excluded; otherwise its two legs are shared by the m flows that may use it:
  β, β' scaled by 1 / m;
* the host path's PCIe up leg is shared by the flows leaving the source that may use
  the host path, its down leg by those entering the destination.

`lp_lower_bound` solves a relaxation of the joint problem (all flows at once, every
NVLink/PCIe port as a capacity constraint) with scipy, for the pin: the fair-share
selection is a feasible point of it, so its makespan can never beat the bound.
"""
from __future__ import annotations

import math
from dataclasses import replace
from typing import List, Sequence, Tuple

from . import model as M


def share_factors(flows: Sequence[Tuple[int, int, int, Sequence[bool]]], paths_of):
    """Per flow: (direct/port divisor, {relay index: divisor or None}, (host up, host down))."""
    k_out, k_in, endpoint = {}, {}, set()
    for s, d, _, _ in flows:
        k_out[s] = k_out.get(s, 0) + 1
        k_in[d] = k_in.get(d, 0) + 1
        endpoint.update((s, d))
    relay_users, host_out, host_in = {}, {}, {}
    for f, (s, d, _, mask) in enumerate(flows):
        for i, p in enumerate(paths_of(f)):
            if not mask[i]:
                continue
            if p.kind == M.GPU_STAGED:
                relay_users[p.via] = relay_users.get(p.via, 0) + 1
            elif p.kind == M.HOST_STAGED:
                host_out[s] = host_out.get(s, 0) + 1
                host_in[d] = host_in.get(d, 0) + 1
    out = []
    for f, (s, d, _, mask) in enumerate(flows):
        port = max(k_out[s], k_in[d])
        relays = {}
        for i, p in enumerate(paths_of(f)):
            if p.kind == M.GPU_STAGED:
                relays[i] = None if p.via in endpoint else relay_users.get(p.via, 1)
        out.append((port, relays, (host_out.get(s, 1), host_in.get(d, 1))))
    return out


def shared_model(paths: Sequence[M.Path], port: M.Port, fac, mask: Sequence[bool]):
    """The per-flow model after the fair-share rule (C19) and the mask after exclusion."""
    pdiv, relays, (hup, hdown) = fac
    new, m = [], list(mask)
    for i, p in enumerate(paths):
        if p.kind == M.DIRECT:
            new.append(replace(p, beta=p.beta / pdiv))
        elif p.kind == M.GPU_STAGED:
            div = relays.get(i)
            if div is None:
                m[i] = False
                new.append(p)
            else:
                new.append(replace(p, beta=p.beta / div, beta2=p.beta2 / div))
        else:
            new.append(replace(p, beta=p.beta / hup, beta2=p.beta2 / hdown))
    nport = M.Port(alpha=port.alpha, beta=port.beta / pdiv if port.beta != math.inf else math.inf)
    return new, nport, m


def select_flows(flows, pair_paths, pair_port, opts: M.Options) -> List[M.Config]:
    """flows: [(src, dst, bytes, mask)], pair_paths(s, d) → [Path], pair_port(s, d) → Port."""
    facs = share_factors(flows, lambda f: pair_paths(flows[f][0], flows[f][1]))
    out = []
    for (s, d, n, mask), fac in zip(flows, facs):
        paths, port, m = shared_model(pair_paths(s, d), pair_port(s, d), fac, mask)
        out.append(M.select(n, paths, opts, port, m))
    return out


def lp_lower_bound(flows, pair_paths, B_nvl: float, B_pcie: float) -> float:
    """A lower bound on the makespan of any schedule of the flows (joint LP relaxation,
    scipy HiGHS): every path carries b at no more than its bottleneck-leg bandwidth
    (T >= b / min(β, β'), no startup terms), every GPU's NVLink egress and ingress
    carry at most T·B_nvl and its PCIe up/down at most T·B_pcie; Σ_paths b = n."""
    from scipy.optimize import linprog
    us = 1e-6
    var = []   # (flow, path index)
    for f, (s, d, n, mask) in enumerate(flows):
        for i, _ in enumerate(pair_paths(s, d)):
            if mask[i]:
                var.append((f, i))
    nv = len(var) + 1
    A_ub, b_ub, A_eq, b_eq = [], [], [], []
    ports = {}
    for j, (f, i) in enumerate(var):
        s, d, n, _ = flows[f]
        p = pair_paths(s, d)[i]
        bw = p.beta if p.kind == M.DIRECT else min(p.beta, p.beta2)
        row = [0.0] * nv
        row[j] = n / bw / us
        row[-1] = -1.0
        A_ub.append(row)
        b_ub.append(0.0)
        use = {M.DIRECT: [("E", s), ("I", d)], M.GPU_STAGED: [("E", s), ("I", p.via), ("E", p.via), ("I", d)],
               M.HOST_STAGED: [("U", s), ("D", d)]}[p.kind]
        for u in use:
            ports.setdefault(u, []).append((j, n))
    for (kind, g), users in ports.items():
        cap = B_pcie if kind in "UD" else B_nvl
        row = [0.0] * nv
        for j, n in users:
            row[j] += n / cap / us
        row[-1] = -1.0
        A_ub.append(row)
        b_ub.append(0.0)
    for f in range(len(flows)):
        A_eq.append([1.0 if ff == f else 0.0 for ff, _ in var] + [0.0])
        b_eq.append(1.0)
    res = linprog([0.0] * (nv - 1) + [1.0], A_ub=A_ub, b_ub=b_ub, A_eq=A_eq, b_eq=b_eq,
                  bounds=[(0, None)] * nv, method="highs")
    assert res.status == 0, res.message
    return res.fun * us
