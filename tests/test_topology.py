"""Topology discovery and topology-keyed parameters (Step 1: parameters are
"extracted once per system topology and stored on each compute node"; P:359, P:385:
the host path depends on "PCIe configuration, and NUMA effects").

CPU: a topology injected into a model-only context decides the pairs' paths (a relay
needs peer access from the source and to the destination), the fingerprint changes
with what defines the paths, and a parameter file measured on another topology is
refused.  GPU: mp_init finds this GPU (UUID, SMs, NUMA node) and a tampered parameter
file is refused by mp_load_params and by mp_init."""
import os

import pytest

from paper_conf_sc_sojoodiasfga25_b200 import mp

MiB = 1 << 20


def topo(world, nvlinks=18, deny=()):
    pa = [[1] * world for _ in range(world)]
    for a, b in deny:
        pa[a][b] = 0
    gpus = [{"uuid": f"{r:02x}" * 16, "nvlinks": nvlinks, "pcie_gen": 5, "pcie_width": 16, "numa_node": r // 4,
             "sms": 148} for r in range(world)]
    return {"world": world, "gpus": gpus, "peer_access": pa}


def test_unknown_topology_assumes_every_path():
    with mp.Context(rank=0, world=4, model_only=True) as c:
        t = c.topology()
        assert t["fingerprint"] == "0" * 16 and t["peer_access"] == [[1] * 4] * 4
        assert [k for k, _ in c.paths(0, 1)] == [0, 1, 1, 2]


def test_relays_follow_peer_access():
    with mp.Context(rank=0, world=4, model_only=True) as c:
        c.set_topology(topo(4, deny=[(3, 1)]))           # GPU3 cannot reach GPU1
        assert c.paths(0, 1) == [(0, -1), (1, 2), (2, -1)]   # relay 3 excluded (A1)
        assert c.paths(1, 0) == [(0, -1), (1, 2), (1, 3), (2, -1)]
        with pytest.raises(mp.MPError) as e:              # no direct path 3 -> 1
            c.select(3, 1, 64 * MiB)
        assert e.value.status == mp.MP_ERR_TOPOLOGY
        d = c.select(0, 1, 1 << 30).as_dict()
        assert sum(d["bytes"]) == 1 << 30 and len(d["paths"]) == 3
        # a config naming the excluded relay is not available
        t = c.topology()
        assert t["peer_access"][3][1] == 0 and t["gpus"][2]["nvlinks"] == 18


def test_fingerprint_tracks_what_defines_the_paths():
    fps = set()
    for kw in ({}, {"nvlinks": 12}, {"deny": [(0, 2)]}):
        with mp.Context(rank=0, world=4, model_only=True) as c:
            c.set_topology(topo(4, **kw))
            fps.add(c.topology()["fingerprint"])
    assert len(fps) == 3 and "0" * 16 not in fps
    with mp.Context(rank=0, world=4, model_only=True) as a, mp.Context(rank=1, world=4, model_only=True) as b:
        a.set_topology(topo(4))
        b.set_topology(topo(4))
        assert a.topology()["fingerprint"] == b.topology()["fingerprint"]


def test_parameter_file_keyed_by_topology(tmp_path):
    f = str(tmp_path / "p.txt")
    with mp.Context(rank=0, world=3, model_only=True) as c:
        c.set_topology(topo(3))
        c.select(0, 1, MiB)                              # materialise a pair model
        prm = c.get_model(0, 1)
        c.save_params(f)
    text = open(f).read()
    assert "topology " in text and text.count("\ngpu ") == 3
    with mp.Context(rank=0, world=3, model_only=True) as same:
        same.set_topology(topo(3))
        same.load_params(f)                              # same topology: accepted
        assert same.get_model(0, 1)[1] == prm[1]
    with mp.Context(rank=0, world=3, model_only=True) as other:
        other.set_topology(topo(3, nvlinks=6))           # another node: refused
        with pytest.raises(mp.MPError) as e:
            other.load_params(f)
        assert e.value.status == mp.MP_ERR_TOPOLOGY
    with mp.Context(rank=0, world=3, model_only=True) as unknown:
        unknown.load_params(f)                           # no topology known: accepted
    # a file without a fingerprint (round-1 format) is accepted
    g = str(tmp_path / "old.txt")
    open(g, "w").write("".join(l for l in text.splitlines(True) if not l.startswith(("topology", "gpu "))))
    with mp.Context(rank=0, world=3, model_only=True) as other:
        other.set_topology(topo(3, nvlinks=6))
        other.load_params(g)


def test_set_topology_needs_model_only_and_matching_world():
    with mp.Context(rank=0, world=2, model_only=True) as c:
        with pytest.raises(mp.MPError) as e:
            c.set_topology(topo(3))
        assert e.value.status == mp.MP_ERR_INVALID


@pytest.mark.gpu
def test_init_discovers_this_gpu_and_refuses_foreign_params(tmp_path):
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    f = str(tmp_path / "p.txt")
    with mp.Context(device=0, n_loop_relays=1, host_path=1, heap_bytes=MiB, slot_bytes=4 * MiB) as c:
        t = c.topology()
        g = t["gpus"][0]
        p = torch.cuda.get_device_properties(0)
        assert t["world"] == 1 and t["fingerprint"] != "0" * 16 and t["peer_access"] == [[1]]
        assert g["sms"] == p.multi_processor_count and g["numa_node"] >= -1
        # all 16 bytes, also when one of them is 0x00 (torch prints it as GPU-xxxxxxxx-...)
        assert g["uuid"] == str(p.uuid).replace("-", "")[-32:], (g["uuid"], str(p.uuid))
        c.save_params(f)
        c.load_params(f)                                 # its own file: accepted
        text = open(f).read()
        fp = t["fingerprint"]
        bad = text.replace(f"topology {fp}", "topology " + ("f" * 16 if fp != "f" * 16 else "e" * 16))
        open(f, "w").write(bad)
        with pytest.raises(mp.MPError) as e:
            c.load_params(f)
        assert e.value.status == mp.MP_ERR_TOPOLOGY
    with pytest.raises(mp.MPError) as e:                 # Step 2 at init refuses it too
        mp.Context(device=0, n_loop_relays=1, host_path=1, heap_bytes=MiB, slot_bytes=4 * MiB, param_file=f)
    assert e.value.status == mp.MP_ERR_TOPOLOGY


def test_uuid_with_zero_bytes_round_trips():
    # a UUID byte of 0x00 must not truncate it (ctypes c_char arrays stop at NUL)
    u = "1420007b081a9ba3ebae706046e09f87"
    t = topo(2)
    t["gpus"][0]["uuid"] = u
    t["gpus"][1]["uuid"] = "00" * 16
    with mp.Context(rank=0, world=2, model_only=True) as c:
        c.set_topology(t)
        got = c.topology()
        assert [g["uuid"] for g in got["gpus"]] == [u, "00" * 16]
