"""Thin ctypes binding of the C ABI in include/mp.h (argument marshalling only).

Every step of the hot path runs in libmpx.so (host C++ model/selector, sm_100a
kernels).  There is no Python or CPU fallback: if the library cannot be loaded the
import raises.
"""
from __future__ import annotations

import ctypes as C
import os
from typing import List, Optional, Sequence

from . import _build

MP_MAX_PATHS = 16
MP_PATH_DIRECT, MP_PATH_GPU, MP_PATH_HOST = 0, 1, 2
MP_MODEL_PAPER, MP_MODEL_B200 = 0, 1
MP_INIT_MODEL_ONLY, MP_INIT_NO_CALIBRATE, MP_INIT_EMULATED = 1, 2, 4
MP_OK, MP_ERR_INVALID, MP_ERR_CUDA, MP_ERR_TOPOLOGY, MP_ERR_NOMEM, MP_ERR_STATE = 0, -1, -2, -3, -4, -5
MP_ERR_UNSUPPORTED, MP_ERR_TIMEOUT, MP_ERR_MISMATCH = -6, -7, -8

STATUS = {0: "MP_OK", -1: "MP_ERR_INVALID", -2: "MP_ERR_CUDA", -3: "MP_ERR_TOPOLOGY",
          -4: "MP_ERR_NOMEM", -5: "MP_ERR_STATE", -6: "MP_ERR_UNSUPPORTED",
          -7: "MP_ERR_TIMEOUT", -8: "MP_ERR_MISMATCH"}


class MPError(RuntimeError):
    def __init__(self, status: int, msg: str = ""):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


class mp_path(C.Structure):
    _fields_ = [("kind", C.c_int32), ("via", C.c_int32)]


class mp_path_params(C.Structure):
    _fields_ = [(n, C.c_double) for n in ("alpha", "beta", "alpha2", "beta2", "eps", "c", "sigma", "w", "wake")]


class mp_port_params(C.Structure):
    _fields_ = [("alpha", C.c_double), ("beta", C.c_double)]


class mp_model_opts(C.Structure):
    _fields_ = [("mode", C.c_int32), ("stagger", C.c_int32), ("refine", C.c_int32),
                ("window", C.c_int32), ("align", C.c_uint64), ("c_min", C.c_uint64),
                ("k_max", C.c_uint64), ("slot_bytes", C.c_uint64)]


class mp_config(C.Structure):
    _fields_ = [("npaths", C.c_int32), ("reserved", C.c_int32),
                ("path", mp_path * MP_MAX_PATHS), ("theta", C.c_double * MP_MAX_PATHS),
                ("bytes", C.c_uint64 * MP_MAX_PATHS), ("chunks", C.c_uint32 * MP_MAX_PATHS),
                ("t_pred", C.c_double), ("t_level", C.c_double)]

    def as_dict(self):
        n = self.npaths
        return dict(paths=[(self.path[i].kind, self.path[i].via) for i in range(n)],
                    theta=[self.theta[i] for i in range(n)],
                    bytes=[int(self.bytes[i]) for i in range(n)],
                    chunks=[int(self.chunks[i]) for i in range(n)],
                    t_pred=self.t_pred, t_level=self.t_level)


class mp_flow(C.Structure):
    _fields_ = [("src", C.c_int32), ("dst", C.c_int32), ("path_mask", C.c_uint32), ("reserved", C.c_uint32),
                ("bytes", C.c_uint64)]


MP_COLL_ALLTOALL, MP_COLL_ALLREDUCE = 0, 1
MP_ALGO_AUTO, MP_ALGO_BRUCK, MP_ALGO_PAIRWISE, MP_ALGO_KNOMIAL, MP_ALGO_RING = 0, 1, 2, 3, 4
MP_BUF_SEND, MP_BUF_RECV, MP_BUF_TMP = 0, 1, 2
MP_DT_U8, MP_DT_I32, MP_DT_I64, MP_DT_F32, MP_DT_F64, MP_DT_BF16 = 0, 1, 2, 3, 4, 5
MP_OP_SUM = 0
MP_COLL_MAX_STEPS, MP_COLL_MAX_SEGS, MP_COLL_MAX_COPIES = 64, 512, 64


class mp_coll_seg(C.Structure):
    _fields_ = [("buf", C.c_int32), ("reserved", C.c_int32), ("off", C.c_uint64), ("len", C.c_uint64)]


class mp_coll_copy(C.Structure):
    _fields_ = [("src_buf", C.c_int32), ("dst_buf", C.c_int32), ("src_off", C.c_uint64), ("dst_off", C.c_uint64),
                ("len", C.c_uint64)]


class mp_coll_step(C.Structure):
    _fields_ = [("send_to", C.c_int32), ("recv_from", C.c_int32), ("reduce", C.c_int32), ("reserved", C.c_int32),
                ("send_seg0", C.c_uint32), ("send_nseg", C.c_uint32), ("recv_seg0", C.c_uint32),
                ("recv_nseg", C.c_uint32), ("bytes", C.c_uint64)]


class mp_coll_plan(C.Structure):
    _fields_ = [("coll", C.c_int32), ("algo", C.c_int32), ("world", C.c_int32), ("rank", C.c_int32),
                ("tmp_bytes", C.c_uint64), ("npre", C.c_int32), ("nsteps", C.c_int32), ("nsegs", C.c_int32),
                ("npost", C.c_int32), ("pre", mp_coll_copy * MP_COLL_MAX_COPIES),
                ("step", mp_coll_step * MP_COLL_MAX_STEPS), ("seg", mp_coll_seg * MP_COLL_MAX_SEGS),
                ("post", mp_coll_copy * MP_COLL_MAX_COPIES)]


class mp_gpu_info(C.Structure):
    # raw bytes (c_ubyte): a c_char array would read back truncated at its first 0x00
    _fields_ = [("uuid", C.c_ubyte * 16)] + [(n, C.c_int32) for n in (
        "device", "pci_domain", "pci_bus", "pci_device", "numa_node", "pcie_gen", "pcie_width", "pcie_gen_cur",
        "nvlinks", "sms", "reserved")]


class mp_topology(C.Structure):
    _fields_ = [("world", C.c_int32), ("reserved", C.c_int32), ("fingerprint", C.c_uint64),
                ("gpu", mp_gpu_info * MP_MAX_PATHS),
                ("peer_access", (C.c_int32 * MP_MAX_PATHS) * MP_MAX_PATHS),
                ("p2p_perf_rank", (C.c_int32 * MP_MAX_PATHS) * MP_MAX_PATHS),
                ("p2p_atomics", (C.c_int32 * MP_MAX_PATHS) * MP_MAX_PATHS)]


ALLGATHER = C.CFUNCTYPE(C.c_int, C.c_void_p, C.c_void_p, C.c_void_p, C.c_uint64)


class mp_init_args(C.Structure):
    _fields_ = [("rank", C.c_int32), ("world", C.c_int32), ("device", C.c_int32), ("flags", C.c_int32),
                ("n_loop_relays", C.c_int32), ("host_path", C.c_int32), ("slots", C.c_int32),
                ("relay_ctas", C.c_int32), ("heap_bytes", C.c_uint64), ("slot_bytes", C.c_uint64),
                ("timeout_s", C.c_double), ("allgather", ALLGATHER), ("allgather_user", C.c_void_p),
                ("param_file", C.c_char_p)]


_lib = None


def lib():
    """Load libmpx.so (building it in-tree with nvcc first if it is missing/stale)."""
    global _lib
    if _lib is None:
        # MPX_LIB: an alternative in-tree build (design experiments, e.g. a variant
        # compiled with other MPX_* defines by _build.build(out=..., defines=...))
        path = os.environ.get("MPX_LIB") or _build.build()
        L = C.CDLL(path, mode=C.RTLD_GLOBAL)
        P = C.c_void_p
        sig = {
            "mp_init": (C.c_int, [C.POINTER(P), C.POINTER(mp_init_args)]),
            "mp_finalize": (C.c_int, [P]),
            "mp_strerror": (C.c_char_p, [C.c_int]),
            "mp_last_error": (C.c_char_p, [P]),
            "mp_abi_version": (C.c_int, []),
            "mp_paths": (C.c_int, [P, C.c_int, C.c_int, C.POINTER(mp_path), C.POINTER(C.c_int)]),
            "mp_set_model": (C.c_int, [P, C.c_int, C.c_int, C.POINTER(mp_path), C.POINTER(mp_path_params),
                                       C.c_int, C.POINTER(mp_port_params)]),
            "mp_get_model": (C.c_int, [P, C.c_int, C.c_int, C.POINTER(mp_path), C.POINTER(mp_path_params),
                                       C.POINTER(C.c_int), C.POINTER(mp_port_params)]),
            "mp_set_options": (C.c_int, [P, C.POINTER(mp_model_opts)]),
            "mp_get_options": (C.c_int, [P, C.POINTER(mp_model_opts)]),
            "mp_predict": (C.c_int, [P, C.c_int, C.c_int, C.c_uint64, C.POINTER(mp_config),
                                     C.POINTER(C.c_double)]),
            "mp_select": (C.c_int, [P, C.c_int, C.c_int, C.c_uint64, C.c_uint32, C.POINTER(mp_config)]),
            "mp_alloc": (C.c_int, [P, C.c_uint64, C.POINTER(P)]),
            "mp_free": (C.c_int, [P, P]),
            "mp_send": (C.c_int, [P, P, C.c_uint64, C.c_int, C.c_int, C.POINTER(mp_config), P]),
            "mp_recv": (C.c_int, [P, P, C.c_uint64, C.c_int, C.c_int, P]),
            "mp_xfer": (C.c_int, [P, P, P, C.c_uint64, C.POINTER(mp_config), P]),
            "mp_sync": (C.c_int, [P]),
            "mp_calibrate": (C.c_int, [P, C.POINTER(C.c_uint64), C.c_int, C.c_int]),
            "mp_save_params": (C.c_int, [P, C.c_char_p]),
            "mp_load_params": (C.c_int, [P, C.c_char_p]),
            "mp_stats": (C.c_int, [P, C.POINTER(C.c_uint64)]),
            "mp_peer_base": (C.c_int, [P, C.c_int, C.POINTER(P)]),
            "mp_register": (C.c_int, [P, P, C.c_uint64, C.POINTER(C.c_int)]),
            "mp_deregister": (C.c_int, [P, C.c_int]),
            "mp_select_flows": (C.c_int, [P, C.c_int, C.POINTER(mp_flow), C.POINTER(mp_config)]),
            "mp_fit_hockney": (C.c_int, [C.POINTER(C.c_double), C.POINTER(C.c_double), C.c_int,
                                         C.POINTER(C.c_double), C.POINTER(C.c_double)]),
            "mp_set_model_band": (C.c_int, [P, C.c_int, C.c_int, C.c_uint64, C.POINTER(mp_path_params),
                                            C.c_int, C.POINTER(mp_port_params)]),
            "mp_get_model_band": (C.c_int, [P, C.c_int, C.c_int, C.c_int, C.POINTER(C.c_uint64),
                                            C.POINTER(mp_path_params), C.POINTER(C.c_int),
                                            C.POINTER(mp_port_params), C.POINTER(C.c_int)]),
            "mp_coll_plan_build": (C.c_int, [C.c_int, C.c_int, C.c_int, C.c_int, C.c_uint64, C.c_uint32,
                                             C.POINTER(mp_coll_plan)]),
            "mp_alltoall": (C.c_int, [P, P, P, C.c_uint64, C.c_int, P]),
            "mp_allreduce": (C.c_int, [P, P, P, C.c_uint64, C.c_int, C.c_int, C.c_int, P]),
            "mp_calibrate_bands": (C.c_int, [P, C.POINTER(C.c_uint64), C.c_int, C.c_int]),
            "mp_set_window_model": (C.c_int, [P, C.c_int, C.c_int, C.POINTER(C.c_double), C.c_int, C.c_double]),
            "mp_get_window_model": (C.c_int, [P, C.c_int, C.c_int, C.POINTER(C.c_double), C.POINTER(C.c_int),
                                              C.POINTER(C.c_double)]),
            "mp_predict_window": (C.c_int, [P, C.c_int, C.c_int, C.c_uint64, C.c_uint32, C.POINTER(mp_config),
                                            C.POINTER(C.c_double)]),
            "mp_select_window": (C.c_int, [P, C.c_int, C.c_int, C.c_uint64, C.c_uint32, C.c_uint32,
                                           C.POINTER(mp_config)]),
            "mp_set_host_duplex": (C.c_int, [P, C.c_int, C.c_double]),
            "mp_calibrate_window": (C.c_int, [P, C.POINTER(C.c_uint64), C.c_int, C.c_int, C.c_int]),
            "mp_calibrate_wake": (C.c_int, [P, C.c_uint64, C.c_int]),
            "mp_fit_window": (C.c_int, [C.POINTER(C.c_int), C.POINTER(C.c_double), C.POINTER(C.c_double),
                                        C.POINTER(C.c_double), C.c_int, C.c_int, C.c_int, C.c_double,
                                        C.POINTER(C.c_double), C.POINTER(C.c_double)]),
            "mp_set_submit_time": (C.c_int, [P, C.c_double]),
            "mp_get_submit_time": (C.c_int, [P, C.POINTER(C.c_double)]),
            "mp_get_host_duplex": (C.c_int, [P, C.c_int, C.POINTER(C.c_double)]),
            "mp_get_topology": (C.c_int, [P, C.POINTER(mp_topology)]),
            "mp_set_topology": (C.c_int, [P, C.POINTER(mp_topology)]),
            "mp_init_emulated": (C.c_int, [C.POINTER(P), C.POINTER(mp_init_args)]),
            "mp_emu_run": (C.c_int, [C.POINTER(P), C.c_int, P, C.POINTER(C.c_double)]),
            "mp_finalize_emulated": (C.c_int, [C.POINTER(P), C.c_int]),
            "mp_emu_register": (C.c_int, [C.POINTER(P), C.c_int, C.POINTER(P), C.POINTER(C.c_uint64),
                                          C.POINTER(C.c_int)]),
            "mp_emu_deregister": (C.c_int, [C.POINTER(P), C.c_int, C.POINTER(C.c_int)]),
            "mp_emu_alltoall": (C.c_int, [C.POINTER(P), C.c_int, C.POINTER(P), C.POINTER(P), C.c_uint64, C.c_int, P]),
            "mp_emu_allreduce": (C.c_int, [C.POINTER(P), C.c_int, C.POINTER(P), C.POINTER(P), C.c_uint64, C.c_int,
                                           C.c_int, C.c_int, P]),
            "mp_fit_bands": (C.c_int, [C.POINTER(C.c_double), C.POINTER(C.c_double), C.c_int,
                                       C.POINTER(C.c_double), C.c_int, C.POINTER(C.c_double),
                                       C.POINTER(C.c_double)]),
        }
        for name, (res, args) in sig.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def exported_symbols() -> List[str]:
    return ["mp_init", "mp_finalize", "mp_strerror", "mp_last_error", "mp_abi_version", "mp_paths",
            "mp_set_model", "mp_get_model", "mp_set_options", "mp_get_options", "mp_predict",
            "mp_select", "mp_alloc", "mp_free", "mp_send", "mp_recv", "mp_xfer", "mp_sync",
            "mp_calibrate", "mp_save_params", "mp_load_params", "mp_stats", "mp_fit_hockney",
            "mp_peer_base", "mp_select_flows", "mp_register", "mp_deregister",
            "mp_set_model_band", "mp_get_model_band", "mp_fit_bands", "mp_calibrate_bands",
            "mp_coll_plan_build", "mp_alltoall", "mp_allreduce",
            "mp_set_window_model", "mp_get_window_model", "mp_predict_window", "mp_select_window",
            "mp_set_host_duplex", "mp_get_host_duplex", "mp_calibrate_window", "mp_calibrate_wake", "mp_fit_window",
            "mp_get_topology", "mp_set_topology", "mp_set_submit_time", "mp_get_submit_time",
            "mp_init_emulated", "mp_emu_run", "mp_finalize_emulated", "mp_emu_alltoall", "mp_emu_allreduce",
            "mp_emu_register", "mp_emu_deregister"]


def fit_hockney(n: Sequence[float], t: Sequence[float]):
    """mp_fit_hockney: (α, β) of the Step-1 weighted Hockney fit (reading C12)."""
    m = len(n)
    a, b = C.c_double(), C.c_double()
    st = lib().mp_fit_hockney((C.c_double * m)(*n), (C.c_double * m)(*t), m, C.byref(a), C.byref(b))
    if st != 0:
        raise MPError(st, "mp_fit_hockney")
    return a.value, b.value


def fit_window(path: Sequence[int], t1: Sequence[float], tw: Sequence[float], pred: Sequence[float],
               window: int, npaths: int, h_sub: float = 0.0):
    """mp_fit_window: (h[npaths], τ) of the C24 estimator (NEXT f2; C27's h_sub)."""
    m = len(path)
    h, tau = (C.c_double * max(1, npaths))(), C.c_double()
    st = lib().mp_fit_window((C.c_int * m)(*path), (C.c_double * m)(*t1), (C.c_double * m)(*tw),
                             (C.c_double * m)(*pred), m, window, npaths, h_sub, h, C.byref(tau))
    if st != 0:
        raise MPError(st, "mp_fit_window")
    return [h[i] for i in range(npaths)], tau.value


def fit_bands(n: Sequence[float], t: Sequence[float], edges: Sequence[float]):
    """mp_fit_bands: [(α_j, β_j)] per size band (reading C20, NEXT f4)."""
    m, B = len(n), len(edges)
    a, b = (C.c_double * B)(), (C.c_double * B)()
    st = lib().mp_fit_bands((C.c_double * max(1, m))(*n), (C.c_double * max(1, m))(*t), m,
                            (C.c_double * B)(*edges), B, a, b)
    if st != 0:
        raise MPError(st, "mp_fit_bands")
    return [(a[j], b[j]) for j in range(B)]


def coll_plan(coll: int, algo: int, world: int, rank: int, nbytes: int, elem_size: int = 1) -> dict:
    """mp_coll_plan_build as plain Python data (NEXT f3)."""
    p = mp_coll_plan()
    st = lib().mp_coll_plan_build(coll, algo, world, rank, nbytes, elem_size, C.byref(p))
    if st != 0:
        raise MPError(st, "mp_coll_plan_build")
    cp = lambda k: dict(src_buf=k.src_buf, dst_buf=k.dst_buf, src_off=k.src_off, dst_off=k.dst_off,  # noqa: E731
                        len=k.len)
    sg = lambda g: dict(buf=g.buf, off=g.off, len=g.len)  # noqa: E731
    steps = []
    for j in range(p.nsteps):
        t = p.step[j]
        steps.append(dict(send_to=t.send_to, recv_from=t.recv_from, reduce=t.reduce, bytes=t.bytes,
                          send_segs=[sg(p.seg[t.send_seg0 + k]) for k in range(t.send_nseg)],
                          recv_segs=[sg(p.seg[t.recv_seg0 + k]) for k in range(t.recv_nseg)]))
    return dict(coll=p.coll, algo=p.algo, world=p.world, rank=p.rank, tmp_bytes=p.tmp_bytes,
                pre=[cp(p.pre[i]) for i in range(p.npre)], post=[cp(p.post[i]) for i in range(p.npost)],
                nsteps=p.nsteps, steps=steps)


def _params_array(params: Sequence[dict]):
    return (mp_path_params * MP_MAX_PATHS)(
        *[mp_path_params(*[float(p.get(f, d)) for f, d in
                           (("alpha", 0), ("beta", 0), ("alpha2", 0), ("beta2", 0), ("eps", 0),
                            ("c", 1), ("sigma", 0), ("w", 0), ("wake", 0))]) for p in params])


def _ptr(x) -> Optional[int]:
    """Device/host pointer of a torch tensor, an int, or None."""
    if x is None:
        return None
    if isinstance(x, int):
        return x
    return x.data_ptr()


def _stream(s) -> Optional[int]:
    if s is None:
        return None
    if isinstance(s, int):
        return s
    return s.cuda_stream


class Context:
    """One mp_ctx.  Methods mirror the C ABI names and raise MPError on failure."""

    def __init__(self, rank=0, world=1, device=0, model_only=False, calibrate=False,
                 n_loop_relays=-1, host_path=-1, slots=0, relay_ctas=0, heap_bytes=0,
                 slot_bytes=0, timeout_s=0.0, allgather=None, param_file=None):
        L = lib()
        a = mp_init_args()
        a.rank, a.world, a.device = rank, world, device
        a.flags = (MP_INIT_MODEL_ONLY if model_only else 0) | (0 if calibrate else MP_INIT_NO_CALIBRATE)
        a.n_loop_relays, a.host_path, a.slots, a.relay_ctas = n_loop_relays, host_path, slots, relay_ctas
        a.heap_bytes, a.slot_bytes, a.timeout_s = heap_bytes, slot_bytes, timeout_s
        self._ag = ALLGATHER(allgather) if allgather else ALLGATHER()
        a.allgather = self._ag
        a.param_file = param_file.encode() if param_file else None
        h = C.c_void_p()
        st = L.mp_init(C.byref(h), C.byref(a))
        if st != 0:
            raise MPError(st, "mp_init failed")
        self.h = h
        self.world, self.rank = world, rank

    @classmethod
    def _wrap(cls, h, rank, world):
        self = cls.__new__(cls)
        self.h, self.rank, self.world = C.c_void_p(h), rank, world
        self._emulated = True
        return self

    def _ck(self, st):
        if st != 0:
            raise MPError(st, lib().mp_last_error(self.h).decode())

    def close(self):
        if getattr(self, "_emulated", False):  # EmulatedWorld.close() tears the world down
            return
        if getattr(self, "h", None):
            lib().mp_finalize(self.h)
            self.h = None

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    def __del__(self):
        # a multi-rank context's mp_finalize is collective: it cannot run from a
        # garbage-collection finaliser (other ranks may be gone); call close() instead.
        if getattr(self, "world", 1) > 1:
            return
        try:
            self.close()
        except Exception:
            pass

    # ---------------------------------------------------------------- model
    def paths(self, src=0, dst=0):
        arr = (mp_path * MP_MAX_PATHS)()
        n = C.c_int()
        self._ck(lib().mp_paths(self.h, src, dst, arr, C.byref(n)))
        return [(arr[i].kind, arr[i].via) for i in range(n.value)]

    def set_model(self, src, dst, paths: Sequence, params: Sequence[dict], port: Optional[dict] = None):
        n = len(paths)
        pa = (mp_path * MP_MAX_PATHS)(*[mp_path(k, v) for k, v in paths])
        pr = _params_array(params)
        po = mp_port_params(port["alpha"], port["beta"]) if port else None
        self._ck(lib().mp_set_model(self.h, src, dst, pa, pr, n, C.byref(po) if po else None))

    def set_model_band(self, src, dst, n_min, params: Sequence[dict], port: Optional[dict] = None):
        """mp_set_model_band (NEXT f4, reading C20)."""
        po = mp_port_params(port["alpha"], port["beta"]) if port else None
        self._ck(lib().mp_set_model_band(self.h, src, dst, n_min, _params_array(params), len(params),
                                         C.byref(po) if po else None))

    def get_model_bands(self, src=0, dst=0):
        """[(n_min, params, port)] of every band of (src, dst), ascending n_min."""
        nb = C.c_int()
        self._ck(lib().mp_get_model_band(self.h, src, dst, -1, None, None, None, None, C.byref(nb)))
        out = []
        for j in range(nb.value):
            lo, n = C.c_uint64(), C.c_int()
            pr = (mp_path_params * MP_MAX_PATHS)()
            po = mp_port_params()
            self._ck(lib().mp_get_model_band(self.h, src, dst, j, C.byref(lo), pr, C.byref(n), C.byref(po), None))
            out.append((lo.value, [{f: getattr(pr[i], f) for f, _ in mp_path_params._fields_}
                                   for i in range(n.value)], dict(alpha=po.alpha, beta=po.beta)))
        return out

    def get_model(self, src=0, dst=0):
        pa = (mp_path * MP_MAX_PATHS)()
        pr = (mp_path_params * MP_MAX_PATHS)()
        n = C.c_int()
        po = mp_port_params()
        self._ck(lib().mp_get_model(self.h, src, dst, pa, pr, C.byref(n), C.byref(po)))
        params = [{f: getattr(pr[i], f) for f, _ in mp_path_params._fields_} for i in range(n.value)]
        return [(pa[i].kind, pa[i].via) for i in range(n.value)], params, dict(alpha=po.alpha, beta=po.beta)

    def set_options(self, mode=MP_MODEL_PAPER, stagger=1, refine=-1, align=256, c_min=65536,
                    k_max=1024, slot_bytes=0, window=1):
        o = mp_model_opts(mode, stagger, refine, window, align, c_min, k_max, slot_bytes)
        self._ck(lib().mp_set_options(self.h, C.byref(o)))

    def get_options(self):
        o = mp_model_opts()
        self._ck(lib().mp_get_options(self.h, C.byref(o)))
        return {f: getattr(o, f) for f, _ in mp_model_opts._fields_}

    def make_config(self, nbytes: Sequence[int], chunks: Sequence[int], src=0, dst=0) -> mp_config:
        cfg = mp_config()
        ps = self.paths(src, dst)
        assert len(nbytes) == len(ps) == len(chunks)
        cfg.npaths = len(ps)
        for i, (k, v) in enumerate(ps):
            cfg.path[i] = mp_path(k, v)
            cfg.bytes[i] = int(nbytes[i])
            cfg.chunks[i] = int(chunks[i])
        return cfg

    def predict(self, src, dst, n, cfg: mp_config) -> float:
        t = C.c_double()
        self._ck(lib().mp_predict(self.h, src, dst, n, C.byref(cfg), C.byref(t)))
        return t.value

    def select(self, src, dst, n, mask=0) -> mp_config:
        cfg = mp_config()
        self._ck(lib().mp_select(self.h, src, dst, n, mask, C.byref(cfg)))
        return cfg

    def select_flows(self, flows):
        """flows: [(src, dst, bytes, mask)] → [mp_config] (NEXT f1, reading C19)."""
        n = len(flows)
        arr = (mp_flow * max(1, n))(*[mp_flow(s, d, m, 0, b) for s, d, b, m in flows])
        out = (mp_config * max(1, n))()
        self._ck(lib().mp_select_flows(self.h, n, arr, out))
        return [out[i] for i in range(n)]

    # ---------------------------------------------------------------- NEXT f2 (C24, C25)
    def set_window_model(self, src, dst, h: Sequence[float], tau: float = 0.0):
        self._ck(lib().mp_set_window_model(self.h, src, dst, (C.c_double * max(1, len(h)))(*h), len(h), tau))

    def get_window_model(self, src=0, dst=0):
        h = (C.c_double * MP_MAX_PATHS)()
        n, tau = C.c_int(), C.c_double()
        self._ck(lib().mp_get_window_model(self.h, src, dst, h, C.byref(n), C.byref(tau)))
        return [h[i] for i in range(n.value)], tau.value

    def predict_window(self, src, dst, n, window, cfg: mp_config) -> float:
        t = C.c_double()
        self._ck(lib().mp_predict_window(self.h, src, dst, n, window, C.byref(cfg), C.byref(t)))
        return t.value

    def select_window(self, src, dst, n, window, mask=0) -> mp_config:
        cfg = mp_config()
        self._ck(lib().mp_select_window(self.h, src, dst, n, window, mask, C.byref(cfg)))
        return cfg

    def set_host_duplex(self, gpu, kappa):
        self._ck(lib().mp_set_host_duplex(self.h, gpu, kappa))

    def calibrate_window(self, sizes: Optional[Sequence[int]] = None, window=16, reps=7):
        """mp_calibrate_window (loopback; readings C24, C25)."""
        arr = (C.c_uint64 * len(sizes))(*sizes) if sizes else None
        self._ck(lib().mp_calibrate_window(self.h, arr, len(sizes) if sizes else 0, window, reps))

    def calibrate_wake(self, nbytes=0, reps=0):
        """mp_calibrate_wake (reading C28; collective, world >= 3)."""
        self._ck(lib().mp_calibrate_wake(self.h, nbytes, reps))

    def set_submit_time(self, seconds: float):
        """mp_set_submit_time (reading C27): the host's time per enqueued message."""
        self._ck(lib().mp_set_submit_time(self.h, seconds))

    def get_submit_time(self) -> float:
        v = C.c_double()
        self._ck(lib().mp_get_submit_time(self.h, C.byref(v)))
        return v.value

    def get_host_duplex(self, gpu) -> float:
        k = C.c_double()
        self._ck(lib().mp_get_host_duplex(self.h, gpu, C.byref(k)))
        return k.value

    # ---------------------------------------------------------------- engine
    def alloc(self, n) -> int:
        p = C.c_void_p()
        self._ck(lib().mp_alloc(self.h, n, C.byref(p)))
        return p.value

    def free(self, p):
        self._ck(lib().mp_free(self.h, p))

    def peer_base(self, rank) -> int:
        v = C.c_void_p()
        self._ck(lib().mp_peer_base(self.h, rank, C.byref(v)))
        return v.value

    def register(self, buf, n=None) -> int:
        """mp_register (collective when world > 1): buf = tensor / pointer / None."""
        if n is None:
            n = 0 if buf is None else buf.numel() * buf.element_size()
        v = C.c_int()
        self._ck(lib().mp_register(self.h, _ptr(buf), n, C.byref(v)))
        return v.value

    def deregister(self, rid):
        self._ck(lib().mp_deregister(self.h, rid))

    def xfer(self, dst, src, n, cfg: Optional[mp_config] = None, stream=None):
        self._ck(lib().mp_xfer(self.h, _ptr(dst), _ptr(src), n, C.byref(cfg) if cfg else None,
                               _stream(stream)))

    def send(self, buf, n, dst, tag=0, cfg: Optional[mp_config] = None, stream=None):
        self._ck(lib().mp_send(self.h, _ptr(buf), n, dst, tag, C.byref(cfg) if cfg else None,
                               _stream(stream)))

    def recv(self, buf, n, src, tag=0, stream=None):
        self._ck(lib().mp_recv(self.h, _ptr(buf), n, src, tag, _stream(stream)))

    def alltoall(self, sendbuf, recvbuf, bytes_per_rank, algo=MP_ALGO_AUTO, stream=None):
        """mp_alltoall (collective, NEXT f3)."""
        self._ck(lib().mp_alltoall(self.h, _ptr(sendbuf), _ptr(recvbuf), bytes_per_rank, algo, _stream(stream)))

    def allreduce(self, sendbuf, recvbuf, count, dtype=MP_DT_F32, algo=MP_ALGO_AUTO, stream=None):
        """mp_allreduce(MP_OP_SUM) (collective, NEXT f3)."""
        self._ck(lib().mp_allreduce(self.h, _ptr(sendbuf), _ptr(recvbuf), count, dtype, MP_OP_SUM, algo,
                                    _stream(stream)))

    def sync(self):
        self._ck(lib().mp_sync(self.h))

    def calibrate(self, sizes: Optional[Sequence[int]] = None, reps=0):
        if sizes:
            arr = (C.c_uint64 * len(sizes))(*sizes)
            self._ck(lib().mp_calibrate(self.h, arr, len(sizes), reps))
        else:
            self._ck(lib().mp_calibrate(self.h, None, 0, reps))

    def calibrate_bands(self, edges: Optional[Sequence[int]] = None, reps=0):
        """mp_calibrate_bands (NEXT f4, readings C20/C21)."""
        if edges:
            arr = (C.c_uint64 * len(edges))(*edges)
            self._ck(lib().mp_calibrate_bands(self.h, arr, len(edges), reps))
        else:
            self._ck(lib().mp_calibrate_bands(self.h, None, 0, reps))

    def save_params(self, path):
        self._ck(lib().mp_save_params(self.h, path.encode()))

    def load_params(self, path):
        self._ck(lib().mp_load_params(self.h, path.encode()))

    def topology(self) -> dict:
        """mp_get_topology: the job's GPUs (UUID, PCI, NUMA, PCIe link, NVLinks) and the
        per-pair peer access / P2P attributes (Step 1)."""
        t = mp_topology()
        self._ck(lib().mp_get_topology(self.h, C.byref(t)))
        w = t.world
        gpus = [{"uuid": bytes(g.uuid).hex(), "device": g.device,
                 "pci": f"{g.pci_domain:04x}:{g.pci_bus:02x}:{g.pci_device:02x}.0", "numa_node": g.numa_node,
                 "pcie_gen": g.pcie_gen, "pcie_width": g.pcie_width, "pcie_gen_cur": g.pcie_gen_cur,
                 "nvlinks": g.nvlinks, "sms": g.sms} for g in list(t.gpu)[:w]]
        mat = lambda m: [[m[a][b] for b in range(w)] for a in range(w)]  # noqa: E731
        return {"world": w, "fingerprint": f"{t.fingerprint:016x}", "gpus": gpus,
                "peer_access": mat(t.peer_access), "p2p_perf_rank": mat(t.p2p_perf_rank),
                "p2p_atomics": mat(t.p2p_atomics)}

    def set_topology(self, topo: dict):
        """mp_set_topology (model-only contexts): inject a topology dict as returned by
        topology() (missing keys default to 0 / full peer access)."""
        t = mp_topology()
        w = int(topo["world"])
        t.world = w
        for r, g in enumerate(topo.get("gpus", [])[:w]):
            raw = bytes.fromhex(g.get("uuid", "00" * 16))[:16].ljust(16, b"\0")
            C.memmove(t.gpu[r].uuid, raw, 16)
            for k in ("device", "numa_node", "pcie_gen", "pcie_width", "pcie_gen_cur", "nvlinks", "sms"):
                setattr(t.gpu[r], k, int(g.get(k, 0)))
        for key in ("peer_access", "p2p_perf_rank", "p2p_atomics"):
            m = topo.get(key)
            for a in range(w):
                for b in range(w):
                    getattr(t, key)[a][b] = int(m[a][b]) if m else (1 if key == "peer_access" else 0)
        self._ck(lib().mp_set_topology(self.h, C.byref(t)))

    def launches(self) -> int:
        v = C.c_uint64()
        self._ck(lib().mp_stats(self.h, C.byref(v)))
        return v.value


class _CudaArray:
    """Minimal __cuda_array_interface__ holder (zero-copy view of device memory)."""

    def __init__(self, ptr: int, n: int):
        self.__cuda_array_interface__ = {"shape": (n,), "typestr": "|u1", "data": (ptr, False),
                                         "version": 3, "strides": None}


def as_tensor(ptr: int, n: int):
    """A torch uint8 tensor viewing n bytes of device memory at ptr (e.g. from mp_alloc)."""
    import torch
    return torch.as_tensor(_CudaArray(ptr, n), device="cuda")


class EmulatedWorld:
    """mp_init_emulated / mp_emu_run / mp_finalize_emulated: every rank of a world as a
    Context of this process on one GPU.  ``ctx[r].send`` / ``ctx[r].recv`` record;
    ``run()`` launches everything recorded as ONE cooperative grid and waits for it."""

    def __init__(self, world, device=0, host_path=-1, slots=0, relay_ctas=0, heap_bytes=0,
                 slot_bytes=0, timeout_s=0.0, param_file=None):
        L = lib()
        a = mp_init_args()
        a.rank, a.world, a.device, a.flags = 0, world, device, MP_INIT_NO_CALIBRATE
        a.n_loop_relays, a.host_path, a.slots, a.relay_ctas = -1, host_path, slots, relay_ctas
        a.heap_bytes, a.slot_bytes, a.timeout_s = heap_bytes, slot_bytes, timeout_s
        a.allgather = ALLGATHER()
        a.param_file = param_file.encode() if param_file else None
        self._h = (C.c_void_p * world)()
        st = L.mp_init_emulated(self._h, C.byref(a))
        if st != 0:
            raise MPError(st, "mp_init_emulated failed")
        self.world = world
        self.ctx = [Context._wrap(self._h[r], r, world) for r in range(world)]

    def run(self, stream=None) -> float:
        """Launch what the contexts recorded as one cooperative grid; returns the grid's
        device time [s] (CUDA events on `stream`)."""
        t = C.c_double()
        st = lib().mp_emu_run(self._h, self.world, _stream(stream), C.byref(t))
        if st != 0:
            raise MPError(st, lib().mp_last_error(self._h[0]).decode())
        return t.value

    def _bufs(self, xs):
        assert len(xs) == self.world
        return (C.c_void_p * self.world)(*[_ptr(x) for x in xs])

    def register(self, tensors):
        """mp_emu_register: tensors[r] (or None) becomes a receive region of rank r;
        returns the region ids."""
        ptrs = (C.c_void_p * self.world)(*[_ptr(t) if t is not None else None for t in tensors])
        sizes = (C.c_uint64 * self.world)(*[t.numel() * t.element_size() if t is not None else 0 for t in tensors])
        ids = (C.c_int * self.world)()
        st = lib().mp_emu_register(self._h, self.world, ptrs, sizes, ids)
        if st != 0:
            raise MPError(st, lib().mp_last_error(self._h[0]).decode())
        return list(ids)

    def deregister(self, ids):
        st = lib().mp_emu_deregister(self._h, self.world, (C.c_int * self.world)(*ids))
        if st != 0:
            raise MPError(st, lib().mp_last_error(self._h[0]).decode())

    def alltoall(self, sendbufs, recvbufs, bytes_per_rank, algo=MP_ALGO_AUTO, stream=None):
        """mp_emu_alltoall: every rank's MPI_Alltoall, one cooperative grid per step."""
        st = lib().mp_emu_alltoall(self._h, self.world, self._bufs(sendbufs), self._bufs(recvbufs), bytes_per_rank,
                                   algo, _stream(stream))
        if st != 0:
            raise MPError(st, lib().mp_last_error(self._h[0]).decode())

    def allreduce(self, sendbufs, recvbufs, count, dtype=MP_DT_F32, algo=MP_ALGO_AUTO, stream=None):
        """mp_emu_allreduce(MP_OP_SUM): every rank's MPI_Allreduce, one grid per step."""
        st = lib().mp_emu_allreduce(self._h, self.world, self._bufs(sendbufs), self._bufs(recvbufs), count, dtype,
                                    MP_OP_SUM, algo, _stream(stream))
        if st != 0:
            raise MPError(st, lib().mp_last_error(self._h[0]).decode())

    def close(self):
        if self.ctx:
            lib().mp_finalize_emulated(self._h, self.world)
            self.ctx = []

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()
