"""sdag -- B200-native FP64 stencil-DAG library (Python binding).

Thin marshalling layer over the C ABI in include/sdag.h (libsdag.so): every
step of the hot path -- parse (a1), analyse (a2), plan (a3), the sm_100a
sweep kernels (a4-a6) and the z-slab halo exchange (a7) -- runs in the native
library.  PyTorch is used only to own device memory and streams.

    import paper_conf_ipps_rawatvsrps19_b200 as sdag
    plan = sdag.Plan(sdag.spec_text("lap25"), (512, 512, 512))
    plan.apply([out, inp], scalars=[c0, c1, c2, c3, c4])   # formal order (B, A, c0..c4)

Reference: Rawat et al., "On Optimizing Complex Stencils on GPUs", IPDPS 2019
(PAPER.md): Listing 1 DSL, streaming, Table I
benchmarks.
"""
from __future__ import annotations

import ctypes
import os

from . import _capi
from ._capi import PlanInfo, PlanOpts, SDAG_DEVICE_CURRENT, SDAG_DEVICE_NONE

__all__ = ["Plan", "Program", "Dist", "SdagError", "registry", "spec_text", "fusion_schedule", "slab_partition", "slab_halo", "slab_partition2", "slab_halo2", "fission", "fuse_program", "program_version", "program_forest",
           "program_forest_tune", "nccl_unique_id",
           "nccl_comm_create", "nccl_comm_destroy", "nccl_sendrecv", "launch_count", "fp64_peak", "version", "SPEC_DIR"]

SPEC_DIR = os.path.join(os.path.dirname(os.path.abspath(__file__)), "specs")


class SdagError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"sdag {_capi.STATUS.get(status, status)}: {msg}")
        self.status = status
        self.code = _capi.STATUS.get(status, str(status))


def _check(st: int):
    if st != 0:
        raise SdagError(st, (_capi.lib().sdag_last_error() or b"").decode())


def _stream_handle(stream):
    if stream is None:
        import torch
        return ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)
    if isinstance(stream, int):
        return ctypes.c_void_p(stream)
    return ctypes.c_void_p(stream.cuda_stream)


def _ptr(t, what):
    """device pointer of a contiguous float64 CUDA tensor (no copies)"""
    import torch
    if not isinstance(t, torch.Tensor):
        raise TypeError(f"{what}: expected a torch.Tensor")
    if t.dtype != torch.float64 or not t.is_cuda or not t.is_contiguous():
        raise TypeError(f"{what}: need a contiguous float64 CUDA tensor (got {t.dtype}, {t.device})")
    return t.data_ptr()


def _check_sizes(arrays3d, arrays1d, dims, axes, batch=1, device=None, host=False):
    """The C ABI takes raw pointers, so an undersized buffer would be read or
    written out of bounds on the device (TMA / stores) or on the host
    (cudaMemcpy): check every 3D array holds batch*nz*ny*nx elements, every 1D
    array batch x the extent of its axis, and (device arrays) the plan's device."""
    n = int(batch) * int(dims[0]) * int(dims[1]) * int(dims[2])
    for q, t in enumerate(arrays3d):
        cnt = int(t.size) if host else int(t.numel())
        if cnt != n:
            raise ValueError(f"grid array #{q} has {cnt} elements; the plan needs {n} "
                             f"({'%d x ' % batch if batch > 1 else ''}{tuple(int(x) for x in dims)})")
        if device is not None and not host and t.device.index != device:
            raise ValueError(f"grid array #{q} is on {t.device}; the plan is on cuda:{device}")
    if axes is not None:
        for q, (t, ax) in enumerate(zip(arrays1d, axes)):
            if ax < 0:  # never read by the stencil
                continue
            cnt = int(t.size) if host else int(t.numel())
            need = int(batch) * int(dims[ax])  # batched: [batch][len] (include/sdag.h)
            if cnt != need:
                raise ValueError(f"1D array #{q} has {cnt} elements; its axis ({'zyx'[ax]}) needs {need}"
                                 + (f" ({batch} x {int(dims[ax])})" if batch > 1 else ""))
            if device is not None and not host and t.device.index != device:
                raise ValueError(f"1D array #{q} is on {t.device}; the plan is on cuda:{device}")


def _arr(ptrs):
    return (ctypes.c_void_p * max(1, len(ptrs)))(*ptrs)


def _scal(s):
    s = [float(x) for x in (s or [])]
    return (ctypes.c_double * max(1, len(s)))(*s), len(s)


def _opts(order=-1, device=None, tune=False, batch=1, variant=None, fusion=True, time_tile=1):
    o = PlanOpts()
    _capi.lib().sdag_plan_opts_init(ctypes.byref(o))
    o.order = int(order)
    if device == "none":
        o.device = SDAG_DEVICE_NONE
    elif device is None:
        # libsdag links its own (static) CUDA runtime, whose "current device" is
        # independent of torch's: bind to the device torch is using.
        o.device = SDAG_DEVICE_CURRENT
        import sys
        torch = sys.modules.get("torch")
        if torch is not None and torch.cuda.is_available():
            o.device = int(torch.cuda.current_device())
    else:
        o.device = int(device)
    o.tune = 1 if tune else 0
    o.batch = int(batch)
    o.force_variant = variant.encode() if variant else None
    o.fusion = 1 if fusion else 0
    o.time_tile = int(time_tile)
    return o


def registry() -> dict:
    """Registered DAGs with hand-written sm_100a bodies: name -> canonical spec text."""
    L = _capi.lib()
    out = {}
    for i in range(L.sdag_registry_count()):
        n, t = ctypes.c_char_p(), ctypes.c_char_p()
        _check(L.sdag_registry_get(i, ctypes.byref(n), ctypes.byref(t)))
        out[n.value.decode()] = t.value.decode()
    return out


def spec_text(name: str) -> str:
    with open(os.path.join(SPEC_DIR, name + ".sdag")) as f:
        return f.read()


class Plan:
    """A planned stencil DAG (a1-a3) bound to grid dims (nz, ny, nx)."""

    def __init__(self, spec: str, dims, order=-1, device=None, tune=False, batch=1, variant=None, fusion=True):
        self._L = _capi.lib()
        self._h = ctypes.c_void_p()
        d = (ctypes.c_int64 * 3)(*[int(x) for x in dims])
        o = _opts(order, device, tune, batch, variant, fusion)
        _check(self._L.sdag_plan_create(spec.encode(), d, ctypes.byref(o), ctypes.byref(self._h)))
        self._owned = True
        self._device = int(o.device) if o.device >= 0 else None

    @classmethod
    def _borrow(cls, handle):
        p = cls.__new__(cls)
        p._L = _capi.lib()
        p._h = ctypes.c_void_p(handle)
        p._owned = False
        p._device = None
        return p

    def _meta(self):
        """(dims, axis of each 1D formal), cached: plans are immutable"""
        m = getattr(self, "_meta_cache", None)
        if m is None:
            dims = self.info["dims"]
            axes = [a[3] for a in self.args() if a[0] == 1]
            m = self._meta_cache = (dims, axes)
        return m

    def _sizes(self, arrays3d, arrays1d, batch=1, host=False):
        dims, axes = self._meta()
        _check_sizes(arrays3d, arrays1d, dims, axes, batch, getattr(self, "_device", None), host)

    def close(self):
        if getattr(self, "_owned", False) and self._h:
            self._L.sdag_plan_destroy(self._h)
        self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    # ---- introspection ----
    @property
    def info(self) -> dict:
        i = PlanInfo()
        _check(self._L.sdag_plan_info_get(self._h, ctypes.byref(i)))
        d = {f: getattr(i, f) for f, _ in PlanInfo._fields_}
        for k in ("radius", "dims", "lo", "hi"):
            d[k] = tuple(d[k])
        d["dag"] = i.dag.decode()
        d["variant"] = i.variant.decode()
        return d

    def args(self):
        """[(kind, index, name, role_or_axis)] in formal order per kind."""
        i = self.info
        out = []
        for kind, n in ((0, i["n_arrays3d"]), (1, i["n_arrays1d"]), (2, i["n_scalars"])):
            for q in range(n):
                nm, r = ctypes.c_char_p(), ctypes.c_int32()
                _check(self._L.sdag_plan_arg(self._h, kind, q, ctypes.byref(nm), ctypes.byref(r)))
                out.append((kind, q, nm.value.decode(), r.value))
        return out

    def arg_names(self, kind: int):
        return [a[2] for a in self.args() if a[0] == kind]

    def variants(self):
        out = []
        for q in range(self.info["n_variants"]):
            nm = ctypes.c_char_p()
            _check(self._L.sdag_plan_variant_name(self._h, q, ctypes.byref(nm)))
            out.append(nm.value.decode())
        return out

    def kernel_name(self, sweeps: int = 1) -> str:
        """symbol of the kernel a launch of `sweeps` fused sweeps runs (as ncu names it)"""
        nm = ctypes.c_char_p()
        _check(self._L.sdag_plan_kernel_name(self._h, int(sweeps), ctypes.byref(nm)))
        return nm.value.decode()

    def describe(self) -> str:
        return self._L.sdag_plan_describe(self._h).decode()

    # ---- apply ----
    def profile(self, arrays3d, arrays1d=(), scalars=(), peak_hbm_gbs=0.0, peak_fp64_tflops=0.0, stream=None):
        """Profile-guided classification (paper Section IV): the plan's kernel timed on
        these arrays, its DRAM / FP64 roofline fractions, code-differenced twins,
        resources, the bound (dram | compute | latency) and the Section IV-A hints.
        Overwrites the outputs; synchronous."""
        p3 = [_ptr(t, "grid array") for t in arrays3d]
        p1 = [_ptr(t, "1D array") for t in arrays1d]
        s, ns = _scal(scalars)
        pr = _capi.Profile()
        _check(self._L.sdag_plan_profile(self._h, _arr(p3), len(p3), _arr(p1), len(p1), s, ns, float(peak_hbm_gbs),
                                         float(peak_fp64_tflops), _stream_handle(stream), ctypes.byref(pr)))
        d = {k: getattr(pr, k) for k, _ in _capi.Profile._fields_}
        d["variant"] = pr.variant.decode()
        d["hints"] = [h for h in pr.hints.decode().split("\n") if h]
        d["bound"] = {0: "dram", 1: "compute", 2: "latency"}[pr.bound]
        return d

    def apply(self, arrays3d, arrays1d=(), scalars=(), stream=None):
        p3 = [_ptr(t, "grid array") for t in arrays3d]
        self._sizes(arrays3d, arrays1d)
        p1 = [_ptr(t, "1D array") for t in arrays1d]
        s, ns = _scal(scalars)
        _check(self._L.sdag_apply(self._h, _arr(p3), len(p3), _arr(p1), len(p1), s, ns, _stream_handle(stream)))

    def apply_batched(self, batch, arrays3d, arrays1d=(), scalars=(), stream=None):
        p3 = [_ptr(t, "grid array") for t in arrays3d]
        self._sizes(arrays3d, arrays1d, batch=batch)
        p1 = [_ptr(t, "1D array") for t in arrays1d]
        s, ns = _scal(scalars)
        _check(self._L.sdag_apply_batched(self._h, int(batch), _arr(p3), len(p3), _arr(p1), len(p1), s, ns,
                                          _stream_handle(stream)))

    def apply_iterated(self, buf0, buf1, T, scalars=(), stream=None):
        s, ns = _scal(scalars)
        _ptr(buf0, "buf0"), _ptr(buf1, "buf1")
        self._sizes([buf0, buf1], ())
        _check(self._L.sdag_apply_iterated(self._h, _ptr(buf0, "buf0"), _ptr(buf1, "buf1"), int(T), s, ns,
                                           _stream_handle(stream)))

    def apply_host(self, host3d, host1d=(), scalars=(), stream=None):
        """End-to-end call with host numpy buffers (outputs/inouts updated in place).
        Returns (h2d_bytes, d2h_bytes)."""
        import numpy as np
        for a in list(host3d) + list(host1d):
            if not (isinstance(a, np.ndarray) and a.dtype == np.float64 and a.flags.c_contiguous):
                raise TypeError("apply_host needs contiguous float64 numpy arrays")
        self._sizes(host3d, host1d, host=True)
        p3 = [a.ctypes.data for a in host3d]
        p1 = [a.ctypes.data for a in host1d]
        s, ns = _scal(scalars)
        up, down = ctypes.c_int64(), ctypes.c_int64()
        _check(self._L.sdag_apply_host(self._h, _arr(p3), len(p3), _arr(p1), len(p1), s, ns, _stream_handle(stream),
                                       ctypes.byref(up), ctypes.byref(down)))
        return up.value, down.value


class Program:
    """A multi-stencil program (several stencils and calls, Fig 3c): one planned
    stage per call, applied in call order.  Arguments are the declared arrays
    and scalars in declaration order (sdag_program_*)."""

    def __init__(self, spec: str, dims, order=-1, device=None, tune=False, batch=1, variant=None):
        self._L = _capi.lib()
        self._h = ctypes.c_void_p()
        d = (ctypes.c_int64 * 3)(*[int(x) for x in dims])
        o = _opts(order, device, tune, batch, variant, True)
        _check(self._L.sdag_program_create(spec.encode(), d, ctypes.byref(o), ctypes.byref(self._h)))
        self._dims = tuple(int(x) for x in dims)
        self._device = int(o.device) if o.device >= 0 else None

    def close(self):
        if self._h:
            self._L.sdag_program_destroy(self._h)
        self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    @property
    def counts(self) -> dict:
        n, a3, a1, sc = ctypes.c_int32(), ctypes.c_int32(), ctypes.c_int32(), ctypes.c_int32()
        _check(self._L.sdag_program_info(self._h, ctypes.byref(n), ctypes.byref(a3), ctypes.byref(a1),
                                         ctypes.byref(sc)))
        return {"n_stages": n.value, "n_arrays3d": a3.value, "n_arrays1d": a1.value, "n_scalars": sc.value}

    def args(self):
        """[(kind, index, name, role_or_axis)] in declaration order per kind."""
        c = self.counts
        out = []
        for kind, n in ((0, c["n_arrays3d"]), (1, c["n_arrays1d"]), (2, c["n_scalars"])):
            for q in range(n):
                nm, r = ctypes.c_char_p(), ctypes.c_int32()
                _check(self._L.sdag_program_arg(self._h, kind, q, ctypes.byref(nm), ctypes.byref(r)))
                out.append((kind, q, nm.value.decode(), r.value))
        return out

    def arg_names(self, kind: int):
        return [a[2] for a in self.args() if a[0] == kind]

    def stage(self, s: int) -> Plan:
        """Borrowed plan of stage s (introspection only; owned by the program)."""
        h = ctypes.c_void_p()
        _check(self._L.sdag_program_stage(self._h, int(s), ctypes.byref(h)))
        p = Plan._borrow(h.value)
        p._program = self  # keep the owner alive
        return p

    def apply(self, arrays3d, arrays1d=(), scalars=(), stream=None, batch=1):
        p3 = [_ptr(t, "grid array") for t in arrays3d]
        p1 = [_ptr(t, "1D array") for t in arrays1d]
        axes = [a[3] for a in self.args() if a[0] == 1]
        _check_sizes(arrays3d, arrays1d, self._dims, axes, batch, self._device)
        s, ns = _scal(scalars)
        _check(self._L.sdag_program_apply(self._h, int(batch), _arr(p3), len(p3), _arr(p1), len(p1), s, ns,
                                          _stream_handle(stream)))


def fusion_schedule(f, T: int):
    """Temporal-fusion schedule (sdag_fusion_schedule): f = {x: cost of an
    x-sweep launch}; returns (sweeps per launch, total cost)."""
    maxdeg = max(f)
    arr = (ctypes.c_double * 8)(*[float(f.get(x, 0.0)) for x in range(8)])
    cap = max(1, int(T))
    seq = (ctypes.c_int32 * cap)()
    n, cost = ctypes.c_int32(), ctypes.c_double()
    _check(_capi.lib().sdag_fusion_schedule(arr, int(maxdeg), int(T), seq, cap, ctypes.byref(n), ctypes.byref(cost)))
    return list(seq[:n.value]), cost.value


def slab_partition(global_nz: int, rz: int, nranks: int, rank: int) -> dict:
    out = (ctypes.c_int64 * 7)()
    _check(_capi.lib().sdag_slab_partition(int(global_nz), int(rz), int(nranks), int(rank), out))
    keys = ("z0", "nz_own", "nz_alloc", "k_lo", "k_hi", "has_lower", "has_upper")
    return dict(zip(keys, list(out)))


def slab_partition2(global_nz: int, rz: int, time_tile: int, nranks: int, rank: int) -> dict:
    """slab_partition with ghost depth H = rz * time_tile (key "halo")."""
    out = (ctypes.c_int64 * 8)()
    _check(_capi.lib().sdag_slab_partition2(int(global_nz), int(rz), int(time_tile), int(nranks), int(rank), out))
    keys = ("z0", "nz_own", "nz_alloc", "k_lo", "k_hi", "has_lower", "has_upper", "halo")
    return dict(zip(keys, list(out)))


def slab_halo2(global_nz: int, rz: int, time_tile: int, nranks: int, rank: int, planes: int) -> dict:
    out = (ctypes.c_int64 * 5)()
    _check(_capi.lib().sdag_slab_halo2(int(global_nz), int(rz), int(time_tile), int(nranks), int(rank), int(planes),
                                        out))
    return dict(zip(("lo_send", "lo_recv", "up_send", "up_recv", "planes"), list(out)))


def slab_halo(global_nz: int, rz: int, nranks: int, rank: int) -> dict:
    out = (ctypes.c_int64 * 5)()
    _check(_capi.lib().sdag_slab_halo(int(global_nz), int(rz), int(nranks), int(rank), out))
    return dict(zip(("lo_send", "lo_recv", "up_send", "up_recv", "planes"), list(out)))


def nccl_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    _check(_capi.lib().sdag_nccl_get_unique_id(buf))
    return buf.raw


def nccl_comm_create(uid: bytes, nranks: int, rank: int, device: int) -> int:
    c = ctypes.c_void_p()
    _check(_capi.lib().sdag_nccl_comm_create(uid, int(nranks), int(rank), int(device), ctypes.byref(c)))
    return c.value


def nccl_comm_destroy(comm: int):
    _capi.lib().sdag_nccl_comm_destroy(ctypes.c_void_p(comm))


def nccl_sendrecv(comm: int, peer: int, send, recv, stream=None):
    """One grouped ncclSend(send -> peer) + ncclRecv(recv <- peer) through the halo
    exchange's code path (sdag_nccl_sendrecv); peer may be this rank."""
    if not send.is_contiguous() or not recv.is_contiguous():
        raise TypeError("send and recv must be contiguous")
    if send.numel() != recv.numel():
        raise ValueError("send and recv must have the same number of elements")
    _check(_capi.lib().sdag_nccl_sendrecv(ctypes.c_void_p(comm), int(peer), ctypes.c_void_p(_ptr(send, "send")),
                                          ctypes.c_void_p(_ptr(recv, "recv")), int(send.numel()),
                                          _stream_handle(stream)))


class Dist:
    """This rank's z-slab of a global stencil problem (a7)."""

    def __init__(self, spec, global_dims, rank, nranks, comm=None, order=-1, device=None, tune=False, variant=None,
                 fusion=True, time_tile=1):
        self._L = _capi.lib()
        self._h = ctypes.c_void_p()
        d = (ctypes.c_int64 * 3)(*[int(x) for x in global_dims])
        o = _opts(order, device, tune, 1, variant, fusion, time_tile)
        _check(self._L.sdag_dist_create(spec.encode(), d, ctypes.byref(o), int(rank), int(nranks),
                                        ctypes.c_void_p(comm or 0), ctypes.byref(self._h)))
        self.rank, self.nranks = rank, nranks
        self._device = int(o.device) if o.device >= 0 else None

    def _sizes(self, arrays3d, arrays1d, host=False):
        """local layout (ghost planes included); 1D arrays sized to it too"""
        dims = self.layout()[0]
        axes = [a[3] for a in self.plan.args() if a[0] == 1]
        _check_sizes(arrays3d, arrays1d, dims, axes, 1, self._device, host)

    @classmethod
    def from_local_plan(cls, plan: "Plan", rank, nranks, comm=None, time_tile=1):
        """SURVEY 8(b)'s form: a dist from a plan of this rank's owned slab
        (nz_own, ny, nx); global nz = nz_own * nranks (sdag_dist_create_local)"""
        d = cls.__new__(cls)
        d._L = _capi.lib()
        d._h = ctypes.c_void_p()
        _check(d._L.sdag_dist_create_local(plan._h, int(rank), int(nranks), ctypes.c_void_p(comm or 0),
                                           int(time_tile), ctypes.byref(d._h)))
        d.rank, d.nranks = rank, nranks
        d._device = getattr(plan, "_device", None)
        return d

    def close(self):
        if self._h:
            self._L.sdag_dist_destroy(self._h)
        self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def layout(self):
        """(local_dims (nz_alloc, ny, nx), global z of local plane 0)"""
        ld = (ctypes.c_int64 * 3)()
        g = ctypes.c_int64()
        _check(self._L.sdag_dist_layout(self._h, ld, ctypes.byref(g)))
        return tuple(ld), g.value

    @property
    def plan(self) -> Plan:
        """Borrowed local plan (owned by this dist, which it keeps alive)."""
        p = Plan._borrow(self._L.sdag_dist_local_plan(self._h))
        p._dist = self
        p._device = self._device
        return p

    def apply(self, arrays3d, arrays1d=(), scalars=(), stream=None, comm_stream=None):
        p3 = [_ptr(t, "grid array") for t in arrays3d]
        self._sizes(arrays3d, arrays1d)
        p1 = [_ptr(t, "1D array") for t in arrays1d]
        s, ns = _scal(scalars)
        cs = ctypes.c_void_p(0) if comm_stream is None else _stream_handle(comm_stream)
        _check(self._L.sdag_dist_apply(self._h, _arr(p3), len(p3), _arr(p1), len(p1), s, ns, _stream_handle(stream),
                                       cs))

    def apply_iterated(self, buf0, buf1, T, scalars=(), stream=None, comm_stream=None):
        s, ns = _scal(scalars)
        _ptr(buf0, "buf0"), _ptr(buf1, "buf1")
        self._sizes([buf0, buf1], ())
        cs = ctypes.c_void_p(0) if comm_stream is None else _stream_handle(comm_stream)
        _check(self._L.sdag_dist_apply_iterated(self._h, _ptr(buf0, "buf0"), _ptr(buf1, "buf1"), int(T), s, ns,
                                                _stream_handle(stream), cs))

    @staticmethod
    def apply_iterated_loopback(dists, bufs0, bufs1, T, scalars=(), stream=None):
        if not (len(dists) == len(bufs0) == len(bufs1)):
            raise ValueError("one buf0 and one buf1 per dist")
        for d, x, y in zip(dists, bufs0, bufs1):
            _ptr(x, "buf0"), _ptr(y, "buf1")
            d._sizes([x, y], ())
        hs = (ctypes.c_void_p * len(dists))(*[d._h.value for d in dists])
        b0 = _arr([_ptr(t, "buf0") for t in bufs0])
        b1 = _arr([_ptr(t, "buf1") for t in bufs1])
        s, ns = _scal(scalars)
        _check(_capi.lib().sdag_dist_apply_iterated_loopback(hs, len(dists), b0, b1, int(T), s, ns,
                                                            _stream_handle(stream)))


    def apply_host(self, host3d, host1d=(), scalars=(), stream=None):
        """One sweep of this slab end to end with host numpy buffers of the local
        layout (ghost planes included): (h2d_bytes, d2h_bytes)"""
        import numpy as np
        for a in list(host3d) + list(host1d):
            if not (isinstance(a, np.ndarray) and a.dtype == np.float64 and a.flags.c_contiguous):
                raise TypeError("apply_host needs contiguous float64 numpy arrays")
        self._sizes(host3d, host1d, host=True)
        p3 = [a.ctypes.data for a in host3d]
        p1 = [a.ctypes.data for a in host1d]
        s, ns = _scal(scalars)
        up, down = ctypes.c_int64(), ctypes.c_int64()
        _check(self._L.sdag_dist_apply_host(self._h, _arr(p3), len(p3), _arr(p1), len(p1), s, ns,
                                            _stream_handle(stream), ctypes.byref(up), ctypes.byref(down)))
        return up.value, down.value

    # ---- peer-memory halo path (NVLink P2P stores from the sweep kernels) ----
    def p2p_alloc(self):
        """(buf0, buf1): the library-owned slab buffers of sdag_dist_p2p_alloc as
        float64 CUDA tensors of the local layout (zero-copy views that keep this
        dist -- the owner of the memory -- alive).  Fill buf0's owned planes; the
        first p2p_apply_iterated initialises buf1 and the ghost planes."""
        import torch
        b0, b1 = ctypes.c_void_p(), ctypes.c_void_p()
        _check(self._L.sdag_dist_p2p_alloc(self._h, ctypes.byref(b0), ctypes.byref(b1)))
        shape = tuple(int(x) for x in self.layout()[0])
        dev = torch.device("cuda", self._device if self._device is not None else torch.cuda.current_device())
        return tuple(torch.as_tensor(_DeviceView(b.value, shape, owner=self), device=dev) for b in (b0, b1))

    def p2p_handle(self) -> bytes:
        h = ctypes.create_string_buffer(64)
        _check(self._L.sdag_dist_p2p_handle(self._h, h))
        return h.raw

    def p2p_attach(self, side, handle):
        """side 0 = rank-1, 1 = rank+1; `handle` from that rank's p2p_handle()
        (another process), or a Dist of this process"""
        if isinstance(handle, Dist):
            _check(self._L.sdag_dist_p2p_attach_local(self._h, int(side), handle._h))
        else:
            if len(handle) != 64:
                raise ValueError("an IPC handle is 64 bytes")
            _check(self._L.sdag_dist_p2p_attach(self._h, int(side), bytes(handle)))

    def p2p_apply_iterated(self, T, scalars=(), stream=None):
        """T sweeps over the p2p buffers; result in buf[T & 1]"""
        s, ns = _scal(scalars)
        _check(self._L.sdag_dist_p2p_apply_iterated(self._h, int(T), s, ns, _stream_handle(stream)))


class _DeviceView:
    """__cuda_array_interface__ of a float64 C-order device buffer (zero copy)"""

    def __init__(self, ptr, shape, owner=None):
        self._owner = owner  # torch.as_tensor keeps this object (and so the owner) alive
        self.__cuda_array_interface__ = {"shape": shape, "typestr": "<f8", "data": (int(ptr), False),
                                         "version": 3, "strides": None}


def fission(spec: str, kind: str = "trivial") -> str:
    """The paper's fission versions (Section VI-B) of a single-stage spec as DSL
    text for Program: kind "trivial" (one stencil per output, Fig 3c) or
    "maxfuse" (the stencil re-printed)"""
    k = {"maxfuse": 0, "trivial": 1}[kind]
    L = _capi.lib()
    n = ctypes.c_int64()
    _check(L.sdag_spec_fission(spec.encode(), k, None, 0, ctypes.byref(n)))
    buf = ctypes.create_string_buffer(n.value + 1)
    _check(L.sdag_spec_fission(spec.encode(), k, buf, n.value + 1, ctypes.byref(n)))
    return buf.value.decode()


def fuse_program(program: str, keep_intermediates: bool = True) -> str:
    """maxfuse of a multi-stencil program with recomputation (sdag_program_fuse):
    one stencil; intermediates inlined at their read offsets"""
    L = _capi.lib()
    n = ctypes.c_int64()
    _check(L.sdag_program_fuse(program.encode(), int(keep_intermediates), None, 0, ctypes.byref(n)))
    buf = ctypes.create_string_buffer(n.value + 1)
    _check(L.sdag_program_fuse(program.encode(), int(keep_intermediates), buf, n.value + 1, ctypes.byref(n)))
    return buf.value.decode()


_VERSION = {"maxfuse": 0, "staged": 1, "recompute": 2, "groups": 3}


def program_version(program: str, kind: str = "recompute", groups=None):
    """Section VI-B versions of a multi-stencil program (sdag_program_version):
    kind "maxfuse", "staged", "recompute" (recompute-fission: groups grown while
    the recomputation halo <= max(4, r)) or "groups" (fuse the calls in groups
    of the given sizes).  Returns (DSL text, group sizes)."""
    L = _capi.lib()
    k = _VERSION[kind]
    if kind == "groups":
        sizes = (ctypes.c_int32 * len(groups))(*[int(x) for x in groups])
        ns = len(groups)
    else:
        sizes = (ctypes.c_int32 * 16)()
        ns = 16
    n = ctypes.c_int64()
    _check(L.sdag_program_version(program.encode(), k, sizes, ns, None, 0, ctypes.byref(n)))
    buf = ctypes.create_string_buffer(n.value + 1)
    _check(L.sdag_program_version(program.encode(), k, sizes, ns, buf, n.value + 1, ctypes.byref(n)))
    g = list(groups) if kind == "groups" else [x for x in sizes if x] if kind == "recompute" else None
    return buf.value.decode(), g


def program_forest(program: str, max_candidates: int = 64):
    """The fusion forest's candidates (sdag_program_forest): list of group-size lists"""
    L = _capi.lib()
    ng = (ctypes.c_int32 * max_candidates)()
    sz = (ctypes.c_int32 * (16 * max_candidates))()
    n = ctypes.c_int32()
    _check(L.sdag_program_forest(program.encode(), int(max_candidates), ng, sz, ctypes.byref(n)))
    return [[sz[c * 16 + g] for g in range(ng[c])] for c in range(n.value)]


def program_forest_tune(program: str, dims, arrays3d, arrays1d=(), scalars=(), stream=None, max_candidates=64,
                        device=None, tune=False):
    """Time every forest candidate on these arrays (program argument order;
    outputs overwritten): (candidates, ms per candidate, index of the fastest)"""
    L = _capi.lib()
    d = (ctypes.c_int64 * 3)(*[int(x) for x in dims])
    o = _opts(-1, device, tune, 1, None, True)
    p3 = [_ptr(t, "grid array") for t in arrays3d]
    p1 = [_ptr(t, "1D array") for t in arrays1d]
    s, ns = _scal(scalars)
    ms = (ctypes.c_double * max_candidates)()
    n, best = ctypes.c_int32(), ctypes.c_int32()
    _check(L.sdag_program_forest_tune(program.encode(), d, ctypes.byref(o), _arr(p3), len(p3), _arr(p1), len(p1), s,
                                      ns, _stream_handle(stream), int(max_candidates), ms, ctypes.byref(n),
                                      ctypes.byref(best)))
    return program_forest(program, max_candidates), list(ms[:n.value]), best.value


def launch_count() -> int:
    return int(_capi.lib().sdag_launch_count())


def fp64_peak(stream=None) -> float:
    f = ctypes.c_double()
    _check(_capi.lib().sdag_measure_fp64_peak(ctypes.byref(f), _stream_handle(stream)))
    return f.value


def version() -> str:
    return _capi.lib().sdag_version().decode()
