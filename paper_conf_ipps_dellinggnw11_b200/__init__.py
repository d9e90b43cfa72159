"""Thin Python binding of libphast.so (include/phast.h) -- argument marshalling only.

Every step of a PHAST query (upward CH search, seeding, the level-ordered downward
sweep, the diameter max) runs in the library's sm_100a kernels; this module only
converts arrays and torch tensors to pointers and checks that output tensors have
the shape, dtype and device the C ABI will write.  There is no CPU path: if the
library is missing, importing this package raises.  PyTorch provides device memory
and streams (plumbing only).

Names follow include/phast.h; see DESIGN.md for the paper passages.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libphast.so")

INF = 0xFFFFFFFF
KMAX = 64
SLOTS = 8
FLAG_HOST_ONLY = 1
FLAG_LEVEL_LAYOUT = 2
FLAG_BFS_IN_LEVEL = 4
FLAG_NO_BANDS = 32
LAYOUT_FLAGS = {"levels-bands": 0, "levels-bfs": FLAG_NO_BANDS, "levels": FLAG_LEVEL_LAYOUT}
LAYOUT_NAMES = {1: "levels", 2: "levels-bfs", 3: "levels-bands"}   # phast_info_t.layout
Q_NO_FUSED, Q_NO_TOP, Q_HYBRID_ON, Q_HYBRID_OFF, Q_NO_MULTI, Q_NO_BANDS = 1, 2, 4, 8, 32, 64

STATUS = {0: "OK", -1: "EINVAL", -2: "ENOMEM", -3: "ECUDA", -4: "ERANGE", -5: "ESTATE", -6: "EIO",
          -7: "EINTERNAL"}


class PhastError(RuntimeError):
    def __init__(self, fn, status):
        self.status = status
        super().__init__(f"{fn}: {STATUS.get(status, status)} ({_lib.phast_strerror(status).decode()})")


class _Opts(ctypes.Structure):
    _fields_ = [("hop_limit_lo", ctypes.c_uint32), ("hop_limit_hi", ctypes.c_uint32),
                ("settled_cap", ctypes.c_uint32), ("threads", ctypes.c_uint32),
                ("flags", ctypes.c_uint32), ("delta", ctypes.c_uint32), ("seed", ctypes.c_uint64)]


class _QOpts(ctypes.Structure):
    _fields_ = [("flags", ctypes.c_uint32), ("top_max_vertices", ctypes.c_uint32),
                ("seed_cap", ctypes.c_uint32), ("up_smem_cap", ctypes.c_uint32),
                ("band_unit", ctypes.c_uint32), ("band_threads", ctypes.c_uint32),
                ("band_variant", ctypes.c_uint32)]


class _Info(ctypes.Structure):
    _fields_ = [("n", ctypes.c_uint32), ("levels", ctypes.c_uint32), ("m", ctypes.c_uint64),
                ("m_up", ctypes.c_uint64), ("m_down", ctypes.c_uint64), ("n_tail", ctypes.c_uint64),
                ("shortcuts", ctypes.c_uint64), ("rounds", ctypes.c_uint32), ("device", ctypes.c_uint32),
                ("layout", ctypes.c_uint32), ("up_space_samples", ctypes.c_uint32),
                ("build_seconds", ctypes.c_double), ("mean_up_space", ctypes.c_double),
                ("max_up_space", ctypes.c_uint32), ("reserved", ctypes.c_uint32)]


def _load_lib():
    if not os.path.exists(LIB_PATH):
        raise RuntimeError(f"{LIB_PATH} is missing: build it with `python __graft_entry__.py` "
                           "(there is no CPU fallback)")
    lib = ctypes.CDLL(LIB_PATH)
    u32, u64, vp, ci = ctypes.c_uint32, ctypes.c_uint64, ctypes.c_void_p, ctypes.c_int
    pp = ctypes.POINTER(vp)
    sig = {
        "phast_build": ([u32, vp, vp, vp, ctypes.POINTER(_Opts), pp], ci),
        "phast_configure": ([vp, ctypes.POINTER(_QOpts)], ci),
        "phast_trees": ([vp, vp, u32, vp, vp], ci),
        "phast_trees_host": ([vp, vp, u32, vp, vp], ci),
        "phast_parents": ([vp, vp, u32, vp, vp, vp], ci),
        "phast_parents_ch": ([vp, vp, u32, vp, vp, vp], ci),
        "phast_sync": ([vp, vp], ci),
        "phast_diameter": ([vp, vp, u64, u32, vp, vp, vp], ci),
        "phast_diameter_witness": ([vp, vp, u64, u32, vp, vp], ci),
        "phast_betweenness": ([vp, vp, u64, u32, vp, vp], ci),
        "phast_reach": ([vp, vp, u64, u32, vp, vp], ci),
        "phast_info": ([vp, ctypes.POINTER(_Info)], ci),
        "phast_level_sizes": ([vp, vp], ci),
        "phast_order": ([vp, vp], ci),
        "phast_export": ([vp, vp, vp, vp, vp, vp, vp, vp], ci),
        "phast_bands": ([vp, vp, vp], ci),
        "phast_band_groups": ([vp, u32, vp], ci),
        "phast_schedule": ([vp, u32, vp], ci),
        "phast_save": ([vp, ctypes.c_char_p], ci),
        "phast_load": ([ctypes.c_char_p, u32, pp], ci),
        "phast_free": ([vp], None),
        "phast_strerror": ([ci], ctypes.c_char_p),
        "phast_launch_count": ([], u64),
        "phast_timing": ([vp, ci], ci),
        "phast_timing_read": ([vp, ctypes.POINTER(ctypes.c_double), ctypes.POINTER(ctypes.c_double),
                               ctypes.POINTER(ctypes.c_uint64)], ci),
        "phast_probe": ([vp, ci, vp, u32, vp, vp], ci),
    }
    for name, (args, res) in sig.items():
        f = getattr(lib, name)
        f.argtypes = args
        f.restype = res
    return lib, tuple(sig)


_lib, EXPORTED = _load_lib()


def _check(fn, rc):
    if rc != 0:
        raise PhastError(fn, rc)


def launch_count() -> int:
    """Kernels launched by libphast in this process."""
    return int(_lib.phast_launch_count())


def _stream_ptr(stream):
    if stream is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    return getattr(stream, "cuda_stream", stream)


def _sources(sources) -> np.ndarray:
    src = np.ascontiguousarray(sources, dtype=np.uint32)
    if src.ndim != 1 or src.size == 0:
        raise ValueError("sources must be a non-empty 1-D array of vertex ids")
    return src


def _check_k(k):
    if not 1 <= k <= KMAX:
        raise ValueError(f"k must be in 1..{KMAX}, got {k}")


def _device_out(t, numel, dtypes, device_index, name):
    """The tensor the library will write: on the handle's CUDA device, contiguous, of
    one of `dtypes`, with exactly `numel` elements (anything else would be an
    out-of-bounds or mistyped device write)."""
    import torch
    if not isinstance(t, torch.Tensor):
        raise TypeError(f"{name}: expected a torch tensor")
    if t.dtype not in dtypes:
        raise TypeError(f"{name}: dtype {t.dtype}, expected one of {dtypes}")
    if not t.is_cuda or (device_index is not None and t.device.index != device_index):
        raise ValueError(f"{name}: must be on cuda:{device_index}, got {t.device}")
    if not t.is_contiguous():
        raise ValueError(f"{name}: must be contiguous")
    if t.numel() != numel:
        raise ValueError(f"{name}: {t.numel()} elements, expected {numel}")
    return t



def _u32_dtypes():
    import torch
    return tuple(d for d in (torch.int32, getattr(torch, "uint32", None)) if d is not None)


@dataclass
class Info:
    n: int
    levels: int
    m: int
    m_up: int
    m_down: int
    n_tail: int
    shortcuts: int
    rounds: int
    device: int
    layout: int
    build_seconds: float
    mean_up_space: float
    max_up_space: int
    up_space_samples: int


class Phast:
    """A built hierarchy bound to one CUDA device (phast_ctx)."""

    def __init__(self, n=None, first=None, head=None, length=None, *, host_only=False, threads=0,
                 hop_limit_lo=0, hop_limit_hi=0, settled_cap=0, layout="levels-bands", _handle=None):
        self._h = None
        if _handle is not None:
            self._h = _handle
        else:
            first = np.ascontiguousarray(first, dtype=np.uint64)
            head = np.ascontiguousarray(head, dtype=np.uint32)
            length = np.ascontiguousarray(length, dtype=np.uint32)
            if head.size == 0:
                head = np.zeros(1, np.uint32)
                length = np.zeros(1, np.uint32)
            if layout not in LAYOUT_FLAGS:
                raise ValueError(f"layout must be one of {sorted(LAYOUT_FLAGS)}")
            flags = (FLAG_HOST_ONLY if host_only else 0) | LAYOUT_FLAGS[layout]
            o = _Opts(hop_limit_lo, hop_limit_hi, settled_cap, threads, flags, 0, 0)
            h = ctypes.c_void_p()
            _check("phast_build", _lib.phast_build(int(n), first.ctypes.data, head.ctypes.data,
                                                   length.ctypes.data, ctypes.byref(o), ctypes.byref(h)))
            self._h = h
        inf = self.info()
        self.n = inf.n
        self.levels = inf.levels
        self.device = inf.device
        self._perm = None

    @classmethod
    def from_graph(cls, g, **kw):
        return cls(g.n, g.first, g.head, g.len, **kw)

    @classmethod
    def load(cls, path, host_only=False):
        h = ctypes.c_void_p()
        _check("phast_load", _lib.phast_load(path.encode(), FLAG_HOST_ONLY if host_only else 0, ctypes.byref(h)))
        return cls(_handle=h)

    def save(self, path):
        _check("phast_save", _lib.phast_save(self._h, path.encode()))

    def configure(self, flags=0, top_max_vertices=0, seed_cap=0, up_smem_cap=0, band_unit=0, band_threads=0,
                  band_variant=0):
        """Query-path options (phast_configure): schedule choices only, same labels."""
        q = _QOpts(flags, top_max_vertices, seed_cap, up_smem_cap, band_unit, band_threads, band_variant)
        _check("phast_configure", _lib.phast_configure(self._h, ctypes.byref(q)))
        return self

    def close(self):
        if self._h is not None:
            _lib.phast_free(self._h)
            self._h = None

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def _out(self, out, numel, dtypes, name):
        import torch
        if out is None:
            return torch.empty(numel, dtype=dtypes[0], device=f"cuda:{self.device}")
        return _device_out(out, numel, dtypes, self.device, name)

    # ------------------------------------------------------------- queries
    def trees(self, sources, out=None, stream=None):
        """k = len(sources) trees (1 <= k <= 64); returns the device tensor [n, k]
        (uint32 bits in int32), rows in internal order (see to_original)."""
        src = _sources(sources)
        k = int(src.size)
        _check_k(k)
        out = self._out(out, self.n * k, _u32_dtypes(), "trees(out)")
        _check("phast_trees", _lib.phast_trees(self._h, src.ctypes.data, k, out.data_ptr(), _stream_ptr(stream)))
        return out.view(self.n, k)

    def trees_into(self, sources: np.ndarray, out_ptr: int, stream_ptr: int):
        """Lowest-overhead form for the bench: raw pointers (the caller owns a device
        buffer of n * len(sources) uint32), no checks beyond the library's."""
        _check("phast_trees", _lib.phast_trees(self._h, sources.ctypes.data, sources.size, out_ptr, stream_ptr))

    def trees_host(self, sources, out: np.ndarray, stream=None):
        """End-to-end entry with host buffers: result copied into `out` (uint32[n, k])."""
        src = _sources(sources)
        _check_k(int(src.size))
        if out.dtype != np.uint32 or out.size != self.n * src.size or not out.flags.c_contiguous:
            raise ValueError("out must be a C-contiguous uint32 array of n * k elements")
        _check("phast_trees_host", _lib.phast_trees_host(self._h, src.ctypes.data, src.size, out.ctypes.data,
                                                         _stream_ptr(stream)))
        return out

    def parents(self, sources, dist, out=None, stream=None):
        """Parent pointers (phast_parents) of the k trees in `dist` (the device tensor
        phast_trees wrote for the same sources); device tensor [n, k] of internal ids
        (see parents_to_original)."""
        src = _sources(sources)
        k = int(src.size)
        _check_k(k)
        _device_out(dist, self.n * k, _u32_dtypes(), self.device, "parents(dist)")
        out = self._out(out, self.n * k, _u32_dtypes(), "parents(out)")
        _check("phast_parents", _lib.phast_parents(self._h, src.ctypes.data, k, dist.data_ptr(), out.data_ptr(),
                                                   _stream_ptr(stream)))
        return out.view(self.n, k)

    def parents_ch(self, sources, dist, out=None, stream=None):
        """Parent pointers in the hierarchy G+ (phast_parents_ch, reading R19): device
        tensor [n, k] of INTERNAL ids (parents may be shortcut tails)."""
        src = _sources(sources)
        k = int(src.size)
        _check_k(k)
        _device_out(dist, self.n * k, _u32_dtypes(), self.device, "parents_ch(dist)")
        out = self._out(out, self.n * k, _u32_dtypes(), "parents_ch(out)")
        _check("phast_parents_ch", _lib.phast_parents_ch(self._h, src.ctypes.data, k, dist.data_ptr(),
                                                         out.data_ptr(), _stream_ptr(stream)))
        return out.view(self.n, k)

    def parents_to_original(self, rows: np.ndarray) -> np.ndarray:
        """[n, k] internal-order parent rows of internal ids -> [k, n] original ids (INF kept)."""
        t = self.to_original(rows)
        iperm = np.empty(self.n, np.uint32)
        iperm[self.order()] = np.arange(self.n, dtype=np.uint32)   # original id of each internal id
        fin = t != INF
        t[fin] = iperm[t[fin]]
        return t

    def sync(self, stream=None):
        _check("phast_sync", _lib.phast_sync(self._h, _stream_ptr(stream)))

    def diameter(self, sources, k_batch=64, stream=None, batch_max=None):
        """Max finite distance over the given sources (device-side; returns int after sync)."""
        src = _sources(sources)
        out = self._out(None, 1, _u32_dtypes(), "max")
        self.diameter_async(src, k_batch, out, stream=stream, batch_max=batch_max)
        self.sync(stream)
        return int(out.cpu().numpy().view(np.uint32)[0])

    def diameter_async(self, sources, k_batch, max_out, stream=None, batch_max=None):
        src = _sources(sources)
        _check_k(k_batch)
        _device_out(max_out, 1, _u32_dtypes(), self.device, "diameter(max_out)")
        bm_ptr = None
        if batch_max is not None:
            nb = -(-src.size // k_batch)
            bm_ptr = _device_out(batch_max, nb, _u32_dtypes(), self.device, "diameter(batch_max)").data_ptr()
        _check("phast_diameter", _lib.phast_diameter(self._h, src.ctypes.data, src.size, k_batch,
                                                     max_out.data_ptr(), bm_ptr, _stream_ptr(stream)))

    def diameter_witness(self, sources, k_batch=64, stream=None):
        """(D, s*, t*) with dist(s*, t*) = D, original ids (phast_diameter_witness)."""
        src = _sources(sources)
        _check_k(k_batch)
        out = np.zeros(3, np.uint32)
        _check("phast_diameter_witness", _lib.phast_diameter_witness(self._h, src.ctypes.data, src.size, k_batch,
                                                                     out.ctypes.data, _stream_ptr(stream)))
        return int(out[0]), int(out[1]), int(out[2])

    def betweenness(self, sources, k_batch=16, out=None, stream=None):
        """Partial betweenness over `sources` (phast_betweenness):
        device float64 tensor [n] in internal order (see vertex_to_original).  The call
        is synchronous on `stream`."""
        import torch
        src = _sources(sources)
        _check_k(k_batch)
        out = self._out(out, self.n, (torch.float64,), "betweenness(out)")
        _check("phast_betweenness", _lib.phast_betweenness(self._h, src.ctypes.data, src.size, k_batch,
                                                           out.data_ptr(), _stream_ptr(stream)))
        return out

    def reach(self, sources, k_batch=16, out=None, stream=None):
        """Partial exact reach over `sources` (phast_reach):
        device tensor [n] (uint32 bits in int32) in internal order.  Synchronous."""
        src = _sources(sources)
        _check_k(k_batch)
        out = self._out(out, self.n, _u32_dtypes(), "reach(out)")
        _check("phast_reach", _lib.phast_reach(self._h, src.ctypes.data, src.size, k_batch, out.data_ptr(),
                                               _stream_ptr(stream)))
        return out

    def probe(self, kind, k, out, sources=None, stream=None):
        """Bandwidth probes A33 (kind 0) / A34 (kind 1) of SURVEY.md §8(d) (phast_probe)."""
        _device_out(out, self.n * k, _u32_dtypes(), self.device, "probe(out)")
        sp = None
        if sources is not None:
            sources = _sources(sources)
            sp = sources.ctypes.data
        _check("phast_probe", _lib.phast_probe(self._h, kind, sp, k, out.data_ptr(), _stream_ptr(stream)))

    def vertex_to_original(self, vec: np.ndarray) -> np.ndarray:
        """[n] per-vertex values in internal order -> original order."""
        return np.ascontiguousarray(np.asarray(vec)[self.order()])

    def schedule(self, k: int) -> dict:
        """Launch schedule of a k-tree query (phast_schedule)."""
        out = np.zeros(6, np.uint32)
        _check("phast_schedule", _lib.phast_schedule(self._h, k, out.ctypes.data))
        return dict(fused=bool(out[0]), top_levels=int(out[1]), top_vertices=int(out[2]),
                    level_launches=int(out[3]), band_launches=int(out[4]), band_levels=int(out[5]))

    def timing(self, enable: bool):
        _check("phast_timing", _lib.phast_timing(self._h, 1 if enable else 0))

    def timing_read(self):
        """(ms of upward+seed, ms of sweep+clear, batches) summed over recorded batches."""
        a, b, c = ctypes.c_double(), ctypes.c_double(), ctypes.c_uint64()
        _check("phast_timing_read", _lib.phast_timing_read(self._h, ctypes.byref(a), ctypes.byref(b), ctypes.byref(c)))
        return a.value, b.value, c.value

    # ------------------------------------------------------------- layout / stats
    def info(self) -> Info:
        i = _Info()
        _check("phast_info", _lib.phast_info(self._h, ctypes.byref(i)))
        return Info(i.n, i.levels, i.m, i.m_up, i.m_down, i.n_tail, i.shortcuts, i.rounds,
                    -1 if i.device == 0xFFFFFFFF else i.device, i.layout, i.build_seconds,
                    i.mean_up_space, i.max_up_space, i.up_space_samples)

    def level_sizes(self) -> np.ndarray:
        out = np.empty(self.levels, np.uint32)
        _check("phast_level_sizes", _lib.phast_level_sizes(self._h, out.ctypes.data))
        return out

    def order(self) -> np.ndarray:
        """internal_of_original[v]."""
        if self._perm is None:
            out = np.empty(self.n, np.uint32)
            _check("phast_order", _lib.phast_order(self._h, out.ctypes.data))
            self._perm = out
        return self._perm

    def export(self) -> dict:
        inf = self.info()
        a = dict(level=np.empty(inf.n, np.uint32), dn_first=np.empty(inf.n + 1, np.uint32),
                 dn_tail=np.empty(max(inf.m_down, 1), np.uint32), dn_len=np.empty(max(inf.m_down, 1), np.uint32),
                 up_first=np.empty(inf.n + 1, np.uint32), up_head=np.empty(max(inf.m_up, 1), np.uint32),
                 up_len=np.empty(max(inf.m_up, 1), np.uint32))
        _check("phast_export", _lib.phast_export(self._h, *[a[k].ctypes.data for k in
                                                           ("level", "dn_first", "dn_tail", "dn_len", "up_first",
                                                            "up_head", "up_len")]))
        a["dn_tail"] = a["dn_tail"][:inf.m_down]
        a["dn_len"] = a["dn_len"][:inf.m_down]
        a["up_head"] = a["up_head"][:inf.m_up]
        a["up_len"] = a["up_len"][:inf.m_up]
        return a

    def bands(self) -> list:
        """The layout's bands (phast_bands / phast_band_groups): per band, top-most first,
        dict(seg_lo, seg_hi, ngroups, goff [seg_hi - seg_lo, ngroups + 1] internal ids)."""
        cnt = ctypes.c_uint32()
        _check("phast_bands", _lib.phast_bands(self._h, ctypes.byref(cnt), None))
        desc = np.zeros(3 * max(cnt.value, 1), np.uint32)
        _check("phast_bands", _lib.phast_bands(self._h, ctypes.byref(cnt), desc.ctypes.data))
        out = []
        for b in range(cnt.value):
            lo, hi, ng = (int(x) for x in desc[3 * b:3 * b + 3])
            goff = np.zeros((hi - lo) * (ng + 1), np.uint32)
            _check("phast_band_groups", _lib.phast_band_groups(self._h, b, goff.ctypes.data))
            out.append(dict(seg_lo=lo, seg_hi=hi, ngroups=ng, goff=goff.reshape(hi - lo, ng + 1)))
        return out

    def to_original(self, rows: np.ndarray) -> np.ndarray:
        """[n, k] internal-order labels (any 32-bit dtype) -> [k, n] uint32 in original ids."""
        rows = np.asarray(rows).view(np.uint32).reshape(self.n, -1)
        return np.ascontiguousarray(rows[self.order()].T)
