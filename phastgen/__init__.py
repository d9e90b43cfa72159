"""phastgen -- seeded synthetic inputs shared by the oracle side and the CUDA side.

This module holds none of PHAST's arithmetic (no shortest paths, no contraction,
no sweep); it only draws graphs and source sets.  Both `oracle/` and the product
package consume its output, and neither imports the other.

Workload shapes (BASELINE.json `configs`; recipe in DESIGN.md "Input recipe"):
  C1  exact 100x100 4-neighbour grid, row-major ids, arc lengths U[1, 2^20)
  C2  road-like, ~1 M vertices                      (k=16)
  C3  road-like, ~18 M vertices / ~42 M arcs        (Europe, §II-A
      "with 18 million vertices and 42 million arcs")
  C4  road-like, ~24 M vertices / ~58 M arcs        (USA, §VIII-G
      "It has 24 million vertices and 58.3 million arcs")
  C5  road-like, ~1 M vertices (diameter over all sources)
"""
from __future__ import annotations

import ctypes
import math
import os
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "libphastgen.so")


class _PgGraph(ctypes.Structure):
    _fields_ = [
        ("n", ctypes.c_uint32),
        ("m", ctypes.c_uint64),
        ("first", ctypes.POINTER(ctypes.c_uint64)),
        ("head", ctypes.POINTER(ctypes.c_uint32)),
        ("len", ctypes.POINTER(ctypes.c_uint32)),
    ]


_lib = None


def _load():
    global _lib
    if _lib is None:
        if not os.path.exists(_LIB_PATH):
            raise RuntimeError(f"{_LIB_PATH} missing: run __graft_entry__.build()")
        lib = ctypes.CDLL(_LIB_PATH)
        P = ctypes.POINTER(_PgGraph)
        lib.pg_grid.argtypes = [ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint32,
                                ctypes.c_uint64, P]
        lib.pg_road.argtypes = [ctypes.c_uint32, ctypes.c_uint32, ctypes.c_double,
                                ctypes.POINTER(ctypes.c_double), ctypes.c_double, ctypes.c_uint32,
                                ctypes.c_uint64, ctypes.c_uint32, P]
        lib.pg_random_digraph.argtypes = [ctypes.c_uint32, ctypes.c_uint64, ctypes.c_uint32,
                                          ctypes.c_uint32, ctypes.c_uint64, P]
        lib.pg_sources.argtypes = [ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int, ctypes.c_uint64,
                                   ctypes.c_void_p]
        lib.pg_free.argtypes = [P]
        for f in (lib.pg_grid, lib.pg_road, lib.pg_random_digraph, lib.pg_sources):
            f.restype = ctypes.c_int
        lib.pg_free.restype = None
        _lib = lib
    return _lib


@dataclass
class Graph:
    """Directed graph as the paper's first/arclist CSR of out-arcs (§IV-A)."""
    n: int
    first: np.ndarray  # uint64[n+1]
    head: np.ndarray   # uint32[m]
    len: np.ndarray    # uint32[m]
    name: str = ""

    @property
    def m(self) -> int:
        return int(self.head.shape[0])

    def tails(self) -> np.ndarray:
        return np.repeat(np.arange(self.n, dtype=np.uint32), np.diff(self.first).astype(np.int64))


def _take(g: _PgGraph, name: str) -> Graph:
    lib = _load()
    n, m = int(g.n), int(g.m)
    first = np.ctypeslib.as_array(g.first, shape=(n + 1,)).copy()
    head = np.ctypeslib.as_array(g.head, shape=(max(m, 1),))[:m].copy()
    ln = np.ctypeslib.as_array(g.len, shape=(max(m, 1),))[:m].copy()
    lib.pg_free(ctypes.byref(g))
    return Graph(n, first, head, ln, name)


def grid(W: int, H: int, lo: int = 1, hi: int = 1 << 20, seed: int = 1) -> Graph:
    """W x H 4-neighbour grid, row-major ids v = W*y + x, independent arc lengths U[lo, hi)."""
    g = _PgGraph()
    rc = _load().pg_grid(W, H, lo, hi, seed, ctypes.byref(g))
    if rc != 0:
        raise ValueError(f"pg_grid failed: {rc}")
    return _take(g, f"grid{W}x{H}")


# shape-point distributions: P(s = 0,1,2,3) shape vertices per kept lattice edge
_ROAD_PRESETS = {
    # Europe: 42/18 = 2.33 arcs per vertex
    "europe": dict(p_keep=0.75, shape=(0.15, 0.35, 0.30, 0.20), oneway=0.02, per_int=3.42),
    # USA: 58.3/24 = 2.43 arcs per vertex
    "usa": dict(p_keep=0.80, shape=(0.20, 0.40, 0.25, 0.15), oneway=0.02, per_int=3.18),
}


def road(n_target: int, seed: int, preset: str = "europe", base: int = 1000, metric: str = "time") -> Graph:
    """Road-like graph with about n_target vertices in DFS layout (see gen.c).
    metric "time" (travel times, road classes 1/2/4/8x faster) or "distance" (every
    class speed 1: the paper's travel-distance metric, deeper hierarchies,
    PAPER.md:26 §VIII-G)."""
    p = _ROAD_PRESETS[preset]
    side = max(2, int(round(math.sqrt(n_target / p["per_int"]))))
    shape = (ctypes.c_double * 4)(*p["shape"])
    g = _PgGraph()
    if metric not in ("time", "distance"):
        raise ValueError("metric must be 'time' or 'distance'")
    rc = _load().pg_road(side, side, p["p_keep"], shape, p["oneway"], base, seed, int(metric == "distance"),
                         ctypes.byref(g))
    if rc != 0:
        raise ValueError(f"pg_road failed: {rc}")
    return _take(g, f"road-{preset}-{metric}-{n_target}-s{seed}")


def random_digraph(n: int, m: int, lo: int, hi: int, seed: int) -> Graph:
    """Uniform random digraph (self-loops, parallel arcs allowed), lengths U[lo, hi] inclusive."""
    g = _PgGraph()
    rc = _load().pg_random_digraph(n, m, lo, hi, seed, ctypes.byref(g))
    if rc != 0:
        raise ValueError(f"pg_random_digraph failed: {rc}")
    return _take(g, f"rand{n}x{m}-s{seed}")


def sources(n: int, count: int, seed: int, distinct: bool = True) -> np.ndarray:
    out = np.empty(count, dtype=np.uint32)
    rc = _load().pg_sources(n, count, 1 if distinct else 0, seed, out.ctypes.data)
    if rc != 0:
        raise ValueError(f"pg_sources failed: {rc}")
    return out


# BASELINE.json configs -> (graph factory, sources seed, k)
CONFIGS = {
    "C1": dict(graph=lambda: grid(100, 100, 1, 1 << 20, seed=1), src_seed=101, k=1,
               desc="100x100 grid, 10k vertices, 39.6k arcs, U[1,2^20) lengths"),
    "C2": dict(graph=lambda: road(1_000_000, seed=2), src_seed=102, k=16,
               desc="road-like ~1M vertices (Europe shape), k=16"),
    "C3": dict(graph=lambda: road(18_000_000, seed=3), src_seed=103, k=64,
               desc="road-like ~18M vertices / ~42M arcs (Europe-scale), k=16/32/64"),
    "C4": dict(graph=lambda: road(24_000_000, seed=4, preset="usa"), src_seed=104, k=64,
               desc="road-like ~24M vertices / ~58M arcs (USA-scale), 8192 sources"),
    "C5": dict(graph=lambda: road(1_000_000, seed=5), src_seed=105, k=64,
               desc="road-like ~1M vertices, diameter over all sources"),
    # NEXT-4: the travel-DISTANCE metric (deeper hierarchy, §VIII-G)
    "C2D": dict(graph=lambda: road(1_000_000, seed=2, metric="distance"), src_seed=102, k=16,
                desc="road-like ~1M vertices, travel-distance metric, k=16"),
}
