"""Shared test helpers: building tiny profile tables and traces (no method arithmetic)."""
import json
import os

import numpy as np

from protean_inputs import Profiles, concat, pack_meta

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")
NAMES = ["1g", "2g", "3g", "4g", "7g"]
CAP = [5120, 10240, 20480, 20480, 40960]       # T2 memory per profile (MiB)
COMPUTE = [1, 2, 3, 4, 7]


def geoms_array(rows):
    g = np.full((len(rows), 8), 255, np.uint8)
    for j, r in enumerate(rows):
        g[j, : len(r)] = r
    return g


def tables(solo, fbr, mem, bsz=None, slo=None, tmo=None, geoms=None, geometry_set=None):
    solo = np.asarray(solo, np.int32).reshape(-1, 5)
    M = solo.shape[0]
    fbr = np.asarray(fbr, np.int32).reshape(M, 5)
    mem = np.asarray(mem, np.int32).reshape(M)
    bsz = np.asarray(bsz if bsz is not None else [1] * M, np.int32)
    slo = np.asarray(slo if slo is not None else 3 * solo[:, 4], np.int32)
    tmo = np.asarray(tmo if tmo is not None else [0] * M, np.int32)
    if geoms is not None:
        return Profiles(solo, fbr, mem, bsz, slo, tmo, 2, geoms_array(geoms))
    return Profiles(solo, fbr, mem, bsz, slo, tmo, geometry_set or 0, None)


def w1():
    g = json.load(open(os.path.join(GOLDEN, "w1_worked_epoch.json")))
    m = g["models"]
    P = tables(m["solo_us"], m["fbr_ppm"], m["mem_mib"], m["batch_size"], m["slo_us"], m["timeout_us"],
               geoms=g["geoms"])
    req = np.array(g["requests"])
    tr = concat([(req[:, 0].astype(np.uint32), pack_meta(req[:, 1], req[:, 2]))], g["trace_len_us"])
    return g, P, tr


def trace_from(rows, trace_len):
    """rows: list of (arrival, model, strict) for one replica."""
    rows = sorted(rows, key=lambda r: r[0])
    a = np.array([r[0] for r in rows], np.uint32)
    return concat([(a, pack_meta([r[1] for r in rows], [r[2] for r in rows]))], trace_len)
