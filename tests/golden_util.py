"""Load tests/golden/*.json fixtures (paper worked examples) into arrays."""
import json
import os

import numpy as np

from tracegen import OBJ_DTYPE, REC_DTYPE, NEVER

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")
KIND = {"ALLOC": 0, "FREE": 1, "MEMCPY": 2, "MEMSET": 3, "KERNEL": 4}


def golden_names():
    """Fixtures given as explicit objects / timeline / records (the ones with
    a "program" spec instead are built by their own helper below)."""
    out = []
    for f in sorted(os.listdir(GOLDEN)):
        if f.endswith(".json") and "program" not in load(f[:-5]):
            out.append(f[:-5])
    return out


def load(name):
    with open(os.path.join(GOLDEN, name + ".json")) as f:
        return json.load(f)


def to_arrays(fx, kinds=None, records=None):
    kinds = np.array([KIND[k] for k in (kinds or fx["kinds"])], dtype=np.uint8)
    objs = np.zeros(len(fx["objects"]), dtype=OBJ_DTYPE)
    names = {}
    for i, o in enumerate(fx["objects"]):
        names[o["name"]] = i
        objs[i] = (o["base"], o["size"], o["elem_size"], o["t_alloc"],
                   NEVER if o["t_free"] is None else o["t_free"], i)
    recs_in = records if records is not None else fx["records"]
    recs = np.zeros(len(recs_in), dtype=REC_DTYPE)
    for k, r in enumerate(recs_in):
        o = objs[names[r["obj"]]]
        E = int(o["elem_size"])
        recs[k] = (int(o["base"]) + r["elem"] * E, r["count"] * E,
                   r["ts"] | (int(r["w"]) << 31))
    return objs, kinds, recs, names


def gramschmidt_polybench(fx):
    """The program of tests/golden/gramschmidt_polybench.json (PolyBench/GPU
    GramSchmidt's access structure on R_gpu, l.400 / Fig. 8): returns
    (objects, kinds, records, kernel3 mask u8[n_api], kernel3 timestamps)."""
    N = int(fx["program"]["N"])
    f = int(fx["program"]["touches_per_element"])
    base = 1 << 30
    kinds = [KIND["ALLOC"], KIND["MEMCPY"]]
    recs = [(base, 4 * N * N, 1 | (1 << 31))]            # H2D copy writes all of R
    k3 = []
    for k in range(N):
        t1 = len(kinds); kinds.append(KIND["KERNEL"])       # kernel1: R[k][k] = sqrt(nrm)
        recs.append((base + 4 * (k * N + k), 4, t1 | (1 << 31)))
        t2 = len(kinds); kinds.append(KIND["KERNEL"])       # kernel2: reads R[k][k]
        recs.append((base + 4 * (k * N + k), 4, t2))
        t3 = len(kinds); kinds.append(KIND["KERNEL"])       # kernel3: row k, j > k
        k3.append(t3)
        if k + 1 < N:
            for rep in range(f):
                recs.append((base + 4 * (k * N + k + 1), 4 * (N - 1 - k), t3 | ((rep != 1) << 31)))
    kinds.append(KIND["FREE"])
    kinds = np.array(kinds, dtype=np.uint8)
    objs = np.zeros(1, dtype=OBJ_DTYPE)
    objs[0] = (base, 4 * N * N, 4, 0, len(kinds) - 1, 0)
    r = np.array(recs, dtype=REC_DTYPE)
    mask = np.zeros(len(kinds), np.uint8)
    mask[k3] = 1
    return objs, kinds, r, mask, k3
