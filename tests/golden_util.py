"""Load tests/golden/*.json fixtures (paper worked examples) into arrays."""
import json
import os

import numpy as np

from tracegen import OBJ_DTYPE, REC_DTYPE, NEVER

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")
KIND = {"ALLOC": 0, "FREE": 1, "MEMCPY": 2, "MEMSET": 3, "KERNEL": 4}


def golden_names():
    return sorted(f[:-5] for f in os.listdir(GOLDEN) if f.endswith(".json"))


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
