"""Run bench.py's step for one config twice (the first is the warm-up), for
ncu captures: `ncu -k regex:attribute_kernel -s <launches of one step> -c 1`.
usage: python tools/ncu_one.py --config C5 [--steps 2]"""
import argparse, os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch
import bench

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C2")
ap.add_argument("--steps", type=int, default=2)
ap.add_argument("--records", type=int, default=None)
a = ap.parse_args()
w = bench.Workload(a.config, a.records)
for _ in range(a.steps):
    w.step()
torch.cuda.synchronize()
print(a.config, "chunks", len(w.chunks), "launches", w.s.launch_count())
