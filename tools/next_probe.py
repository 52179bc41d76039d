"""Run the NEXT-2 / NEXT-3 passes once on a (possibly shortened) C2 trace, for ncu."""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
from paper_conf_asplos_linzs23_b200 import Session
from tracegen import build_config, gen_records

n = int(float(sys.argv[1])) if len(sys.argv) > 1 else 20_000_000
feature = sys.argv[2] if len(sys.argv) > 2 else "frequency"
p = build_config("C2", n_records=n)
r = torch.from_numpy(gen_records(p, 0, p.n_records).view(np.uint8)).cuda()
s = Session(p.objects, p.kinds, **{feature: True})
for _ in range(2):
    s.reset()
    s.attribute(r)
torch.cuda.synchronize()
print("ok", n, feature)
