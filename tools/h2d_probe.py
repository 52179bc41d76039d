"""Host->device copy ceiling from pinned memory (one stream, one and two
concurrent streams) vs the library's host-ingest path (drgpum_trace_attribute_host)."""
import json, sys, os, time
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch
import bench
n = 1 << 28
src = torch.empty(16 * n, dtype=torch.uint8, pin_memory=True)
dst = torch.empty(16 * n, dtype=torch.uint8, device="cuda")
out = {}
for _ in range(2): dst.copy_(src, non_blocking=True)
torch.cuda.synchronize()
t0 = time.perf_counter(); dst.copy_(src, non_blocking=True); torch.cuda.synchronize()
out["one_copy_GBs"] = 16 * n / (time.perf_counter() - t0) / 1e9
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
half = 8 * n
torch.cuda.synchronize(); t0 = time.perf_counter()
with torch.cuda.stream(s1): dst[:half].copy_(src[:half], non_blocking=True)
with torch.cuda.stream(s2): dst[half:].copy_(src[half:], non_blocking=True)
torch.cuda.synchronize()
out["two_streams_GBs"] = 16 * n / (time.perf_counter() - t0) / 1e9
chunk = 1 << 26   # 64 MiB copies back to back
torch.cuda.synchronize(); t0 = time.perf_counter()
for c in range(0, 16 * n, chunk): dst[c:c + chunk].copy_(src[c:c + chunk], non_blocking=True)
torch.cuda.synchronize()
out["64MiB_chunks_GBs"] = 16 * n / (time.perf_counter() - t0) / 1e9
w = bench.Workload("C5", 1 << 28)
w.s.attribute(src); torch.cuda.synchronize()
t0 = time.perf_counter()
for _ in range(3):
    w.s.reset(); w.s.attribute(src)
torch.cuda.synchronize()
out["attribute_host_GBs"] = 3 * 16 * n / (time.perf_counter() - t0) / 1e9
print(json.dumps(out))
