"""Probe: does torch symmetric memory expose an NVLS multicast pointer on this
box (one rank)?  Prints one JSON line."""
import json, os, socket
import torch
import torch.distributed as dist
import torch.distributed._symmetric_memory as symm_mem

with socket.socket() as s:
    s.bind(("127.0.0.1", 0)); port = s.getsockname()[1]
os.environ.setdefault("MASTER_ADDR", "127.0.0.1"); os.environ["MASTER_PORT"] = str(port)
torch.cuda.set_device(0)
dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
out = {}
try:
    buf = symm_mem.empty(1 << 20, dtype=torch.uint8, device="cuda")
    h = symm_mem.rendezvous(buf, dist.group.WORLD)
    out["has_multicast_support"] = bool(getattr(h, "has_multicast_support", False))
    out["multicast_ptr"] = int(getattr(h, "multicast_ptr", 0) or 0)
    out["buffer_ptrs"] = [int(p) for p in h.buffer_ptrs]
except Exception as e:
    out["error"] = f"{type(e).__name__}: {e}"
try:
    import subprocess
    out["nvidia_smi_topo"] = subprocess.run(["nvidia-smi", "topo", "-m"], capture_output=True, text=True).stdout[:800]
    out["fabric"] = subprocess.run(["nvidia-smi", "-q", "-d", "FABRIC"], capture_output=True, text=True).stdout[:800]
except Exception as e:
    out["smi_error"] = str(e)
print(json.dumps(out))
dist.destroy_process_group()
