#!/usr/bin/env python
"""Benchmark: DrGPUM per-access attribution on B200 (BASELINE.json metric).

One *step* is one pass of the whole hot path over the workload's records:
reset the shadow (bitmaps / hit rows / first / last / counters), attribute
every record (A1-A5), [merge across ranks], and the per-object reductions +
pattern classification (A6-A7), all on the device.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config C5]
  python bench.py --impl reference ...   # the CPU oracle as the reference arm
  python bench.py --gpus 2 --dry-run     # rank plumbing only (gloo, no GPU)

Default workload: C5, BASELINE.json's scaling sweep (1.6e10 records over 10^6
objects), the largest config; it does not fit one GPU's HBM (256 GB of
records), so at N=1 it is streamed through HBM in 2^30-record chunks generated
on the device (generation outside the timed events), and at N>=4 every rank's
shard is resident.  Extra key ``other_configs``: C4 (the largest config that
is resident on one GPU) and C2, measured in the same run.

--gpus N > 1 without torchrun in the environment re-launches this script
under ``torch.distributed.run`` with N ranks (one per GPU, NCCL): rank r
attributes records [r*N/P, (r+1)*N/P) of the same trace, then the one
exchange step merges the shadows (paper_conf_asplos_linzs23_b200/parallel.py)
-- strong scaling.  Rank 0 prints ONE JSON line.

Every run checks its results against the oracle's golden digests
(tests/golden/digests/<config>.json, written by tools/make_golden_digests.py
from oracle/ alone) when they exist for the measured record count: key
``parity``.
"""
import argparse
import json
import os
import socket
import statistics
import subprocess
import sys
import tempfile
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "access records/sec (and HBM GB/s vs peak) at 1/2/4/8 B200 vs CPU oracle"
WORKLOADS = {
    "C1": "C1 synthetic (BASELINE configs[0]): 2^20 records, 4-8 B accesses, 64 objects (16 MiB), 100 access APIs",
    "C2": "C2 Rodinia-style HPC trace (BASELINE configs[1]): 1e8 records over 1000 objects (4 GiB), "
          "strided + partial-object access, 3700 access APIs",
    "C3": "C3 ResNet-50 training-iteration-shaped trace (BASELINE configs[2]): 1e9 records over 20K tensors "
          "in a 12 GiB best-fit caching pool (address reuse), short-lived activations",
    "C4": "C4 LLM-inference-shaped trace (BASELINE configs[3]): 4e9 records over 100K objects "
          "(120 GiB live footprint, reused 4 GiB activation arena), Zipf-skewed hot weights / KV blocks",
    "C5": "C5 scaling sweep (BASELINE configs[4]): 1.6e10 records over 1M objects, record-range sharded; "
          "streamed through HBM in 2^30-record chunks generated on the device when a shard exceeds 96 GiB",
}
# traces above RESIDENT_BYTES per rank are streamed in GEN_CHUNK chunks
GEN_CHUNK = 1 << 30
RESIDENT_BYTES = 96 << 30
CONSUME = False   # reduce-and-clear in Workload steps (main(): --consume)
FALLBACK_HBM_GBS = 6650.0
GOLDEN_DIR = os.path.join(ROOT, "tests", "golden", "digests")


def args_():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="C5", choices=sorted(WORKLOADS))
    ap.add_argument("--records", type=int, default=None, help="override the record count")
    ap.add_argument("--e2e-steps", type=int, default=None)
    ap.add_argument("--merge", default="owned", choices=["owned", "owned-nvls", "peers", "nccl"],
                    help="N>1 exchange step over torch symmetric memory (NVLink P2P): owned = "
                         "drgpum_merge_peers_owned + per-rank finalize of its objects + "
                         "drgpum_gather_peers; owned-nvls = the same with objects several ranks "
                         "touched read through the NVSwitch multicast mapping (NVLS OR, when the "
                         "box provides one); peers = drgpum_merge_peers (every rank gets the "
                         "whole merged shadow, finalizes everything); nccl = all-to-all + "
                         "merge_or + all-gather")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-next", action="store_true", help="skip the SURVEY §8(f) NEXT-row timings")
    ap.add_argument("--consume", action="store_true",
                    help="reduce-and-clear: finalize zeroes the bitmaps it reduces, the next reset skips them "
                         "(measured slower than the separate sparse reset: DESIGN.md section 6)")
    ap.add_argument("--no-graph", action="store_true",
                    help="time eager launches instead of CUDA-graph replays of the step")
    ap.add_argument("--no-parity", action="store_true", help="skip the golden-digest check")
    ap.add_argument("--extra-configs", default="C4,C2",
                    help="comma list of configs measured after the main one at N=1 (key other_configs); '' = none")
    ap.add_argument("--cpu-sample", type=int, default=250_000_000,
                    help="target records of the oracle's timed sample (an object_sample of the workload)")
    ap.add_argument("--e2e-sample", type=int, default=1 << 28,
                    help="records per step of the host-buffer (e2e) leg")
    ap.add_argument("--ref-sample", type=int, default=4_000_000,
                    help="target records per reference-arm step (an object_sample of the workload)")
    ap.add_argument("--dry-run", action="store_true",
                    help="launch the ranks and check the process-group plumbing only (gloo; no GPU)")
    return ap.parse_args()


def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            mp = json.load(f)
        return float(mp["hbm_gbs"]), "MEASURED_PEAKS.json hbm_gbs (measured copy, burst)"
    except Exception:
        return FALLBACK_HBM_GBS, "fallback 6.65 TB/s from B200_PROFILING.md (MEASURED_PEAKS.json absent)"


class ClockSampler:
    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index):
        self.f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
        try:
            self.p = subprocess.Popen(["nvidia-smi", "-i", str(gpu_index), f"--query-gpu={self.FIELDS}",
                                       "--format=csv,noheader,nounits", "-lms", "100"],
                                      stdout=self.f, stderr=subprocess.DEVNULL)
        except Exception:
            self.p = None

    def stop(self):
        if self.p is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.p.terminate()
        self.p.wait()
        self.f.flush()
        self.f.seek(0)
        sm, smax, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in self.f.read().splitlines():
            c = [x.strip() for x in line.split(",")]
            if len(c) < 9:
                continue
            try:
                sm.append(float(c[1]))
                smax.append(float(c[2]))
            except ValueError:
                continue
            for nm, v in zip(names, c[5:9]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        os.unlink(self.f.name)
        return {"sm_mhz": statistics.median(sm) if sm else None,
                "sm_max_mhz": max(smax) if smax else None,
                "samples": len(sm), "reasons": sorted(reasons)}


def cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def relaunch(a):
    """--gpus N > 1 outside torchrun: run this script under
    torch.distributed.run with N ranks on this node and pass its exit code on."""
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={a.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(free_port()),
           os.path.abspath(__file__)] + sys.argv[1:]
    print(f"bench.py: launching {a.gpus} ranks: {' '.join(cmd)}", file=sys.stderr, flush=True)
    return subprocess.call(cmd)


def world_env():
    return (int(os.environ.get("WORLD_SIZE", "1")), int(os.environ.get("RANK", "0")),
            int(os.environ.get("LOCAL_RANK", "0")))


def dry_run(a):
    """The rank plumbing of an N-GPU run without a GPU: every rank joins a
    gloo process group, the ranks are counted with an all_reduce, rank 0
    prints one line."""
    import torch
    import torch.distributed as dist
    world, rank, _ = world_env()
    if world != a.gpus:
        raise SystemExit(f"bench.py: WORLD_SIZE={world} but --gpus {a.gpus}")
    if world > 1:
        dist.init_process_group("gloo")
    t = torch.tensor([1, rank], dtype=torch.int64)
    if world > 1:
        dist.all_reduce(t)
    if rank == 0:
        print(json.dumps({"dry_run": True, "n_gpus": world, "ranks_reporting": int(t[0]),
                          "rank_sum": int(t[1]), "backend": "gloo" if world > 1 else "none",
                          "config": {"workload": WORKLOADS[a.config]}}), flush=True)
    if world > 1:
        dist.destroy_process_group()


# ---------------------------------------------------------------- CPU oracle
def oracle_sample(prog, target):
    """A bounded sample of the workload for the CPU oracle: 1/k of the objects
    (index % k == 0) with every record that targets them, over the full
    timeline (tracegen.object_sample), k chosen for ~target records."""
    from tracegen import object_sample
    k = max(1, int(round(prog.n_records / max(1, target))))
    sub = object_sample(prog, k, 0) if k > 1 else prog
    desc = (f"1/{k} of the {prog.name} objects (index % {k} == 0, {sub.n_obj} of {prog.n_obj}) with every "
            f"record that targets them: {sub.n_records} of {prog.n_records} records, the full {prog.n_api}-API "
            f"timeline; one pass: load + attribute + stats + patterns (O1, single thread)")
    return sub, desc


def time_oracle(objs, kinds, recs):
    """The oracle as it stands (single-threaded C++), one full pass."""
    from oracle import Oracle
    t0 = time.perf_counter()
    o = Oracle(objs, kinds)
    o.attribute(recs)
    o.stats()
    o.patterns()
    return time.perf_counter() - t0


def reference_arm(a):
    """--impl reference: the CPU oracle, timed on the host cores, on our
    config (a bounded object sample of it per step)."""
    world, rank, _ = world_env()
    if rank != 0:
        return
    from tracegen import build_config, gen_records
    prog = build_config(a.config, **({"n_records": a.records} if a.records else {}))
    sub, desc = oracle_sample(prog, a.ref_sample)
    recs = gen_records(sub, 0, sub.n_records)
    for _ in range(a.warmup):
        time_oracle(sub.objects, sub.kinds, recs)
    ts = [time_oracle(sub.objects, sub.kinds, recs) for _ in range(a.steps)]
    t = sum(ts) / len(ts)
    v = sub.n_records / t
    print(json.dumps({
        "impl": "reference", "metric": METRIC, "value": v, "unit": "records/s",
        "n_gpus": a.gpus, "steps": a.steps, "warmup": a.warmup, "ms_per_step": t * 1e3,
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "u32",
        "data": f"synthetic (tracegen {prog.name}, seed {prog.seed:#x})",
        "config": {"workload": WORKLOADS[a.config], "records": prog.n_records, "objects": prog.n_obj,
                   "sample_records": sub.n_records, "sample_objects": sub.n_obj},
        "same_config": True,
        "cpu_baseline": {"value": v, "unit": "records/s", "cores": 1, "kind": "oracle",
                         "sample": desc, "cpu": cpu_model()},
        "e2e": {"value": v, "unit": "records/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }), flush=True)


# ---------------------------------------------------------------- GPU workload
class Workload:
    """One config's records (resident, or regenerated chunk by chunk on the
    device), its Session, and the step that bench.py times.  The GPU parity
    tests (tests/test_gpu_fullsize.py) run exactly this step."""

    def __init__(self, cfg, records=None, rank=0, world=1, merge="owned", resident_bytes=RESIDENT_BYTES):
        import torch
        from paper_conf_asplos_linzs23_b200 import Session
        from tracegen import build_config
        from tracegen.device import DeviceProgram
        from paper_conf_asplos_linzs23_b200.parallel import shard_range
        self.torch = torch
        self.cfg, self.rank, self.world = cfg, rank, world
        self.prog = build_config(cfg, **({"n_records": records} if records else {}))
        self.N = self.prog.n_records
        self.lo, self.hi = shard_range(self.N, rank, world)
        self.n_local = self.hi - self.lo
        self.chunked = 16 * self.n_local > resident_bytes
        self.dp = DeviceProgram(self.prog)
        gen = [(c, min(c + GEN_CHUNK, self.n_local)) for c in range(0, self.n_local, GEN_CHUNK)]
        self.d_recs = torch.empty(16 * max(1, GEN_CHUNK if self.chunked else self.n_local),
                                  dtype=torch.uint8, device="cuda")
        if self.chunked:
            self.chunks = gen
        else:
            for c0, c1 in gen:   # device generation, never timed
                self.dp.gen(self.lo + c0, self.lo + c1, out=self.d_recs[16 * c0:16 * c1])
            self.chunks = [(0, self.n_local)]
        torch.cuda.synchronize()
        self.sm, self.merge_note = None, "none (1 rank)"
        self.nvls = merge == "owned-nvls"
        if self.nvls:
            merge = "owned"
        if world > 1 and merge in ("peers", "owned"):
            from paper_conf_asplos_linzs23_b200.parallel import SymmetricMerge
            try:
                self.sm = SymmetricMerge()
                self.s = Session(self.prog.objects, self.prog.kinds, workspace_alloc=self.sm.alloc)
                mc = self.sm.multicast_ptr() if self.nvls else 0
                self.merge_note = (("drgpum_merge_peers_owned" + ("_nvls (NVSwitch multicast OR)" if mc else "") +
                                    " + finalize of the owned objects + "
                                    "drgpum_gather_peers over torch symmetric memory (NVLink P2P)" +
                                    (" [nvls requested, no multicast mapping]" if self.nvls and not mc else ""))
                                   if merge == "owned" else
                                   "drgpum_merge_peers over torch symmetric memory (one kernel per rank, NVLink P2P)")
            except Exception as e:   # symmetric memory unavailable: the NCCL exchange instead, said so
                self.sm = None
                self.merge_note = f"NCCL all_to_all + merge_or + all_gather (symmetric memory unavailable: {e})"
        if self.sm is None:
            self.s = Session(self.prog.objects, self.prog.kinds)
            if world > 1 and merge == "nccl":
                self.merge_note = "NCCL all_to_all + merge_or + all_gather"
        self.owned = self.sm is not None and merge == "owned"
        self.stream = torch.cuda.current_stream()
        self.graph = None
        # reduce-and-clear: the step's finalize zeroes the bitmap words it
        # reduces, so the next step's reset skips them (one shadow pass per
        # step instead of two; no effect after an owned merge)
        self.consume = CONSUME
        self.s.set_finalize_consume(self.consume)

    def keep_shadow(self):
        """One more (untimed) step without reduce-and-clear, so that the
        shadow holds the trace's bitmaps for the touched-word count and the
        parity digests read after the timed region (collective at N > 1)."""
        if self.consume:
            self.s.set_finalize_consume(False)
            self.consume = False
            self.step()
            self.torch.cuda.synchronize()

    # -- the step ------------------------------------------------------------
    def do_merge(self):
        if self.world > 1:
            from paper_conf_asplos_linzs23_b200.parallel import merge_session
            if self.owned:
                self.sm.merge_owned(self.s, nvls=self.nvls)
            elif self.sm is not None:
                self.sm.merge(self.s)
            else:
                merge_session(self.s)

    def do_finalize(self):
        self.s.finalize()
        if self.owned:
            self.sm.gather(self.s)

    def step(self, ev=None):
        """ev: per-phase event pairs [reset, attribute (per chunk), merge,
        finalize]; generation of a chunk lies outside its attribute pair."""
        st = self.stream
        if ev: ev["reset"][0].record(st)
        self.s.reset()
        if ev: ev["reset"][1].record(st)
        for k, (c0, c1) in enumerate(self.chunks):
            if self.chunked:
                self.dp.gen(self.lo + c0, self.lo + c1, out=self.d_recs)
            if ev: ev["attr"][k][0].record(st)
            self.s.attribute(self.d_recs[:16 * (c1 - c0)])
            if ev: ev["attr"][k][1].record(st)
        if ev: ev["merge"][0].record(st)
        self.do_merge()
        if ev: ev["merge"][1].record(st)
        if ev: ev["fin"][0].record(st)
        self.do_finalize()
        if ev: ev["fin"][1].record(st)

    def events(self):
        E = lambda: (self.torch.cuda.Event(enable_timing=True), self.torch.cuda.Event(enable_timing=True))
        return {"reset": E(), "attr": [E() for _ in self.chunks], "merge": E(), "fin": E()}

    @staticmethod
    def phases(ev):   # ms
        el = lambda e: e[0].elapsed_time(e[1])
        return [el(ev["reset"]), sum(el(e) for e in ev["attr"]), el(ev["merge"]), el(ev["fin"])]

    def capture(self, warmup):
        """The step as one CUDA graph (resident traces only): reset, attribute
        + range expansion, [barrier, merge, barrier, finalize, barrier,
        gather, barrier -- the symmetric-memory device barriers], finalize.
        Every rank agrees on graph vs eager before any replay."""
        torch = self.torch
        ok, why = not self.chunked, "chunked trace (device generation between the chunks)"
        if ok and self.world > 1 and self.sm is None:
            ok, why = False, "NCCL exchange (host-side collectives)"
        g = None
        if ok:
            try:
                g = torch.cuda.CUDAGraph()
                with torch.cuda.graph(g):
                    self.step()
                why = None
            except Exception as e:   # noqa: BLE001 -- reported in the JSON line
                g, ok, why = None, False, f"capture failed: {type(e).__name__}: {e}"
        if self.world > 1:
            import torch.distributed as dist
            t = torch.tensor([1 if g is not None else 0], device="cuda")
            dist.all_reduce(t, op=dist.ReduceOp.MIN)
            if int(t) == 0 and g is not None:
                g, why = None, "another rank could not capture"
        self.graph = g
        self.graph_note = why
        if g is not None:
            for _ in range(warmup):
                g.replay()
            torch.cuda.synchronize()
        return g is not None

    def run(self):
        if self.graph is not None:
            self.graph.replay()
        else:
            self.step()

    def close(self):
        self.graph = None
        self.s.close()
        del self.s, self.d_recs, self.dp
        self.torch.cuda.synchronize()
        self.torch.cuda.empty_cache()


def golden(cfg, n_records):
    path = os.path.join(GOLDEN_DIR, f"{cfg}.json")
    if not os.path.exists(path):
        return None, path
    with open(path) as f:
        g = json.load(f)
    return (g if int(g.get("records", -1)) == int(n_records) else None), path


def parity_check(w, full):
    """Compare this run's results with the oracle's golden digests (stats,
    reports, counters; with full=True also every bitmap and accessing-API
    set).  After an owned merge every rank holds all stats / reports."""
    from tests.digest_util import compare, results_digest, session_digest
    g, path = golden(w.cfg, w.N)
    if g is None:
        return {"checked": False, "why": f"no golden digest for {w.cfg} at {w.N} records ({os.path.relpath(path, ROOT)})"}
    t0 = time.perf_counter()
    if full:
        d = session_digest(w.s)
        keys = ("counters", "stats_sha", "reports_sha", "bitmap_sha", "access_sha")
    else:
        stats, ctr = w.s.object_stats()
        d = results_digest(w.s.objects, ctr, stats, w.s.patterns())
        keys = ("counters", "stats_sha", "reports_sha")
    bad = compare(d, g, keys)
    return {"checked": True, "golden": os.path.relpath(path, ROOT), "compared": list(keys),
            "ok": not bad, "mismatches": bad[:20], "seconds": time.perf_counter() - t0}


def measure(w, a, steps, warmup, clocks=False, use_graph=True):
    """Warm up, phase breakdown (eager, events between phases), then the timed
    region: K steps (graph replays when the trace is resident) bracketed by
    barrier + synchronize, device time from events on the launching stream
    (chunked traces: the sum of the steps' phase events, generation excluded)."""
    import torch
    import torch.distributed as dist
    world = w.world
    barrier = (lambda: dist.barrier()) if world > 1 else (lambda: None)
    for _ in range(warmup):
        w.step()
    torch.cuda.synchronize()
    l0 = w.s.launch_count()
    w.step()
    step_launches = w.s.launch_count() - l0
    evs = [w.events() for _ in range(steps)]
    torch.cuda.synchronize()
    for k in range(steps):
        w.step(evs[k])
    torch.cuda.synchronize()
    ph_mean = np.array([w.phases(e) for e in evs]).mean(axis=0)
    graphed = use_graph and w.capture(warmup)
    clk = ClockSampler(int(os.environ.get("LOCAL_RANK", "0"))) if clocks else None
    if clk:
        time.sleep(0.3)
    t_start, t_end = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    launches0 = w.s.launch_count()
    barrier()
    torch.cuda.synchronize()
    wall0 = time.perf_counter()
    t_start.record(w.stream)
    tev = [w.events() for _ in range(steps)] if w.chunked else None
    for k in range(steps):
        if graphed:
            w.graph.replay()
        else:
            w.step(tev[k] if w.chunked else None)
    t_end.record(w.stream)
    torch.cuda.synchronize()
    barrier()
    wall = time.perf_counter() - wall0
    clocks_v = clk.stop() if clk else None
    # graph replays do not pass through the library's launch counter
    launches = step_launches * steps if graphed else w.s.launch_count() - launches0
    ms_total = t_start.elapsed_time(t_end)
    if w.chunked:
        ms_total = float(sum(sum(w.phases(e)) for e in tev))
    if world > 1:
        t = torch.tensor([ms_total] + ph_mean.tolist(), dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms_total = float(t[0])
        ph_mean = t[1:].cpu().numpy()
    return {"ms_step": ms_total / steps, "phases": ph_mean, "launches": launches, "graphed": graphed,
            "wall": wall, "clocks": clocks_v, "step_launches": step_launches}


def touched_words(w):
    """Touched shadow words of THIS rank's attribution (the algorithmic
    write-back of A3/A4).  At N>1 the merged shadow is not what the rank's
    kernel wrote, so the shard is attributed once more alone, counted, and
    the merged step re-run (collectively) for the results read afterwards."""
    import torch
    if w.world > 1:
        import torch.distributed as dist
        w.s.reset()
        for c0, c1 in w.chunks:
            if w.chunked:
                w.dp.gen(w.lo + c0, w.lo + c1, out=w.d_recs)
            w.s.attribute(w.d_recs[:16 * (c1 - c0)])
        n = int(torch.count_nonzero(w.s.or_words()).item())
        dist.barrier()
        w.step()
        torch.cuda.synchronize()
        return n
    return int(torch.count_nonzero(w.s.or_words()).item())


def roofline(w, m, touched, hbm, hbm_src):
    attr_ms = float(m["phases"][1])
    alg_bytes = 16.0 * w.n_local + 4.0 * touched
    achieved = alg_bytes / (attr_ms / 1e3) / 1e9
    traffic = None
    tfile = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tfile):
        try:
            t = json.load(open(tfile)).get(w.cfg)
            traffic = None if t is None else int(t["bytes_per_launch"])   # one launch of w.chunks
        except Exception:
            traffic = None
    return {"bound": "hbm", "achieved": achieved, "peak": hbm, "unit": "GB/s",
            "frac": achieved / hbm, "traffic": traffic,
            "algorithmic_bytes_per_launch": alg_bytes / len(w.chunks),
            "launches_per_step": len(w.chunks),
            "kernel": "drgpum_trace_attribute (attribute_kernel + range_expand_kernel)",
            "algorithmic_bytes": alg_bytes, "records_per_rank": w.n_local,
            "bytes_rule": "16 B per record + 4 B per touched shadow word",
            "peak_source": hbm_src}


def e2e_leg(w, a, steps):
    """The same metric through the public API with HOST buffers: every step
    copies its records from pinned host memory (drgpum_trace_attribute_host,
    pipelined H2D staging) and reads the results back (object_stats +
    patterns).  The sample is the first e2e_sample records of the rank's
    shard (generated on the device, copied into the pinned buffer once)."""
    import torch
    import torch.distributed as dist
    n = min(w.n_local, a.e2e_sample)
    pinned = torch.empty(n * 16, dtype=torch.uint8, pin_memory=True)
    tmp = torch.empty(16 * min(n, GEN_CHUNK), dtype=torch.uint8, device="cuda")
    for c0 in range(0, n, GEN_CHUNK):
        c1 = min(n, c0 + GEN_CHUNK)
        w.dp.gen(w.lo + c0, w.lo + c1, out=tmp)
        pinned[16 * c0:16 * c1].copy_(tmp[:16 * (c1 - c0)])
    del tmp
    torch.cuda.synchronize()
    from paper_conf_asplos_linzs23_b200 import pinned_array, STATS_DTYPE, REPORT_DTYPE
    h_stats = pinned_array(w.prog.n_obj, STATS_DTYPE)      # result buffers a serving caller
    h_reps = pinned_array(w.prog.n_obj, REPORT_DTYPE)      # keeps, page-locked like the input

    def one():
        w.s.reset()
        w.s.attribute(pinned)                 # drgpum_trace_attribute_host: H2D inside
        w.do_merge()
        if w.owned:
            w.do_finalize()
        w.s.object_stats(out=h_stats)         # D2H of the results
        w.s.patterns(out=h_reps)

    for _ in range(2):
        one()
    torch.cuda.synchronize()
    if w.world > 1:
        dist.barrier()
    w0 = time.perf_counter()
    for _ in range(steps):
        one()
    torch.cuda.synchronize()
    e2e_s = (time.perf_counter() - w0) / steps
    if w.world > 1:
        t = torch.tensor([e2e_s], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        e2e_s = float(t[0])
    return {"value": n * w.world / e2e_s, "unit": "records/s", "h2d_bytes_per_step": 16 * n,
            "records_per_rank": n, "d2h_bytes_per_step": int(w.prog.n_obj * (56 + 32) + 40),
            "ms_per_step": e2e_s * 1e3,
            "path": "Session.attribute(pinned host tensor) -> drgpum_trace_attribute_host; "
                    "object_stats + patterns (D2H into pinned result arrays)",
            "sample": f"first {n} records of the rank's shard per step"}


def next_rows(prog, d_recs, plain_attr_ms, reps=5):
    """SURVEY §8(f) rows on the same resident trace, each timed on its own
    (not part of the step): NEXT-3 SA and NEXT-2 NUAF as the extra device time
    their passes add to drgpum_trace_attribute (CUDA events), NEXT-1 RA and
    NEXT-4 (graph + Kahn + patterns on T, 8 streams) as host wall time of the
    synchronous C-ABI calls."""
    import torch
    from paper_conf_asplos_linzs23_b200 import Session
    from tracegen.streams import assign_streams
    stream = torch.cuda.current_stream()
    N = prog.n_records
    out = {}
    # NEXT-2 processes a call in sub-calls of at most frequency_capacity
    # records; one sub-call per (1e8-record) call here
    for name, kw, query in (("NEXT-3 structured access", {"structured": True}, lambda s: s.structured()),
                            ("NEXT-2 non-uniform access frequency",
                             {"frequency": True, "frequency_capacity": min(N, 1 << 27)},
                             lambda s: s.frequency(20))):
        s = Session(prog.objects, prog.kinds, **kw)
        for _ in range(2):
            s.reset(); s.attribute(d_recs); query(s)
        torch.cuda.synchronize()
        ms = []
        for _ in range(reps):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            s.reset()
            e0.record(stream)
            s.attribute(d_recs)
            e1.record(stream)
            torch.cuda.synchronize()
            ms.append(e0.elapsed_time(e1))
        w0 = time.perf_counter()
        query(s)
        q_ms = (time.perf_counter() - w0) * 1e3
        m = float(np.median(ms))
        out[name] = {"attribute_with_pass_ms": m, "pass_ms": m - plain_attr_ms,
                     "records_per_s_pass": N / ((m - plain_attr_ms) / 1e3) if m > plain_attr_ms else None,
                     "pass_gbs_records_only": 16.0 * N / ((m - plain_attr_ms) / 1e3) / 1e9
                     if m > plain_attr_ms else None,
                     "query_ms": q_ms}
        s.close()
        del s
        torch.cuda.empty_cache()
    s = Session(prog.objects, prog.kinds)
    s.attribute(d_recs)
    s.object_stats()
    w0 = time.perf_counter()
    pairs = s.redundant_allocations(10)
    out["NEXT-1 redundant allocation"] = {"ms": (time.perf_counter() - w0) * 1e3, "pairs": len(pairs)}
    streams = assign_streams(prog.n_api, 8, 0)
    s.dependency_graph(streams)
    w0 = time.perf_counter()
    T, src, dst, lab = s.dependency_graph(streams)
    g_ms = (time.perf_counter() - w0) * 1e3
    w0 = time.perf_counter()
    s.patterns_topo(T)
    out["NEXT-4 multi-stream graph + Kahn"] = {
        "graph_and_levels_ms": g_ms, "patterns_topo_ms": (time.perf_counter() - w0) * 1e3,
        "streams": 8, "edges": int(src.shape[0]), "levels": int(T.max()) + 1 if T.size else 0}
    s.close()
    return out


def other_config(cfg, a, hbm, hbm_src):
    """One extra config at N=1: value, phases, roofline, parity (stats /
    reports / counters), and for C2 the NEXT rows."""
    import torch
    w = Workload(cfg)
    steps = max(3, min(a.steps, 10))
    m = measure(w, a, steps, max(2, min(a.warmup, 3)), use_graph=not a.no_graph)
    w.keep_shadow()
    touched = touched_words(w)
    out = {"workload": WORKLOADS[cfg], "records": w.N, "value": w.N / (m["ms_step"] / 1e3),
           "unit": "records/s", "ms_per_step": m["ms_step"], "steps": steps,
           "phases_ms": dict(zip(("reset", "attribute", "merge", "finalize"), map(float, m["phases"]))),
           "step_exec": "cuda_graph_replay" if m["graphed"] else "eager",
           "gpu_launches": m["launches"], "roofline": roofline(w, m, touched, hbm, hbm_src),
           "resident": not w.chunked}
    if not a.no_parity:
        out["parity"] = parity_check(w, full=False)
    if cfg == "C2" and not a.no_next:
        out["next"] = next_rows(w.prog, w.d_recs[:16 * w.n_local], float(m["phases"][1]))
    w.close()
    torch.cuda.empty_cache()
    return out


def main():
    global CONSUME
    a = args_()
    CONSUME = a.consume
    world, rank, local = world_env()
    if a.gpus > 1 and "WORLD_SIZE" not in os.environ and a.impl == "ours":
        sys.exit(relaunch(a))
    if a.dry_run:
        return dry_run(a)
    if a.impl == "reference":
        return reference_arm(a)
    if world != a.gpus:
        raise SystemExit(f"bench.py: WORLD_SIZE={world} but --gpus {a.gpus}")
    import torch
    import torch.distributed as dist
    torch.cuda.set_device(local)
    ranks = None
    if world > 1:
        os.environ.setdefault("NCCL_DEBUG", "INFO")   # communicator lines on stderr (rank evidence)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        t = torch.tensor([1, rank], dtype=torch.int64, device="cuda")
        dist.all_reduce(t)
        ranks = {"world": world, "backend": dist.get_backend(), "ranks_reporting": int(t[0]),
                 "nccl_version": ".".join(map(str, torch.cuda.nccl.version()))}
    w = Workload(a.config, a.records, rank, world, a.merge)
    if ranks is not None and w.sm is not None:
        ranks["symmetric_memory_peers"] = len(w.sm.peer_ptrs())
    m = measure(w, a, a.steps, a.warmup, clocks=True, use_graph=not a.no_graph)
    value = w.N / (m["ms_step"] / 1e3)
    w.keep_shadow()
    touched = touched_words(w)
    parity = None if a.no_parity else parity_check(w, full=(world == 1))
    if world > 1:   # every rank's verdict: all must hold the whole-trace results
        ok = torch.tensor([1 if (parity or {}).get("ok", True) else 0], device="cuda")
        dist.all_reduce(ok, op=dist.ReduceOp.MIN)
        if parity is not None:
            parity["all_ranks_ok"] = bool(int(ok))
    stats, ctr = w.s.object_stats()     # the whole trace's (before the e2e leg resets it)
    paths = w.s.path_stats()
    e2e = e2e_leg(w, a, a.e2e_steps or min(a.steps, 5))
    hbm, hbm_src = peaks()
    rl = roofline(w, m, touched, hbm, hbm_src)
    line = {
        "metric": METRIC, "value": value, "unit": "records/s", "n_gpus": world,
        "steps": a.steps, "warmup": a.warmup, "ms_per_step": m["ms_step"],
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "u32",
        "data": f"synthetic (tracegen {w.prog.name}, seed {w.prog.seed:#x}; records generated on the device)",
        "config": {"workload": WORKLOADS[a.config], "records": w.N, "objects": w.prog.n_obj,
                   "n_api": w.prog.n_api, "parallelism": f"record-range x{world}", "merge": w.merge_note,
                   "records_per_rank": w.n_local,
                   "residency": (f"streamed: {len(w.chunks)} chunks of <= {GEN_CHUNK} records generated on the "
                                 f"device per step, outside the timed events (value = records / sum of the "
                                 f"steps' reset + attribute + merge + finalize events)") if w.chunked
                   else "resident in HBM for the whole timed region",
                   "l2": f"inputs larger than L2 ({16 * w.n_local / 2**30:.2f} GiB of records per rank per step)",
                   "shadow_words": int(w.s.view.or_words), "touched_words": touched,
                   "finalize": ("reduce-and-clear (drgpum_set_finalize_consume): the step's finalize zeroes "
                                "the bitmap words it reduces and the next step's reset skips them; one "
                                "untimed plain step after the timed region restores the bitmaps for the "
                                "touched-word count and the parity digests") if CONSUME and not w.owned
                               else "plain (the reset clears the touched bitmaps)"},
        "phases_ms": dict(zip(("reset", "attribute", "merge", "finalize"), map(float, m["phases"]))),
        "roofline": rl,
        "parity": parity,
        "ranks": ranks,
        "e2e": e2e,
        "gpu_launches": m["launches"],
        "step_exec": "cuda_graph_replay" if m["graphed"] else f"eager ({w.graph_note})",
        "clocks": m["clocks"],
        "counters": {k: int(ctr[k]) for k in ctr.dtype.names},
        "attribution_paths_tiles": paths,
        "wall_s_device_region": m["wall"],
    }
    cpu = None
    if world == 1 and not a.no_cpu_baseline:
        from tracegen import gen_records
        sub, desc = oracle_sample(w.prog, a.cpu_sample)
        recs = gen_records(sub, 0, sub.n_records)
        tcpu = time_oracle(sub.objects, sub.kinds, recs)
        del recs
        cpu = {"value": sub.n_records / tcpu, "unit": "records/s", "cores": 1, "kind": "oracle",
               "sample": desc, "seconds": tcpu, "cpu": cpu_model(), "host_cores": os.cpu_count()}
    line["cpu_baseline"] = cpu
    w.close()
    if world == 1 and a.extra_configs:
        line["other_configs"] = {}
        for cfg in [c for c in a.extra_configs.split(",") if c in WORKLOADS and c != a.config]:
            try:
                line["other_configs"][cfg] = other_config(cfg, a, hbm, hbm_src)
            except Exception as e:   # noqa: BLE001 -- an extra must not lose the main line
                line["other_configs"][cfg] = {"error": f"{type(e).__name__}: {e}"}
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
