#!/usr/bin/env python
"""Benchmark: DrGPUM per-access attribution on B200 (BASELINE.json metric).

One *step* is one pass of the whole hot path over the workload's records,
already resident in HBM: reset the shadow (bitmaps / hit rows / first / last /
counters), attribute every record (A1-A5), [merge across ranks], and the
per-object reductions + pattern classification (A6-A7), all on the device.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config C2]
  python bench.py --impl reference ...   # the CPU oracle as the reference arm

N>1 runs under torchrun (one rank per GPU, NCCL): rank r attributes records
[r*N/P, (r+1)*N/P) of the same trace, then the one exchange step merges the
shadows (paper_conf_asplos_linzs23_b200/parallel.py) -- strong scaling.
Rank 0 prints ONE JSON line.
"""
import argparse
import json
import os
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
    "C5": "C5 scaling sweep (BASELINE configs[4]): 1.6e10 records over 1M objects, streamed through HBM "
          "in 2^30-record chunks generated on the device",
}
# configs whose records are generated on the device (tracegen/gen.cu) rather
# than on the host; traces above RESIDENT_BYTES are streamed in GEN_CHUNK chunks
DEVICE_GEN = ("C3", "C4", "C5")
GEN_CHUNK = 1 << 30
RESIDENT_BYTES = 96 << 30
FALLBACK_HBM_GBS = 6650.0


def args_():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="C2", choices=sorted(WORKLOADS))
    ap.add_argument("--records", type=int, default=None, help="override the record count")
    ap.add_argument("--e2e-steps", type=int, default=None)
    ap.add_argument("--merge", default="owned", choices=["owned", "peers", "nccl"],
                    help="N>1 exchange step over torch symmetric memory (NVLink P2P): owned = "
                         "drgpum_merge_peers_owned + per-rank finalize of its objects + "
                         "drgpum_gather_peers; peers = drgpum_merge_peers (every rank gets the "
                         "whole merged shadow, finalizes everything); nccl = all-to-all + "
                         "merge_or + all-gather")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-next", action="store_true", help="skip the SURVEY §8(f) NEXT-row timings")
    ap.add_argument("--no-graph", action="store_true",
                    help="time eager launches instead of CUDA-graph replays of the step")
    ap.add_argument("--cpu-sample", type=int, default=None,
                    help="records in the oracle's timed sample (default: whole workload up to 1e8; "
                         "2e7 for the device-generated configs)")
    ap.add_argument("--e2e-sample", type=int, default=1 << 26,
                    help="records of the host-buffer (e2e) leg for the device-generated configs")
    ap.add_argument("--ref-sample", type=int, default=8_000_000,
                    help="records per reference-arm step")
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
    """--impl reference: the CPU oracle, timed on the host cores, on our config."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    from tracegen import build_config, gen_records
    prog = build_config(a.config, **({"n_records": a.records} if a.records else {}))
    m = min(a.ref_sample, prog.n_records)
    recs = gen_records(prog, 0, m)
    for _ in range(a.warmup):
        time_oracle(prog.objects, prog.kinds, recs)
    ts = [time_oracle(prog.objects, prog.kinds, recs) for _ in range(a.steps)]
    t = sum(ts) / len(ts)
    v = m / t
    sample = (f"first {m} records of the {prog.n_records}-record {a.config} trace per step "
              f"(prefix-timed; oracle = O1 std::map replay, single thread)")
    print(json.dumps({
        "impl": "reference", "metric": METRIC, "value": v, "unit": "records/s",
        "n_gpus": a.gpus, "steps": a.steps, "warmup": a.warmup, "ms_per_step": t * 1e3,
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "u32",
        "data": "synthetic", "config": {"workload": WORKLOADS[a.config], "records": m},
        "cpu_baseline": {"value": v, "unit": "records/s", "cores": 1, "kind": "oracle",
                         "sample": sample, "cpu": cpu_model()},
        "e2e": {"value": v, "unit": "records/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }), flush=True)


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
    for name, kw, query in (("NEXT-3 structured access", {"structured": True}, lambda s: s.structured()),
                            ("NEXT-2 non-uniform access frequency", {"frequency": True},
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
    return out


def main():
    a = args_()
    if a.impl == "reference":
        return reference_arm(a)
    import torch
    import torch.distributed as dist
    from paper_conf_asplos_linzs23_b200 import Session
    from paper_conf_asplos_linzs23_b200.parallel import shard_range, merge_session
    from tracegen import build_config, gen_records

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    prog = build_config(a.config, **({"n_records": a.records} if a.records else {}))
    N = prog.n_records
    lo, hi = shard_range(N, rank, world)
    n_local = hi - lo
    devgen = a.config in DEVICE_GEN
    chunked = devgen and 16 * n_local > RESIDENT_BYTES
    recs = None
    if not devgen:
        recs = gen_records(prog, lo, hi)
        d_recs = torch.from_numpy(recs.view(np.uint8)).cuda()
        chunks = [(0, n_local)]
    else:
        # device generation (never timed): the whole shard resident, or one
        # GEN_CHUNK buffer refilled per chunk inside every step
        from tracegen.device import DeviceProgram
        dp = DeviceProgram(prog)
        gen_chunks = [(c, min(c + GEN_CHUNK, n_local)) for c in range(0, n_local, GEN_CHUNK)]
        d_recs = torch.empty(16 * (GEN_CHUNK if chunked else n_local), dtype=torch.uint8, device="cuda")
        if chunked:
            chunks = gen_chunks
        else:
            for c0, c1 in gen_chunks:
                dp.gen(lo + c0, lo + c1, out=d_recs[16 * c0:16 * c1])
            chunks = [(0, n_local)]
        torch.cuda.synchronize()
    sm, merge_note = None, "none (1 rank)"
    if world > 1 and a.merge in ("peers", "owned"):
        from paper_conf_asplos_linzs23_b200.parallel import SymmetricMerge
        try:
            sm = SymmetricMerge()
            s = Session(prog.objects, prog.kinds, workspace_alloc=sm.alloc)
            merge_note = ("drgpum_merge_peers_owned + finalize of the owned objects + drgpum_gather_peers "
                          "over torch symmetric memory (NVLink P2P)" if a.merge == "owned" else
                          "drgpum_merge_peers over torch symmetric memory (one kernel per rank, NVLink P2P)")
        except Exception as e:   # symmetric memory unavailable: the NCCL exchange instead, said so
            sm = None
            merge_note = f"NCCL all_to_all + merge_or + all_gather (symmetric memory unavailable: {e})"
    if sm is None:
        s = Session(prog.objects, prog.kinds)
        if world > 1 and a.merge == "nccl":
            merge_note = "NCCL all_to_all + merge_or + all_gather"
    stream = torch.cuda.current_stream()
    owned = sm is not None and a.merge == "owned"

    def do_merge():
        if world > 1:
            if owned:
                sm.merge_owned(s)
            elif sm is not None:
                sm.merge(s)
            else:
                merge_session(s)

    def do_finalize():
        s.finalize()
        if owned:
            sm.gather(s)

    def barrier():
        if world > 1:
            dist.barrier()

    def one_step(src, ev=None):
        """ev: per-phase event pairs [reset, attribute, merge, finalize]; the
        attribute pair is per chunk (generation of a chunk lies outside it)."""
        if ev: ev["reset"][0].record(stream)
        s.reset()
        if ev: ev["reset"][1].record(stream)
        for k, (c0, c1) in enumerate(chunks):
            if chunked:
                dp.gen(lo + c0, lo + c1, out=src)
            if ev: ev["attr"][k][0].record(stream)
            s.attribute(src[:16 * (c1 - c0)])
            if ev: ev["attr"][k][1].record(stream)
        if ev: ev["merge"][0].record(stream)
        do_merge()
        if ev: ev["merge"][1].record(stream)
        if ev: ev["fin"][0].record(stream)
        do_finalize()
        if ev: ev["fin"][1].record(stream)

    def events():
        E = lambda: (torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
        return {"reset": E(), "attr": [E() for _ in chunks], "merge": E(), "fin": E()}

    def phases(ev):   # ms
        el = lambda e: e[0].elapsed_time(e[1])
        return [el(ev["reset"]), sum(el(e) for e in ev["attr"]), el(ev["merge"]), el(ev["fin"])]

    for _ in range(a.warmup):
        one_step(d_recs)
    torch.cuda.synchronize()
    l0 = s.launch_count()
    one_step(d_recs)
    graph_launches = s.launch_count() - l0   # kernels of the library per step

    # ---------------- device-resident timed region
    # Phase breakdown: eager launches with events between the phases.
    evs = [events() for _ in range(a.steps)]
    torch.cuda.synchronize()
    for k in range(a.steps):
        one_step(d_recs, evs[k])
    torch.cuda.synchronize()
    ph = np.array([phases(e) for e in evs])  # ms
    ph_mean = ph.mean(axis=0)
    # The step itself: one CUDA graph of the library's launches (reset,
    # attribute + range expansion, finalize), replayed K times -- the same
    # kernels without per-launch host gaps.  Multi-rank steps (NCCL merge)
    # run eagerly; chunked traces (generation between the chunks) are timed
    # as the sum of their phase events.
    use_graph = world == 1 and not a.no_graph and not chunked
    if use_graph:
        graph = torch.cuda.CUDAGraph()
        with torch.cuda.graph(graph):
            one_step(d_recs)
        for _ in range(a.warmup):
            graph.replay()
        torch.cuda.synchronize()
    clk = ClockSampler(local)
    time.sleep(0.3)
    t_start = torch.cuda.Event(enable_timing=True)
    t_end = torch.cuda.Event(enable_timing=True)
    launches0 = s.launch_count()
    barrier()
    torch.cuda.synchronize()
    wall0 = time.perf_counter()
    t_start.record(stream)
    tev = [events() for _ in range(a.steps)] if chunked else None
    for k in range(a.steps):
        if use_graph:
            graph.replay()
        else:
            one_step(d_recs, tev[k] if chunked else None)
    t_end.record(stream)
    torch.cuda.synchronize()
    barrier()
    wall_dev = time.perf_counter() - wall0
    # graph replays do not pass through the library's launch counter: count
    # the captured launches once per replay
    launches = (s.launch_count() - launches0) if not use_graph else graph_launches * a.steps
    ms_total = t_start.elapsed_time(t_end)
    if chunked:   # generation excluded: the steps are the sum of their phases
        ms_total = float(sum(sum(phases(e)) for e in tev))
    if world > 1:
        t = torch.tensor([ms_total] + ph_mean.tolist(), dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms_total = float(t[0])
        ph_mean = t[1:].cpu().numpy()
    ms_step = ms_total / a.steps
    value = N / (ms_step / 1e3)

    # calibration: attainable streaming-read bandwidth over the same record
    # buffer (a torch reduction, not part of the path), so that the
    # attribution can also be read as a fraction of "just reading the records"
    cal = None
    if not chunked:
        v64 = d_recs.view(torch.int64)
        for _ in range(3):
            v64.sum()
        c0, c1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        c0.record(stream)
        for _ in range(5):
            v64.sum()
        c1.record(stream)
        torch.cuda.synchronize()
        rd_ms = c0.elapsed_time(c1) / 5
        cal = {"read_gbs": 16.0 * n_local / (rd_ms / 1e3) / 1e9, "ms": rd_ms,
               "how": "torch.sum over the resident record buffer viewed as int64 (read-only stream)"}

    # touched shadow words (algorithmic write-back of A3/A4) of THIS rank's
    # attribution: at N>1 the merged shadow is not what the rank's kernel
    # wrote, so the shard is attributed once more alone, counted, and the
    # merged step re-run (collectively) for the stats below
    if world > 1:
        s.reset()
        for c0, c1 in chunks:
            if chunked:
                dp.gen(lo + c0, lo + c1, out=d_recs)
            s.attribute(d_recs[:16 * (c1 - c0)])
        touched = int(torch.count_nonzero(s.or_words()).item())
        barrier()
        one_step(d_recs)
    else:
        touched = int(torch.count_nonzero(s.or_words()).item())
    stats, ctr = s.object_stats()
    paths = s.path_stats()

    # ---------------- end-to-end through the public API with HOST buffers
    e2e_steps = a.e2e_steps or min(a.steps, 10)
    n_e2e = n_local if not devgen else min(n_local, a.e2e_sample)
    pinned = torch.empty(n_e2e * 16, dtype=torch.uint8, pin_memory=True)
    pinned.numpy()[:] = (recs if recs is not None else gen_records(prog, lo, lo + n_e2e)).view(np.uint8)
    for _ in range(2):
        s.reset(); s.attribute(pinned); s.object_stats(); s.patterns()
    torch.cuda.synchronize()
    barrier()
    w0 = time.perf_counter()
    for _ in range(e2e_steps):
        s.reset()
        s.attribute(pinned)                 # drgpum_trace_attribute_host: H2D inside
        do_merge()
        if owned:
            do_finalize()
        st_h, ctr_h = s.object_stats()      # D2H of the result
        rep_h = s.patterns()
    torch.cuda.synchronize()
    e2e_s = (time.perf_counter() - w0) / e2e_steps
    if world > 1:
        t = torch.tensor([e2e_s], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        e2e_s = float(t[0])
    clocks = clk.stop()
    nxt = None
    if world == 1 and not a.no_next and not devgen:
        nxt = next_rows(prog, d_recs, float(ph_mean[1]))

    if rank != 0:
        dist.destroy_process_group()
        return
    hbm, hbm_src = peaks()
    attr_ms = float(ph_mean[1])
    alg_bytes = 16.0 * n_local + 4.0 * touched
    achieved = alg_bytes / (attr_ms / 1e3) / 1e9
    traffic = None
    tfile = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tfile):
        try:
            t = json.load(open(tfile)).get(a.config)
            traffic = None if t is None else int(t["bytes_per_launch"])
        except Exception:
            traffic = None

    cpu = None
    if world == 1 and not a.no_cpu_baseline:
        m = min(a.cpu_sample or (20_000_000 if devgen else N), N, 100_000_000)
        tcpu = time_oracle(prog.objects, prog.kinds, recs[:m] if recs is not None else gen_records(prog, 0, m))
        cpu = {"value": m / tcpu, "unit": "records/s", "cores": 1, "kind": "oracle",
               "sample": (f"{'all' if m == N else 'first'} {m} records of the {a.config} trace, "
                          f"one pass: load + attribute + stats + patterns (O1, single thread)"),
               "seconds": tcpu, "cpu": cpu_model(), "host_cores": os.cpu_count()}

    line = {
        "metric": METRIC, "value": value, "unit": "records/s", "n_gpus": world,
        "steps": a.steps, "warmup": a.warmup, "ms_per_step": ms_step,
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "u32",
        "data": f"synthetic (tracegen {prog.name}, seed {prog.seed:#x})",
        "config": {"workload": WORKLOADS[a.config], "records": N, "objects": prog.n_obj,
                   "n_api": prog.n_api, "parallelism": f"record-range x{world}", "merge": merge_note,
                   "l2": f"inputs larger than L2 ({16 * N / 2**30:.2f} GiB of records streamed per step)",
                   "shadow_words": int(s.view.or_words), "touched_words": touched},
        "phases_ms": {"reset": float(ph_mean[0]), "attribute": attr_ms,
                      "merge": float(ph_mean[2]), "finalize": float(ph_mean[3])},
        "roofline": {"bound": "hbm", "achieved": achieved, "peak": hbm, "unit": "GB/s",
                     "frac": achieved / hbm, "traffic": traffic,
                     "kernel": "drgpum_trace_attribute (attribute_kernel + range_expand_kernel)",
                     "algorithmic_bytes": alg_bytes,
                     "bytes_rule": "16 B per record + 4 B per touched shadow word",
                     "peak_source": hbm_src},
        "calibration": None if cal is None else dict(cal, attribution_frac_of_read=cal["read_gbs"] and
                                                     (16.0 * n_local / (attr_ms / 1e3) / 1e9) / cal["read_gbs"]),
        "cpu_baseline": cpu,
        "e2e": {"value": n_e2e * world / e2e_s, "unit": "records/s", "h2d_bytes_per_step": 16 * n_e2e,
                "records_per_rank": n_e2e,
                "d2h_bytes_per_step": int(prog.n_obj * (56 + 32) + 40),
                "ms_per_step": e2e_s * 1e3,
                "path": "Session.attribute(pinned host tensor) -> drgpum_trace_attribute_host; "
                        "object_stats + patterns (D2H)"},
        "gpu_launches": launches,
        "step_exec": "cuda_graph_replay" if use_graph else "eager",
        "clocks": clocks,
        "counters": {k: int(ctr[k]) for k in ctr.dtype.names},
        "attribution_paths_tiles": paths,
        "wall_s_device_region": wall_dev,
        "next": nxt,
    }
    print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
