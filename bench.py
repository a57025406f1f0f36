#!/usr/bin/env python
"""Benchmark of the Fringe-SGC hot path on B200 (driver contract).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl fsgc|reference]
                    [--workload internet|pl2k|rmat22|pl10m|rmat26]

One STEP = one pass of the whole hot path (core matching + Venn diagrams +
fringe counting + 128-bit reduction, and for N>1 the one all-reduce) over
the workload's graph for all of its patterns.  Default workload: BASELINE.json
configs[1] -- k-tailed triangles k = 1..4 on the synthetic Internet-like graph
(124,651 vertices / 193,620 edges); the four patterns share the edge core and
are counted in ONE batched pass.

value       core matches / s, device-timed (CUDA events on the launching
            stream), graph resident in HBM, L2 flushed (256 MiB write) before
            every timed step; N>1: max over ranks.  core matches = core
            instances in the graph x patterns (edge core: m per pattern).
e2e         same metric through the public API from HOST buffers: pinned
            edge list -> fsgc_load_graph (H2D + CSR build on the GPU) ->
            fsgc_count -> counts on the host, every step.
roofline    dominant kernel (the core/Venn/fc kernel): algorithmic bytes per
            launch / its CUDA-event duration, against
            the measured HBM copy bandwidth (MEASURED_PEAKS.json).
cpu_baseline  the oracle (oracle/, unmodified) on a bounded sample of the
            same workload on the host cores, same unit.
--impl reference  the oracle as the reference arm (CPU), see DESIGN.md.
"""
import argparse
import json
import os
import random
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

METRIC = "count time (s) and core matches/s per pattern×graph at 1/2/4/8 B200"
UNIT = "core matches/s"

WORKLOAD_DESC = {
    "internet": "k-tailed triangles k=1..4 on synthetic Internet-like power-law graph, "
                "124,651 V / 193,620 E (BASELINE configs[1])",
    "pl2k": "tailed triangle on synthetic power-law graph 2,000 V / 10,000 E (configs[0])",
    "rmat22": "triangle, diamond and k-tailed triangles (k=1..4) on RMAT scale 22 (configs[2] graph)",
    "rmat16": "4-clique cores with 1-6 and a diamond core with 1 mixed fringe on RMAT scale 16 "
              "(configs[2] patterns; Table 1's rmat16.sym scale)",
    "pl10m": "Fig. 4 16-vertex/25-edge pattern on synthetic power-law graph, 10M edges (configs[3])",
    "rmat26": "triangle and k-tailed triangles (k=1..4) on RMAT scale 26, 1.07B raw / 1.05B "
              "distinct edges (configs[4] graph; patterns decomposed to the edge core)",
}


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--impl", default="fsgc", choices=["fsgc", "reference"])
    ap.add_argument("--workload", default="internet", choices=list(WORKLOAD_DESC))
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-budget", type=float, default=12.0, help="seconds of oracle work")
    return ap.parse_args()


# ------------------------------------------------------------------ helpers

class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region."""
    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}",
                 "--format=csv,noheader,nounits", "-lms", "50"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for ln in self.proc.stdout:
            self.lines.append(ln.strip())

    def stop(self):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        self.t.join(timeout=2)
        sm, smax, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            parts = [x.strip() for x in ln.split(",")]
            if len(parts) < 8:
                continue
            try:
                sm.append(float(parts[0]))
                smax.append(float(parts[1]))
            except ValueError:
                continue
            for nm, v in zip(names, parts[4:8]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None,
                "sm_max_mhz": max(smax) if smax else None,
                "reasons": sorted(reasons), "samples": len(sm)}


def measured_peaks():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(path):
        d = json.load(open(path))
        return d.get("hbm_gbs", 6650.0), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md: 6.65 TB/s)"


def ncu_traffic(workload, kernel):
    """dram__bytes_read + dram__bytes_write per launch of `kernel` from the
    committed `ncu --set full` summary (profiles/ncu_summary.json), or None."""
    path = os.path.join(ROOT, "profiles", "ncu_summary.json")
    if not os.path.exists(path):
        return None
    d = json.load(open(path)).get(workload, {}).get("kernels", {})
    for k, v in d.items():
        if kernel.startswith(k):
            return v.get("dram_bytes_per_launch")
    return None


def load_workload(name, device):
    from inputs import workload_edges
    from inputs.patterns import CONFIG_PATTERNS, PATTERNS
    if name in ("rmat16", "rmat22", "rmat26"):
        n, e = workload_edges(name, device=device)
    else:
        n, e = workload_edges(name)
    pats = [PATTERNS[x] for x in CONFIG_PATTERNS[name]]
    return n, e, pats


# ------------------------------------------------------------------ oracle arm

def oracle_prepare(n, edges, pats):
    """The oracle's own graph (degree-ordered CSR by definition) and pattern
    decompositions, built once outside the timed sample."""
    import oracle
    offs, adj, _ = oracle.degree_ordered_csr(n, edges)
    gadj = oracle.csr_to_adjacency(offs, adj)
    decs = [(P, list(oracle.decompose(P.n, P.edges, P.core).core)) for P in pats]
    return gadj, decs


def oracle_sample(prep, budget_s, seed=0, sample=None):
    """Run the unmodified oracle (core+fringe mode, per root vertex, no
    symmetry breaking) on root vertices in a seeded random order until
    ``budget_s`` seconds are spent (or on exactly ``sample`` vertices).
    Returns (core instances processed, seconds, vertices)."""
    import oracle
    gadj, decs = prep
    verts = list(range(len(gadj)))
    random.Random(seed).shuffle(verts)
    if sample is not None:
        verts = verts[:sample]
    maps = 0.0
    done = 0
    t0 = time.perf_counter()
    for r in verts:
        for P, cs in decs:
            oracle.root_raw_sum(gadj, P.n, P.edges, P.core, cs[0], r)
            if len(cs) == 2:       # edge core: deg(r) core maps rooted at r, 2 per instance
                maps += len(gadj[r]) / 2.0
            elif len(cs) == 1:
                maps += 1
        done += 1
        if sample is None and time.perf_counter() - t0 >= budget_s:
            break
    return maps, time.perf_counter() - t0, done


def run_reference(args, rank, world):
    if rank != 0:
        return
    n, e, pats = load_workload(args.workload, None)
    if hasattr(e, "cpu"):
        e = e.cpu().numpy()
    # size one step so the whole run stays within a few minutes
    prep = oracle_prepare(n, e, pats)
    step_budget = max(0.2, 120.0 / max(1, args.steps + args.warmup))
    _, _, nv = oracle_sample(prep, step_budget, seed=99)
    nv = max(1, nv)
    vals, secs = [], []
    for s in range(args.warmup + args.steps):
        maps, dt, _ = oracle_sample(prep, 0, seed=s, sample=nv)
        if s >= args.warmup:
            vals.append(maps)
            secs.append(dt)
    value = sum(vals) / sum(secs)
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * sum(secs) / len(secs),
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "python-int",
        "data": "synthetic",
        "config": {"workload": WORKLOAD_DESC[args.workload], "patterns": [p.name for p in pats]},
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": 1, "kind": "oracle",
                         "sample": f"{nv} seeded random root vertices per step x {len(pats)} patterns"},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------ GPU arm

def main():
    args = parse()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        run_reference(args, rank, world)
        return

    import numpy as np
    import torch
    import torch.distributed as dist
    # FSGC_BENCH_BACKEND=gloo (testing the N>1 path on a 1-GPU box: ranks
    # share the visible GPUs round-robin); the product path is NCCL
    backend = os.environ.get("FSGC_BENCH_BACKEND", "nccl")
    local = local % max(1, torch.cuda.device_count())
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        if backend == "nccl":
            dist.init_process_group("nccl", rank=rank, world_size=world, device_id=dev)
        else:
            dist.init_process_group(backend, rank=rank, world_size=world)
    import paper_conf_sc_bradleyab25_b200 as F

    n, e, pats = load_workload(args.workload, dev)
    if isinstance(e, np.ndarray):
        e_host = torch.from_numpy(np.ascontiguousarray(e.astype(np.int32))).pin_memory()
        e_dev = e_host.to(dev)
    else:
        e_dev = e.contiguous()
        e_host = e_dev.cpu().pin_memory()
    g = F.fsgc_load_graph(e_dev, n)
    cps = [F.compile_named(P) for P in pats]

    # core instances per step (graph property, untimed): degree filter off
    probe = F.fsgc_count(g, cps, no_degree_filter=True, shard_index=0, shard_count=1)
    core_matches = sum(r.core_matches for r in probe)

    stream = torch.cuda.current_stream()
    if world > 1:
        def step():
            return F.fsgc_count_distributed(g, cps)
        replay = None
        plan = None
    else:
        # one CUDA graph per step: workspace zeroing, every kernel of every
        # pass, and the copy of the raw 128-bit results into pinned memory
        plan = F.fsgc_plan_create(g, cps)
        side = torch.cuda.Stream()
        side.wait_stream(stream)
        with torch.cuda.stream(side):
            plan.enqueue(side)
        side.synchronize()
        cg = torch.cuda.CUDAGraph()
        with torch.cuda.graph(cg):
            plan.enqueue(torch.cuda.current_stream())
        torch.cuda.synchronize()

        def step():
            cg.replay()
            torch.cuda.current_stream().synchronize()
            return plan.decode()
        replay = cg

    flush = torch.empty(64 * 1024 * 1024, dtype=torch.int32, device=dev)   # 256 MiB > 126 MB L2
    for _ in range(args.warmup):
        res = step()
    counts = [r.count for r in res]
    ref = F.fsgc_count(g, cps)                       # the synchronous API agrees
    assert [r.count for r in ref] == counts, (counts, [r.count for r in ref])
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()

    sampler = ClockSampler(local)
    sampler.start()
    time.sleep(0.2)
    ev0 = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    ev1 = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    kms, ams, launches = [], [], 0
    for s in range(args.steps):
        flush.fill_(s)
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        if replay is not None:
            ev0[s].record(stream)
            replay.replay()
            ev1[s].record(stream)
            torch.cuda.synchronize()
            res = plan.decode()
        else:
            ev0[s].record(stream)
            res = step()
            ev1[s].record(stream)
            torch.cuda.synchronize()
        assert [r.count for r in res] == counts
        passes = {}
        for r in res:
            passes[r.pass_index] = r
        kms.append({k: r.kernel_ms for k, r in passes.items()})
        ams.append({k: r.aux_ms for k, r in passes.items()})
        launches += sum(r.kernel_launches for r in passes.values())
    step_ms = [a.elapsed_time(b) for a, b in zip(ev0, ev1)]
    clocks = sampler.stop()
    total_ms = sum(step_ms)
    pass_ids = sorted(kms[0].keys())
    kms_sum = {k: sum(x[k] for x in kms) for k in pass_ids}
    ams_sum = {k: sum(x[k] for x in ams) for k in pass_ids}
    if world > 1:
        t = torch.tensor([total_ms] + [kms_sum[k] for k in pass_ids] + [ams_sum[k] for k in pass_ids],
                         dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        vals = t.tolist()
        total_ms = vals[0]
        kms_sum = {k: vals[1 + i] for i, k in enumerate(pass_ids)}
        ams_sum = {k: vals[1 + len(pass_ids) + i] for i, k in enumerate(pass_ids)}
    ms_per_step = total_ms / args.steps
    value = core_matches / (ms_per_step / 1e3)
    kind_of = {r.pass_index: r.pass_kind for r in res}

    # ---- roofline of the dominant kernel: algorithmic
    # bytes per launch / CUDA-event duration, against the measured HBM peak
    offs, adj_h, _ = g.download()
    deg = np.diff(offs).astype(np.int64)
    rows = np.repeat(np.arange(n, dtype=np.int64), deg)
    up = adj_h.astype(np.int64) > rows
    out = np.bincount(rows[up], minlength=n).astype(np.float64)
    indeg = deg - out
    m = g.m
    share = 1.0 / world
    # support pass: wedge-hash part -- per in-entry
    # (a, b) of a table middle b: 4 B a + 4 B rev + 24 B split/oofs/offs of a,
    # 4 B per tail element c > b of N+(a) streamed, 4 B per N+(b) entry staged
    # (+ its c(b, x) flush), 8 B per triangle (the c(a, c) reduction); merge
    # part -- per heavy-middle edge 40 B + 4 B per merged out-list entry
    CAP = 4096
    a_o = rows[up]
    b_o = adj_h[up].astype(np.int64)
    oofs_h = np.concatenate([[0], np.cumsum(out)]).astype(np.int64)
    tail = out[a_o] - (np.arange(len(a_o), dtype=np.int64) - oofs_h[a_o]) - 1
    ob = out[b_o]
    light = (ob >= 1) & (ob <= CAP)
    heavy = ob > CAP
    tri = 0
    if plan is not None and plan.support() is not None:
        tri = int(plan.support().to(torch.int64).sum().item()) // 3
    mid = (out >= 1) & (out <= CAP) & (indeg >= 1)
    sup_bytes = (32.0 * float(light.sum()) + 4.0 * float(tail[light].sum()) + 8.0 * float(out[mid].sum())
                 + 8.0 * tri + 40.0 * float(heavy.sum()) + 4.0 * float((out[a_o] + ob)[heavy].sum()))
    # fc pass: per root edge 8 B (u,v) + 32 B (4 offsets) + 4 B support
    fc_bytes = 44.0 * m * share
    # general / triangle core passes: compulsory graph bytes (CSR + oriented
    # view + supports read once) -- these kernels are latency/ALU bound
    graph_bytes = (8.0 * 2 * m + 8.0 * (n + 1) + 8.0 * m + 4.0 * m + 16.0 * n) * share
    names = {0: "vertex_core_kernel", 1: "edge_fc_kernel (Venn + Sec. 3.1 fc, lane per root edge)",
             2: "core_kernel (general core: DFS + min-list Venn + fc)",
             3: "tri_core_kernel (triangle core: listing + Venn + fc)"}
    kernels = []
    for k in pass_ids:
        kind = kind_of[k]
        byts = fc_bytes if kind == 1 else (8.0 * (n + 1) * share if kind == 0 else graph_bytes)
        kernels.append((names[kind] + f" [pass {k}]", byts, kms_sum[k] / args.steps))
        if kind != 0:
            kernels.append((f"support_kernel (per-edge |N(u)&N(v)| by oriented listing) [pass {k}]",
                            sup_bytes, ams_sum[k] / args.steps))
    kernels.sort(key=lambda kk: -kk[2])
    peak, peak_src = measured_peaks()
    def roof(name, byts, ms):
        traffic = ncu_traffic(args.workload, name)
        ach = byts / (ms / 1e3) / 1e9 if ms > 0 else 0.0
        return {"bound": "hbm", "achieved": ach, "peak": peak, "unit": "GB/s", "frac": ach / peak,
                "traffic": traffic, "kernel": name, "kernel_ms": ms,
                "algorithmic_bytes_per_launch": byts, "peak_source": peak_src}

    # ---- e2e through the public API from pinned host buffers
    e2e = None
    if not args.no_e2e:
        h2d = e_host.numel() * e_host.element_size()
        d2h = 36 + 16 * 32 + 8
        tms = []
        for s in range(3 + min(args.steps, 50)):
            flush.fill_(s)
            torch.cuda.synchronize()
            if world > 1:
                dist.barrier()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(stream)
            g2 = F.fsgc_load_graph(e_host, n)
            r2 = F.fsgc_count_distributed(g2, cps) if world > 1 else F.fsgc_count(g2, cps)
            b.record(stream)
            torch.cuda.synchronize()
            assert [x.count for x in r2] == counts
            g2.free()
            if s >= 3:
                tms.append(a.elapsed_time(b))
        et = sum(tms)
        if world > 1:
            t = torch.tensor([et], dtype=torch.float64, device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            et = t.item()
        e2e = {"value": core_matches / (et / len(tms) / 1e3), "unit": UNIT,
               "h2d_bytes_per_step": int(h2d), "d2h_bytes_per_step": int(d2h),
               "ms_per_step": et / len(tms)}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        e_np = e if isinstance(e, np.ndarray) else e.cpu().numpy()
        maps, secs, nv = oracle_sample(oracle_prepare(n, e_np, pats), args.cpu_budget)
        cpu = {"value": maps / secs, "unit": UNIT, "cores": 1, "kind": "oracle",
               "sample": f"{nv} seeded random root vertices x {len(pats)} patterns "
                         f"({secs:.1f} s, per-root core+fringe oracle, 1 Python thread)"}

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "u128", "data": "synthetic",
            "config": {"workload": WORKLOAD_DESC[args.workload], "patterns": [p.name for p in pats],
                       "graph": {"n": n, "m": m, "max_degree": g.max_degree},
                       "core_matches_per_step": core_matches,
                       "count_time_s": ms_per_step / 1e3,
                       "counts": {p.name: str(c) for p, c in zip(pats, counts)},
                       "l2": "flushed before every timed step (256 MiB write)",
                       "parallelism": f"{world} GPU(s): graph replicated, root-edge chunks dealt "
                                      f"round-robin, 1 all-reduce of 128-bit partials"},
            "gpu_launches": launches,
            "roofline": roof(*kernels[0]),
            "roofline_other_kernels": [roof(*k) for k in kernels[1:]],
            "clocks": clocks,
            "e2e": e2e,
            "cpu_baseline": cpu,
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
