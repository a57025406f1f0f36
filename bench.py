#!/usr/bin/env python
"""Benchmark of the Fringe-SGC hot path on B200 (driver contract).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl fsgc|reference]
                    [--workload rmat26|internet|pl2k|rmat22|rmat16|pl10m|...]
                    [--no-e2e] [--no-cpu-baseline] [--no-per-config]

Headline workload (default): BASELINE.json configs[4], the largest
configuration that fits one GPU -- triangle cores with fringes on RMAT scale
26 (2^26 vertices, 1.07e9 raw / 1.05e9 distinct edges, 4.9e10 triangles), the
core forced to the triangle (R13).  All its patterns share the
triangle core, so one STEP = the per-edge support pass + ONE triangle-core
listing pass (core matching + Venn diagrams + fringe counting + 128-bit
reduction; for N>1 the support all-reduce and the one 128-bit all-reduce).

value       core matches / s, device-timed (CUDA events on the launching
            stream), graph resident in HBM, L2 flushed (256 MiB write) before
            every timed step; N>1: max over ranks.  core matches = the
            DISTINCT core instances the step enumerates (each triangle once,
            however many patterns share the pass).  ``edges_per_s`` = m / step
            time (the paper's Sec. 6 throughput).
e2e         same metric through the public API from HOST buffers: pinned
            edge list -> fsgc_load_graph (H2D + CSR build) -> fsgc_count ->
            counts on the host, every step.
roofline    dominant kernel: algorithmic bytes per launch (DESIGN.md Sec. 5,
            from the graph's own degree statistics) / its CUDA-event duration,
            against the measured HBM copy bandwidth (MEASURED_PEAKS.json).
per_config  configs[0..3] (and the RMAT-26 edge-core decomposition): count
            time of the batched pass and of every pattern alone, core
            matches/s and edges/s, per pattern x graph.
cpu_baseline  the oracle (oracle/cfast.py, C with OpenMP on all host cores,
            unmodified) on a bounded sample of the same workload, same unit.
--impl reference  the oracle as the reference arm.
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
    "rmat26": "triangle cores with fringes (core forced to the triangle: triangle, 1..4 tails on one "
              "vertex, tails on two vertices, a wedge fringe) on RMAT scale 26, 1.07B raw / 1.05B distinct "
              "edges (BASELINE configs[4])",
    "rmat26-edge": "triangle and k-tailed triangles (k=1..4) decomposed to the edge core (Sec. 3.4 "
                   "heuristic) on RMAT scale 26 (configs[4] graph)",
    "internet": "k-tailed triangles k=1..4 on synthetic Internet-like power-law graph, "
                "124,651 V / 193,620 E (BASELINE configs[1])",
    "pl2k": "tailed triangle on synthetic power-law graph 2,000 V / 10,000 E (configs[0])",
    "rmat22": "triangle, diamond and k-tailed triangles (k=1..4) on RMAT scale 22 (configs[2] graph)",
    "rmat22-tri": "the configs[4] triangle-core set (core forced to the triangle, 7 patterns) on RMAT scale 22 "
                  "(configs[2] graph)",
    "rmat16": "4-clique cores with 1-6 and a diamond core with 1 mixed fringe on RMAT scale 16 "
              "(configs[2] patterns; Table 1's rmat16.sym scale)",
    "pl10m": "Fig. 4 16-vertex/25-edge pattern on synthetic power-law graph, 10M edges (configs[3])",
}

# per_config block of the default run: (workload, reps per timing)
PER_CONFIG = [("pl2k", 20), ("internet", 20), ("rmat16", 2), ("rmat22", 3), ("rmat22-tri", 2), ("pl10m", 3),
              ("rmat26-edge", 2)]


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="fsgc", choices=["fsgc", "reference"])
    ap.add_argument("--workload", default="rmat26", choices=list(WORKLOAD_DESC))
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-per-config", action="store_true")
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--cpu-budget", type=float, default=15.0, help="seconds of oracle work")
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


def ncu_r02(workload):
    """per-kernel ncu numbers of this round's capture (profiles/ncu_r02_summary.json,
    written by scripts/ncu_r02_summary.py from an ncu run of the same build)"""
    path = os.path.join(ROOT, "profiles", "ncu_r02_summary.json")
    if not os.path.exists(path):
        return {}
    return json.load(open(path)).get(workload, {}).get("kernels", {})


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


def graph_key(name):
    return "rmat26" if name.startswith("rmat26") else "rmat22" if name.startswith("rmat22") else name


def load_workload(name, device):
    """(n, edges, patterns): RMAT graphs generated with torch on ``device``
    (int32 tensor), the others with numpy (int64 array)."""
    from inputs import workload_edges
    from inputs.patterns import CONFIG_PATTERNS, PATTERNS
    gk = graph_key(name)
    if gk.startswith("rmat"):
        n, e = workload_edges(gk, device=device if device is not None else "cpu")
    else:
        n, e = workload_edges(gk)
    return n, e, [PATTERNS[x] for x in CONFIG_PATTERNS[name]]


def simple_csr_torch(n, e):
    """The simple graph of an edge list as a CSR with sorted adjacency lists
    and ORIGINAL ids (loops dropped, duplicates merged) -- plain torch
    sort/unique on the edge tensor's device, then to host numpy.  Input
    preparation of the oracle's CPU baseline for graphs too large for numpy
    (the oracle's own oracle.cfast.simple_csr builds the same arrays)."""
    import torch
    a = e[:, 0].to(torch.int64)
    b = e[:, 1].to(torch.int64)
    ok = a != b
    a, b = a[ok], b[ok]
    key = torch.unique(torch.cat([a * n + b, b * n + a]))
    src = key // n
    offs = torch.zeros(n + 1, dtype=torch.int64, device=key.device)
    offs[1:] = torch.cumsum(torch.bincount(src, minlength=n), 0)
    return offs.cpu().numpy(), (key % n).to(torch.int32).cpu().numpy()


def host_csr(n, e):
    import numpy as np
    if isinstance(e, np.ndarray):
        from oracle.cfast import simple_csr
        return simple_csr(n, e)
    return simple_csr_torch(n, e)


SAMPLE_MAX_DEG = 64    # sampled roots: degree <= this (per-root oracle cost stays bounded on hub-heavy graphs)


def oracle_cpu_sample(csr, pats, budget_s, seed=0, max_deg=SAMPLE_MAX_DEG, nroots=None):
    """The unmodified C oracle (oracle.cfast.root_raw_sum_c: every core map
    with the root pattern vertex on the sampled graph vertices, explicit Venn,
    Listing 5; OpenMP on all host cores) on seeded random root vertices of
    degree <= max_deg, in batches until ``budget_s`` seconds are spent (or on
    exactly ``nroots`` roots).  Returns (core matches processed, seconds,
    roots, threads): core matches = core maps / |Aut(core)|, the unit of the
    GPU line."""
    import numpy as np
    import oracle
    from oracle.cfast import root_raw_sum_c
    offs, _ = csr
    n = len(offs) - 1
    deg = np.diff(offs)
    rng = np.random.default_rng(seed)
    cand = np.nonzero((deg >= 1) & (deg <= max_deg))[0]
    roots = rng.permutation(cand)[: (nroots if nroots is not None else 2_000_000)]
    threads = os.cpu_count() or 1
    decs = []
    for P in pats:
        dec = oracle.decompose(P.n, P.edges, P.core)
        cs = list(dec.core)
        rel = {v: i for i, v in enumerate(cs)}
        cedges = [(rel[x], rel[y]) for x, y in P.edges if x in rel and y in rel]
        decs.append((P, cs[0], oracle.automorphism_count(len(cs), cedges)))
    matches, done, t0 = 0.0, 0, time.perf_counter()
    batch = 4   # doubled per batch: the budget check stays fine-grained on hub-heavy graphs
    while done < len(roots):
        chunk = roots[done:done + batch]
        for P, pv, autc in decs:
            _, maps = root_raw_sum_c(csr, P.n, P.edges, P.core, pv, chunk, threads=threads)
            matches += maps / autc
        done += len(chunk)
        if nroots is None and time.perf_counter() - t0 >= budget_s:
            break
        batch = min(batch * 2, 1 << 16)
    return matches, time.perf_counter() - t0, done, threads


# ------------------------------------------------------------------ oracle arm

def run_reference(args, rank, world):
    """--impl reference: the oracle (C, all host cores) timed on the host on
    the same workload, metric and unit; rank 0 only."""
    if rank != 0:
        return
    dev = None
    try:
        import torch
        if torch.cuda.is_available():
            dev = torch.device("cuda", 0)
    except ImportError:
        pass
    n, e, pats = load_workload(args.workload, dev)
    csr = host_csr(n, e)
    del e
    # size one step so the whole run stays within a few minutes
    step_budget = max(0.5, 150.0 / max(1, args.steps + args.warmup))
    _, _, nr, _ = oracle_cpu_sample(csr, pats, step_budget, seed=99)
    # every step repeats the calibrated sample (same seed, same roots): a
    # bounded, reproducible amount of oracle work per step
    vals, secs, threads = [], [], 1
    for s in range(args.warmup + args.steps):
        maps, dt, _, threads = oracle_cpu_sample(csr, pats, 0, seed=99, nroots=nr)
        if s >= args.warmup:
            vals.append(maps)
            secs.append(dt)
    value = sum(vals) / sum(secs)
    sample = (f"{nr} seeded random root vertices (degree <= {SAMPLE_MAX_DEG}, the same every step) x {len(pats)} "
              f"patterns, "
              f"C oracle root sums, {threads} OpenMP threads")
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * sum(secs) / len(secs),
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "u128/u256 (C oracle)",
        "data": "synthetic",
        "config": {"workload": WORKLOAD_DESC[args.workload], "patterns": [p.name for p in pats]},
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": threads, "kind": "oracle", "sample": sample},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------ roofline

def listing_stats(n, e):
    """Degree-orientation statistics of the graph (plain torch on the edge
    tensor's device): m, sum over oriented edges (a, b) of the tail length of
    N+(a) after b (the listing kernels' streamed elements), and the merge
    kernel's sum of out(a) + out(b)."""
    import numpy as np
    import torch
    et = e if isinstance(e, torch.Tensor) else torch.from_numpy(np.ascontiguousarray(e))
    dev = et.device
    a = et[:, 0].to(torch.int64)
    b = et[:, 1].to(torch.int64)
    ok = a != b
    lo = torch.minimum(a[ok], b[ok])
    hi = torch.maximum(a[ok], b[ok])
    k = torch.unique(lo * n + hi)
    del a, b, ok, lo, hi
    a, b = k // n, k % n
    del k
    deg = torch.bincount(a, minlength=n) + torch.bincount(b, minlength=n)
    rank = torch.empty(n, dtype=torch.int64, device=dev)
    rank[torch.argsort(deg * n + torch.arange(n, device=dev))] = torch.arange(n, device=dev)
    ra, rb = rank[a], rank[b]
    del a, b
    u, v = torch.minimum(ra, rb), torch.maximum(ra, rb)
    del ra, rb
    out = torch.bincount(u, minlength=n)
    s = torch.argsort(u * n + v)
    u, v = u[s], v[s]
    del s
    oofs = torch.zeros(n + 1, dtype=torch.int64, device=dev)
    oofs[1:] = torch.cumsum(out, 0)
    tail = out[u] - (torch.arange(u.numel(), device=dev) - oofs[u]) - 1
    st = {"m": int(u.numel()), "tail": float(tail.sum()), "merge": float((out[u] + out[v]).sum())}
    del u, v, tail, oofs, out, deg, rank
    if dev.type != "cpu":
        torch.cuda.empty_cache()
    return st


def support_bytes(st, tri, hash_mode):
    """listing support pass 44 B per oriented edge (in-entry
    a, rev, split/oofs/offs of a; table staging and c(b, x) flush) + 4 B per
    streamed tail element + 8 B per triangle (c(a, c) reduction); merge
    kernel 40 B per edge + 4 B per merged out-list element"""
    if hash_mode:
        return 44.0 * st["m"] + 4.0 * st["tail"] + 8.0 * tri
    return 40.0 * st["m"] + 4.0 * st["merge"]


def tricore_bytes(st, tri):
    """triangle-core listing pass: 32 B per in-entry (a, rev, split/oofs/offs)
    + 20 B per in-entry (deg a, c(ab)) + 24 B per N+(b) entry staged (adj, c,
    deg) + 4 B per tail element + 4 B per triangle (c(a, c))"""
    return 76.0 * st["m"] + 4.0 * st["tail"] + 4.0 * tri


# ------------------------------------------------------------------ GPU arm

def pass_core_matches(F, g, cps):
    """distinct core instances per step: per pass, the core-match count of its
    first pattern with the degree filter off (untimed)"""
    probe = F.fsgc_count(g, cps, no_degree_filter=True)
    seen = {}
    for r in probe:
        seen.setdefault(r.pass_index, r.core_matches)
    return sum(seen.values()), probe


def time_counts(F, g, cps, reps, flush):
    """device time (ms) of `reps` synchronous fsgc_count calls (min), counts"""
    import torch
    best, res = None, None
    st = torch.cuda.current_stream()
    for _ in range(reps):
        flush.fill_(1)
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(st)
        res = F.fsgc_count(g, cps)
        b.record(st)
        torch.cuda.synchronize()
        ms = a.elapsed_time(b)
        best = ms if best is None else min(best, ms)
    return best, res


def per_config_block(F, dev, flush, skip):
    """configs[0..3] and the RMAT-26 edge-core decomposition: batched pass
    time and every pattern alone, per pattern x graph"""
    import torch
    out = []
    for wl, reps in PER_CONFIG:
        if wl == skip:
            continue
        try:
            n, e, pats = load_workload(wl, dev)
            g = F.fsgc_load_graph(e, n)
            del e
            cps = [F.compile_named(P) for P in pats]
            cm, _ = pass_core_matches(F, g, cps)
            time_counts(F, g, cps, 1, flush)                       # warm-up (plans, tables)
            ms, res = time_counts(F, g, cps, reps, flush)
            per = {}
            for P, p, r in zip(pats, cps, res):
                time_counts(F, g, [p], 1, flush)
                pms, pr = time_counts(F, g, [p], reps, flush)
                per[P.name] = {"count": str(r.count) if r.count is not None else None,
                               "overflow": r.overflow, "count_time_s": pms / 1e3,
                               "core_matches": pr[0].core_matches,
                               "core_matches_per_s": pr[0].core_matches / (pms / 1e3)}
            log(f"per-config {wl}: batched {ms:.2f} ms")
            out.append({"workload": WORKLOAD_DESC[wl], "graph": {"n": n, "m": g.m, "max_degree": g.max_degree},
                        "batched": {"count_time_s": ms / 1e3, "core_matches": cm,
                                    "core_matches_per_s": cm / (ms / 1e3), "edges_per_s": g.m / (ms / 1e3),
                                    "passes": len({r.pass_index for r in res})},
                        "patterns": per})
            g.free()
            del g
            torch.cuda.empty_cache()
        except Exception as ex:  # a failing side config must not hide the headline line
            out.append({"workload": wl, "error": repr(ex)[:300]})
    return out


T0 = time.perf_counter()


def log(msg):
    """progress on stderr (the JSON line stays the only stdout output)"""
    print(f"[bench {time.perf_counter() - T0:8.1f}s] {msg}", file=sys.stderr, flush=True)


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
    del e
    log(f"workload {args.workload}: n={n} edges={e_dev.shape[0]}")
    st_graph = listing_stats(n, e_dev)
    g = F.fsgc_load_graph(e_dev, n)
    log(f"graph loaded: m={g.m} max_degree={g.max_degree}")
    cps = [F.compile_named(P) for P in pats]
    core_matches, _ = pass_core_matches(F, g, cps)
    log(f"core matches per step: {core_matches}")

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
        log("warm-up step done")
    counts = [r.count for r in res]
    ref = F.fsgc_count_distributed(g, cps) if world > 1 else F.fsgc_count(g, cps)   # the synchronous API agrees
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
        log(f"timed step {s}: {ev0[s].elapsed_time(ev1[s]):.1f} ms")
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
    m = g.m
    share = 1.0 / world
    tri = 0
    if plan is not None and plan.support() is not None:
        tri = int(plan.support().to(torch.int64).sum().item()) // 3
    hash_mode = g.m >= int(os.environ.get("FSGC_SUP_HASH_MIN_M", str(1 << 20)))
    sup_b = support_bytes(st_graph, tri, hash_mode) * share
    names = {0: "vertex_core_kernel", 1: "edge_fc_kernel (Venn + Sec. 3.1 fc, lane per root edge)",
             2: "core_kernel (general core: DFS + min-list Venn + fc)",
             3: "list_*_kernel<tri> (triangle cores: listing by middle vertex + Venn + fc)"}
    kernels = []
    for k in pass_ids:
        kind = kind_of[k]
        if kind == 1:
            byts = 44.0 * m * share
        elif kind == 3:
            byts = tricore_bytes(st_graph, tri) * share
        elif kind == 0:
            byts = 8.0 * (n + 1) * share
        else:   # compulsory graph bytes: CSR + oriented view + supports, read once
            byts = (8.0 * 2 * m + 8.0 * (n + 1) + 8.0 * m + 4.0 * m + 16.0 * n) * share
        kernels.append((names[kind] + f" [pass {k}]", byts, kms_sum[k] / args.steps, kind))
        if kind != 0 and ams_sum[k] > 0:
            kernels.append((("list_*_kernel<support> (per-edge |N(u)&N(v)|, listing by middle vertex)"
                             if hash_mode else "support_kernel (per-edge |N(u)&N(v)|, merge)") + f" [pass {k}]",
                            sup_b, ams_sum[k] / args.steps, "support"))
    kernels.sort(key=lambda kk: -kk[2])
    peak, peak_src = measured_peaks()
    nsm = torch.cuda.get_device_properties(dev).multi_processor_count
    ncu = ncu_r02(args.workload)

    def ncu_sum(prefixes, field):
        vals = [v.get(field) for k, v in ncu.items() if any(k.startswith(p) for p in prefixes)]
        vals = [x for x in vals if x is not None]
        return sum(vals) if vals else None

    def roof(name, byts, ms, kind):
        hbm_ach = byts / (ms / 1e3) / 1e9 if ms > 0 else 0.0
        if kind == "support":
            traffic = ncu_sum(("list_block_kernel<support>", "list_warp_kernel<support>", "support_kernel"),
                              "dram_bytes_per_launch")
        elif kind == 3:
            traffic = ncu_sum(("list_block_kernel<tri", "list_warp_kernel<tri"), "dram_bytes_per_launch")
        else:
            traffic = ncu_traffic(graph_key(args.workload), name)
        out = {"bound": "hbm", "achieved": hbm_ach, "peak": peak, "unit": "GB/s", "frac": hbm_ach / peak,
               "traffic": traffic, "kernel": name, "kernel_ms": ms, "share_of_step": ms / ms_per_step,
               "algorithmic_bytes_per_launch": byts, "peak_source": peak_src}
        inst = ncu_sum(("list_block_kernel<tri", "list_warp_kernel<tri"), "inst_per_launch") if kind == 3 else None
        if inst and ms > 0 and clocks.get("sm_mhz"):
            # the triangle-core pass is bound by instruction issue (fc
            # arithmetic + listing), not by bytes: DESIGN.md Sec. 5 -- warp
            # instructions of the pass (ncu, same build and workload) per
            # second of the live-timed pass, against SMs x 4 schedulers x 1
            # warp-instruction / clock at the sampled SM clock
            ipk = nsm * 4 * clocks["sm_mhz"] * 1e6
            ach = inst * share / (ms / 1e3)
            out = {"bound": "alu", "achieved": ach, "peak": ipk, "unit": "warp-inst/s", "frac": ach / ipk,
                   "traffic": traffic, "kernel": name, "kernel_ms": ms, "share_of_step": ms / ms_per_step,
                   "inst_per_launch": inst * share, "peak_source": f"{nsm} SMs x 4 issue slots x {clocks['sm_mhz']} MHz "
                                                                 "(sampled under load)",
                   "hbm_view": {"algorithmic_bytes_per_launch": byts, "achieved_gbs": hbm_ach, "peak_gbs": peak,
                                "frac": hbm_ach / peak}}
        return out

    # ---- e2e through the public API from pinned host buffers
    e2e = None
    if not args.no_e2e:
        h2d = e_host.numel() * e_host.element_size()
        d2h = 36 + 16 * 32 + 8
        del plan, replay
        if world == 1:
            del cg
        torch.cuda.empty_cache()
        tms = []
        for s in range(1 + max(1, args.e2e_steps)):
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
            log(f"e2e step {s}: {a.elapsed_time(b):.1f} ms")
            if s >= 1:
                tms.append(a.elapsed_time(b))
        et = sum(tms)
        if world > 1:
            t = torch.tensor([et], dtype=torch.float64, device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            et = t.item()
        e2e = {"value": core_matches / (et / len(tms) / 1e3), "unit": UNIT,
               "h2d_bytes_per_step": int(h2d), "d2h_bytes_per_step": int(d2h),
               "ms_per_step": et / len(tms), "steps": len(tms)}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        csr = host_csr(n, e_dev)
        maps, secs, nr, threads = oracle_cpu_sample(csr, pats, args.cpu_budget)
        log(f"cpu baseline: {nr} roots in {secs:.1f} s")
        del csr
        cpu = {"value": maps / secs, "unit": UNIT, "cores": threads, "kind": "oracle",
               "sample": f"{nr} seeded random root vertices (degree <= {SAMPLE_MAX_DEG}) x {len(pats)} patterns "
                         f"({secs:.1f} s, C oracle root sums: every core map, explicit Venn, Listing 5; "
                         f"{threads} OpenMP threads)"}
    del e_dev

    per_config = None
    if rank == 0 and world == 1 and not args.no_per_config:
        g.free()
        torch.cuda.empty_cache()
        per_config = per_config_block(F, dev, flush, args.workload)

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "u128", "data": "synthetic",
            "config": {"workload": WORKLOAD_DESC[args.workload], "patterns": [p.name for p in pats],
                       "graph": {"n": n, "m": m, "max_degree": g.max_degree,
                                 "triangles": tri or None},
                       "core_matches_per_step": core_matches,
                       "count_time_s": ms_per_step / 1e3,
                       "edges_per_s": m / (ms_per_step / 1e3),
                       "counts": {p.name: str(c) for p, c in zip(pats, counts)},
                       "l2": "flushed before every timed step (256 MiB write); graph >> L2",
                       "parallelism": f"{world} GPU(s): graph replicated, support units and triangle-listing "
                                      f"units dealt round-robin, support all-reduce + 1 all-reduce of "
                                      f"128-bit partials"},
            "edges_per_s": m / (ms_per_step / 1e3),
            "gpu_launches": launches,
            "roofline": roof(*kernels[0]),
            "roofline_other_kernels": [roof(*k) for k in kernels[1:]],
            "clocks": clocks,
            "e2e": e2e,
            "cpu_baseline": cpu,
            "per_config": per_config,
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
