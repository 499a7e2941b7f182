#!/usr/bin/env python3
"""bench.py -- matched embeddings/s of the GAMMA hot path on B200 (BASELINE.json metric).

Default workload (N=1): configs[1], k-clique counting k = 4, 5, 6 on the
cit-Patents-shaped R-MAT (scale 22, a,b,c = 0.53,0.20,0.20, 16.6M raw samples,
seed 1).  One step = the hot path from "CSR resident" to "global result on host" (SURVEY.md
§8(d)): the k-clique counts for every k (A2-A8) from one gamma_kclique_multi pass
(--per-k: one gamma_kclique per k).  Before each step the A1 CSR + DAG build runs
from the raw edge samples resident in HBM (untimed, reported as build_ms_per_step;
a fresh graph per step, so no per-graph cache outlives a step), then L2 is flushed
(256 MiB write).  value = matched embeddings (sum of the k-clique counts) / device
time of the steps (CUDA events, max over ranks).  e2e = the whole step through the
public API from pinned host buffers: H2D of the raw samples + build + hot path.

Other workloads (not the default line): c1 (configs[0]), heavy (kCL scaling
workload), c3 (labeled SM, 4 queries x 2 labelings), c4 (FPM, l=3, MNI).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--workload c2|c1|heavy|c3|c4] [--impl gamma|reference]

Multi-GPU: torchrun one rank per GPU; roots are partitioned (snake-LPT on cost),
the CSR is replicated, one NCCL SUM all-reduce per count.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

METRIC = "matched embeddings/s (kCL, SM, FPM) at 1/2/4/8 B200; % of HBM-BW roofline"
UNIT = "embeddings/s"
COMPUTE_CLASSES = ("extend", "count", "fused", "bitmap", "sm_extend", "sm_count", "fpm")

SM_QUERIES = ["c4", "diamond", "tailed_triangle", "house"]

WORKLOADS = {
    "c2": {"kind": "kcl", "cfg": "c2", "ks": (4, 5, 6),
           "desc": "configs[1]: kCL k=4,5,6 on cit-Patents-shaped R-MAT scale 22 (a,b,c=0.53,0.20,0.20), "
                   "16.6M raw samples, seed 1"},
    "c1": {"kind": "kcl", "cfg": "c1", "ks": (4,),
           "desc": "configs[0]: 4-clique count on R-MAT scale 12 (0.57,0.19,0.19), 90K samples, seed 1"},
    "heavy": {"kind": "kcl", "cfg": "heavy", "ks": (4, 5),
              "desc": "heavy kCL: Graph500-skew R-MAT scale 22 (0.57,0.19,0.19), 20M samples, k=4,5, seed 1"},
    "c3": {"kind": "sm", "cfg": "c3",
           "desc": "configs[2]: labeled SM (4-cycle, diamond, tailed triangle, house) x labels {all 0, i mod 8} "
                   "on LiveJournal-shaped R-MAT scale 23 (0.50,0.20,0.20), 43.5M samples, L=8, seed 1"},
    "c4": {"kind": "fpm", "cfg": "c4", "l": 3, "minsup": 3000,
           "desc": "configs[3]: FPM l=3 edges, MNI minsup=3000, on cit-Patents-shaped R-MAT scale 22 "
                   "(0.40,0.25,0.25), 16.6M samples, L=37, seed 1"},
    "c5": {"kind": "kcl", "cfg": "c5", "ks": (3, 4), "device_gen": True,
           "desc": "configs[4]: triangle + 4-clique count on Friendster-shaped R-MAT scale 26 (0.55,0.20,0.20), "
                   "2.0e9 raw samples drawn in HBM, seed 1 (level-3 table 1.08e11 x 8 B > HBM)"},
}


def sm_runs():
    import gamma_gen as gg
    runs = []
    for q in SM_QUERIES:
        nv, e = gg.QUERIES[q]
        runs.append((q, "all0", nv, e, [0] * nv))
        runs.append((q, "imod8", nv, e, [i % 8 for i in range(nv)]))
    return runs


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        j = json.load(open(p))
        return float(j["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md)"


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled every 200 ms during the timed region
    (the profiling recipe's query).  Note: the polling itself stalls host threads that
    wait on the driver -- C3's batched step (kernel time constant to 0.5 %) took 100-190 ms
    stalls in some steps with it and none without (--no-clocks, profiles/sm_r02b)."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "200"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except (OSError, FileNotFoundError):
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.25)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=2)
        except subprocess.TimeoutExpired:
            self.proc.kill()
        sm, smax, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 9:
                continue
            try:
                sm.append(float(f[1]))
                smax.append(float(f[2]))
            except ValueError:
                continue
            for nm, v in zip(names, f[5:9]):
                if v.lower() == "active":
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None,
                "sm_max_mhz": max(smax) if smax else None,
                "reasons": sorted(reasons), "samples": len(sm)}


def max_over_ranks(value: float, world: int, op: str = "max") -> float:
    """Max (or sum) of a per-rank number over the default process group (identity at world 1)."""
    if world <= 1:
        return float(value)
    import torch
    import torch.distributed as dist
    dev = torch.device("cuda", torch.cuda.current_device()) if dist.get_backend() == "nccl" else torch.device("cpu")
    t = torch.tensor([float(value)], dtype=torch.float64, device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.MAX if op == "max" else dist.ReduceOp.SUM)
    return float(t.item())


def dist_env():
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return rank, world, local


def load_traffic(workload: str, kernel_class: str):
    """dram bytes per launch of the dominant kernel on this workload from the committed
    ncu --set full summary (profiles/ncu_<workload>_<class>.json), or None."""
    p = os.path.join(ROOT, "profiles", f"ncu_{workload}_{kernel_class}.json")
    if os.path.exists(p):
        try:
            j = json.load(open(p))
            return j.get("dram_bytes_per_launch"), os.path.relpath(p, ROOT)
        except (OSError, ValueError):
            pass
    return None, None


def issue_roofline(workload: str, kernel_class: str, ms_per_launch: float, clk: dict):
    """The ceiling that binds an L2-resident, integer path: instruction issue.  Warp
    instructions per launch (committed ncu --set full summaries of this workload's
    dominant class, profiles/ncu_<workload>_<class>[_*].json -- e.g. the kCL hub-part
    kernel is summarised apart from the team kernels but is a launch of the same class:
    smsp__inst_executed.sum over the captured launches of one step / their number) /
    (148 SMs x 4 schedulers x SM clock x the live event-timed ms per launch).  1.0 =
    every scheduler issues every cycle."""
    import glob
    files = sorted(glob.glob(os.path.join(ROOT, "profiles", f"ncu_{workload}_{kernel_class}.json")) +
                   glob.glob(os.path.join(ROOT, "profiles", f"ncu_{workload}_{kernel_class}_*.json")))
    inst_total, launches, thr_w, srcs = 0.0, 0, 0.0, []
    for p in files:
        try:
            j = json.load(open(p))
        except (OSError, ValueError):
            continue
        inst, nl = j.get("inst_executed_per_launch"), j.get("launches_captured") or 0
        if not inst or not nl:
            continue
        inst_total += inst * nl
        launches += nl
        thr_w += (j.get("threads_per_warp_inst") or 0) * inst * nl
        srcs.append(os.path.relpath(p, ROOT))
    if not launches:
        return None
    inst = inst_total / launches
    mhz = (clk or {}).get("sm_mhz") or (clk or {}).get("sm_max_mhz") or 1965.0
    peak = 148 * 4 * mhz * 1e6                     # warp instructions / s
    achieved = inst / (ms_per_launch / 1000.0)
    if achieved > peak:   # the committed summary predates the kernel that ran: no claim
        return {"bound": "issue", "achieved": None, "peak": peak, "unit": "warp-inst/s", "frac": None,
                "stale": f"{srcs} count more instructions than this launch time can issue; "
                         "re-capture them for this build"}
    return {"bound": "issue", "achieved": achieved, "peak": peak, "unit": "warp-inst/s", "frac": achieved / peak,
            "inst_per_launch": inst, "sm_mhz": mhz, "threads_per_inst": thr_w / inst_total if inst_total else None,
            "source": srcs}


def load_alg_bytes(workload: str):
    """SURVEY §8(d) algorithmic bytes of one kCL step, counted over the oracle's
    enumeration by tools/alg_bytes.py (profiles/alg_bytes.json), or None."""
    p = os.path.join(ROOT, "profiles", "alg_bytes.json")
    if os.path.exists(p):
        try:
            return json.load(open(p)).get(workload)
        except (OSError, ValueError):
            return None
    return None


def make_input(name, seed=1):
    import gamma_gen as gg
    w = WORKLOADS[name]
    if w.get("device_gen"):
        # too large for a host-side numpy pass: drawn in HBM by the torch twin of the
        # generator (same words, thresholds and bijection; tests/test_gen.py)
        from gamma_gen.torch_gen import config_graph_torch
        n, s, d = config_graph_torch(w["cfg"], seed=seed)
        return n, s, d, None, w
    n, s, d, lab = gg.config_graph(w["cfg"], seed=seed)
    return n, s, d, lab, w


# ------------------------------------------------------------------------------------
# CPU baseline: the oracle, as it stands, on a bounded seeded sample of the workload.
# ------------------------------------------------------------------------------------
def _aut(nv, edges, plab):
    """|Aut_L(P)| by brute force over the nv! vertex permutations (plain Python)."""
    import itertools
    E = {frozenset(e) for e in edges}
    return sum(1 for p in itertools.permutations(range(nv))
               if all(plab[p[i]] == plab[i] for i in range(nv)) and {frozenset((p[a], p[b])) for a, b in edges} == E)


def cpu_oracle_sample(n, s, d, lab, w, budget_s=12.0, seed=7):
    import oracle
    t0 = time.perf_counter()
    g = oracle.Graph(n, s, d, lab)
    t_build = time.perf_counter() - t0
    cores = os.cpu_count()
    rng = np.random.default_rng(seed)
    if w["kind"] == "fpm":
        # the oracle's FPM has no per-root form: time it on the same generator at a
        # smaller scale until the budget is used
        import gamma_gen as gg
        emb, t_count, scale = 0, 0.0, 12
        while True:
            ns, ss, ds, ls = gg.config_graph(w["cfg"], seed=seed, scale=scale)
            gs = oracle.Graph(ns, ss, ds, ls)
            t1 = time.perf_counter()
            res = gs.fpm(w["l"], max(1, int(w["minsup"] * 2.0 ** (scale - 22))), threads=cores, pattern_cap=1 << 21)
            dt = time.perf_counter() - t1
            emb_l = sum(r[5] for r in res if r[0] == w["l"])
            if t_count + dt > budget_s * 3 and t_count > 0:
                break
            emb, t_count = emb_l, dt
            if dt >= budget_s / 4 or scale >= 22:
                break
            scale += 1
        return {"value": emb / t_count if t_count else None, "unit": UNIT, "cores": cores, "kind": "oracle",
                "sample": f"oracle FPM l={w['l']} on the same generator at scale {scale} (minsup scaled by "
                          f"2^(scale-22)); embeddings counted = frequent-pattern instances at level {w['l']} "
                          f"({emb}) in {t_count:.2f}s on {cores} OpenMP threads",
                "embeddings": emb, "seconds": t_count}
    perm = rng.permutation(n).astype(np.uint32)
    frac, emb, t_count, used = 0.0005, 0.0, 0.0, 0
    threads = cores   # all host cores (torchrun sets OMP_NUM_THREADS=1 per rank)
    while True:
        cnt = min(max(1, int(n * frac)), n - used)
        roots = perm[used:used + cnt]
        t1 = time.perf_counter()
        if w["kind"] == "kcl":
            for k in w["ks"]:
                emb += int(g.kclique_roots(k, roots, threads=threads).sum())
        else:
            for (q, lname, nv, e, plab) in sm_runs():
                mp = int(g.match_roots(nv, e, roots, plab, threads=threads).sum())
                emb += mp / _aut(nv, e, plab)
        dt = time.perf_counter() - t1
        t_count += dt
        used += cnt
        if t_count >= budget_s or used >= n:
            break
        # next chunk: double, but stay within the budget at the rate just seen
        rate = cnt / max(dt, 1e-6)
        frac = min(2 * cnt, max(1, int(rate * (budget_s - t_count)))) / n
    what = (f"k-clique counts k={list(w['ks'])}" if w["kind"] == "kcl" else
            "SM mappings / |Aut_L| over the 8 (query, labeling) runs")
    return {"value": emb / t_count if t_count > 0 else None, "unit": UNIT, "cores": cores, "kind": "oracle",
            "sample": f"oracle {what} for a seeded random sample of {used} of {n} roots ({used / n:.2%}; full CSR "
                      f"build {t_build:.2f}s excluded), {emb:.0f} embeddings in {t_count:.2f}s on {cores} OpenMP threads",
            "embeddings": emb, "seconds": t_count}


def run_reference(args):
    rank, world, _ = dist_env()
    if rank != 0:
        return 0
    if WORKLOADS[args.workload].get("device_gen"):
        print(json.dumps({"impl": "reference", "unavailable": "the CPU oracle cannot time C5 within the bench "
                          "budget (host build of 2e9 samples); C5 parity is sampled in tests/test_gpu_c5.py"}))
        return 0
    n, s, d, lab, w = make_input(args.workload)
    vals, secs, samples = [], [], []
    per_step_budget = max(2.0, 60.0 / max(1, args.steps + args.warmup))
    for i in range(args.warmup + args.steps):
        r = cpu_oracle_sample(n, s, d, lab, w, budget_s=per_step_budget, seed=11 + i)
        if i >= args.warmup:
            vals.append(r["value"])
            secs.append(r["seconds"])
            samples.append(r)
    v = statistics.median(vals)
    out = {"impl": "reference", "metric": METRIC, "value": v, "unit": UNIT, "n_gpus": args.gpus,
           "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1000 * statistics.median(secs),
           "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "u32/u64 integer",
           "data": "synthetic", "config": {"workload": w["desc"], "parallelism": "cpu-oracle"},
           "cpu_baseline": {"value": v, "unit": UNIT, "cores": samples[0]["cores"], "kind": "oracle",
                            "sample": samples[0]["sample"]},
           "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out))
    return 0


# ------------------------------------------------------------------------------------
# The product path.
# ------------------------------------------------------------------------------------
def run_gamma(args):
    import torch
    import torch.distributed as dist
    rank, world, local = dist_env()
    if world > 1:
        # one rank per GPU over NCCL; GAMMA_DIST_BACKEND=gloo lets several ranks share
        # one GPU to exercise the multi-rank path on a single-GPU box
        backend = os.environ.get("GAMMA_DIST_BACKEND", "nccl")
        local = local % torch.cuda.device_count()
        torch.cuda.set_device(local)
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)
    dev = torch.cuda.current_device()
    import paper_conf_icde_hu0o23_b200 as G

    n, s, d, lab, w = make_input(args.workload)
    hd = args.host_dag_cache_mb
    ctx = G.Context(device=dev, time_kernels=True,
                    **({"flags": G._native.GAMMA_FLAG_HOST_DAG, "dag_cache_bytes": int(hd * 2 ** 20)} if hd >= 0 else {}))
    stream = torch.cuda.current_stream()
    if isinstance(s, torch.Tensor):   # drawn on the device
        m_raw = s.numel()
        src_dev, dst_dev = s, d
        src_pin = torch.empty(m_raw, dtype=torch.int32, pin_memory=True)
        dst_pin = torch.empty(m_raw, dtype=torch.int32, pin_memory=True)
        src_pin.copy_(src_dev)
        dst_pin.copy_(dst_dev)
    else:
        m_raw = s.size
        src_dev = torch.from_numpy(s.view(np.int32)).cuda()
        dst_dev = torch.from_numpy(d.view(np.int32)).cuda()
        src_pin = torch.from_numpy(s.view(np.int32)).pin_memory()
        dst_pin = torch.from_numpy(d.view(np.int32)).pin_memory()
    lab_dev = None if lab is None else torch.from_numpy(lab.view(np.int32)).cuda()
    lab_pin = None if lab is None else torch.from_numpy(lab.view(np.int32)).pin_memory()
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    agg = {"_total_launches": {"n": 0}}
    sm_retries = []   # SM: careful-path reruns per timed step (a chain overflowed its tables)
    kern_ms = []      # event-timed compute-kernel ms per collect() (diagnostics: GPU vs host time)
    host_ms = []      # host wall time of each timed step's work() call (diagnostics)

    def collect():
        st = ctx.stats()
        for name, c in st["classes"].items():
            a = agg.setdefault(name, {"launches": 0, "ms": 0.0, "alg_bytes": 0})
            for key in a:
                a[key] += c[key]
        agg["_total_launches"]["n"] += st["total_launches"]
        kern_ms.append(sum(c["ms"] for name, c in st["classes"].items() if name in COMPUTE_CLASSES))
        return st

    def build(src, dst, labels, coll):
        g = ctx.load_edges(n, src, dst, labels)   # A1 (reported as t_build)
        if coll:
            collect()
        return g

    def work(g, coll):
        """One step of the hot path from "CSR resident" to "global result on host"
        (SURVEY §8(d)): A2 root selection / partition, every extension level, the
        aggregate and (N > 1) the collectives."""
        results = {}
        if w["kind"] == "kcl":
            if args.per_k:
                for k in w["ks"]:
                    results[f"k{k}"] = g.kclique(k)
                    if coll:
                        collect()
            else:
                # all sizes from one DFS pass (gamma_kclique_multi): the k=6 walk
                # visits every 4- and 5-clique of the DAG anyway
                for k, c in zip(w["ks"], g.kclique_multi(w["ks"])):
                    results[f"k{k}"] = c
                if coll:
                    collect()
            emb = sum(results.values())
        elif w["kind"] == "sm":
            runs = sm_runs()
            if args.sm_sequential:
                for (q, lname, nv, e, plab) in runs:
                    results[f"{q}/{lname}"] = g.match(nv, e, plab)[0]
                    if coll:
                        collect()
            else:   # one gamma_match_batch: the eight level chains on concurrent streams
                got = g.match_many([(nv, e, plab) for (q, lname, nv, e, plab) in runs])
                for (q, lname, nv, e, plab), (cnt, _) in zip(runs, got):
                    results[f"{q}/{lname}"] = cnt
                if coll:
                    st = collect()
                    sm_retries.append(st.get("retries"))
            emb = sum(results.values())
        else:
            pats = g.fpm_array(w["l"], w["minsup"])   # the result records, no per-pattern Python objects
            st = collect() if coll else ctx.stats()
            per = np.bincount(pats["ne"], minlength=w["l"] + 1) if len(pats) else np.zeros(w["l"] + 1, int)
            results = {f"frequent_l{l}": int(per[l]) for l in range(1, w["l"] + 1)}
            emb = st["level_entries"][w["l"]]
            results["embeddings_per_level"] = st["level_entries"][1:w["l"] + 1]
            results["embeddings_l"] = emb
            results["domain_chunk_passes"] = st.get("chunks")
            results["table_retries"] = st.get("retries")
        return emb, results

    def barrier():
        if world > 1:
            dist.barrier()

    def fresh_graph(coll):
        """The graph of the next step: built from the raw samples in HBM (untimed, a
        fresh handle so no per-graph cache such as the root order outlives a step), then
        L2 flushed so the timed step starts cold."""
        g = build(src_dev, dst_dev, lab_dev, coll)
        flush.fill_(1)
        return g

    for _ in range(args.warmup):
        g = fresh_graph(False)
        work(g, False)
        g.free()
    torch.cuda.synchronize()
    if os.environ.get("GAMMA_BENCH_GC", "1") == "0":   # diagnostics: no cyclic GC in the timed region
        import gc
        gc.collect()
        gc.freeze()
        gc.disable()

    clocks = ClockSampler(dev)
    if not args.no_clocks:
        clocks.start()
    times, builds, emb, results, info = [], [], 0, None, None
    for _ in range(args.steps):
        g = fresh_graph(True)
        info = g.info()
        builds.append(info["build_ms"])
        barrier()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        h0 = time.perf_counter()
        emb, results = work(g, True)
        host_ms.append(1e3 * (time.perf_counter() - h0))
        e1.record(stream)
        torch.cuda.synchronize()
        barrier()
        times.append(e0.elapsed_time(e1))
        g.free()
    clk = clocks.stop()
    total_ms = max_over_ranks(sum(times), world)
    # load imbalance of the root partition = max / mean of the ranks' times
    imbalance = total_ms / (max_over_ranks(sum(times), world, "sum") / world) if world > 1 else 1.0
    value = emb * args.steps / (total_ms / 1000.0)

    # ---- e2e: the whole step through the public API from pinned host buffers: H2D of
    # the raw samples, A1 build, the hot path, results D2H ----
    e2e_times = []
    for _ in range(max(1, min(args.steps, 3))):
        flush.fill_(1)
        barrier()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        g = build(src_pin, dst_pin, lab_pin, False)   # H2D inside gamma_load_edges
        work(g, False)                                  # results D2H per call
        e1.record(stream)
        torch.cuda.synchronize()
        barrier()
        e2e_times.append(e0.elapsed_time(e1))
        g.free()
    e2e_value = emb * len(e2e_times) / (max_over_ranks(sum(e2e_times), world) / 1000.0)

    if rank != 0:
        if world > 1:
            dist.destroy_process_group()
        return 0

    hbm, peak_src = peaks()
    cand = {k: v for k, v in agg.items() if not k.startswith("_") and k in COMPUTE_CLASSES}
    dom = max(cand, key=lambda k: cand[k]["ms"]) if cand else None
    roof = None
    if dom and cand[dom]["ms"] > 0:
        launches = max(1, cand[dom]["launches"])
        per_launch_ms = cand[dom]["ms"] / launches
        summed_ms = sum(v["ms"] for v in cand.values())
        concurrent = summed_ms > total_ms * 1.02   # SM batch chains / kCL team launches overlap on side streams
        if concurrent:
            # overlapping launches each see part of the GPU, so their event durations
            # overstate the time the class holds it: charge the class its share of the
            # summed kernel time of the wall-clock step instead
            per_launch_ms = total_ms * (cand[dom]["ms"] / summed_ms) / launches
        kernel_bytes = cand[dom]["alg_bytes"] / launches   # the kernel's own counters
        ab = load_alg_bytes(args.workload) if not args.per_k else None
        step_bytes = None
        if ab and w["kind"] == "kcl" and ab.get("kmax") == max(w["ks"]):
            step_bytes = ab["bytes_per_step"]
            bytes_src = "SURVEY §8(d) B_l summed over the step's extension levels, counted over the oracle's " \
                        "enumeration (profiles/alg_bytes.json, tools/alg_bytes.py)"
        elif ab and w["kind"] == "sm" and dom in ab.get("class_bytes_per_step", {}):
            step_bytes = ab["class_bytes_per_step"][dom]
            bytes_src = ("SURVEY §8(d) B_t of the " + dom + " steps of the 8 (query, labeling) runs, counted by the "
                         "oracle's O-2b (og_match_levels) in the method's order and constraints (DESIGN R21; "
                         "profiles/alg_bytes.json, tools/alg_bytes.py)")
        elif ab and w["kind"] == "fpm" and ab.get("l") == w["l"]:
            step_bytes = ab["bytes_per_step"]
            bytes_src = ("FPM bytes per step (DESIGN §6): 4 B per adjacency element the extensions read + 32 B per "
                         "recorded embedding, levels 1..l, from closed forms over the oracle's CSR and triangle "
                         "count at minsup = 1 (an upper bound at the bench's minsup; profiles/alg_bytes.json)")
        if step_bytes:
            # the method's bytes per step (oracle-counted), spread over the dominant class's
            # launches of one step (at N > 1 this rank's 1/N share)
            per_launch_bytes = step_bytes / world * args.steps / launches
        else:
            per_launch_bytes = kernel_bytes
            bytes_src = "SURVEY §8(d) B_l from the kernel's own counters (list elements read, entries in/out)"
        achieved = per_launch_bytes / (per_launch_ms / 1000.0) / 1e9
        traffic, traffic_src = load_traffic(args.workload, dom)
        roof = {"bound": "hbm", "achieved": achieved, "peak": hbm, "unit": "GB/s", "frac": achieved / hbm,
                "traffic": traffic, "kernel": dom, "peak_source": peak_src,
                "alg_bytes_per_launch": per_launch_bytes, "alg_bytes_source": bytes_src,
                "kernel_counted_bytes_per_launch": kernel_bytes,
                "ms_per_launch": per_launch_ms, "launches_per_step": launches / args.steps,
                "share_of_step": cand[dom]["ms"] / (summed_ms if concurrent else total_ms),
                **({"timing_basis": "concurrent launches (side streams: SM batch chains, kCL warp and CTA teams): ms_per_launch = step time x the "
                                    "class's share of the summed kernel time / its launches"} if concurrent else {}),
                "traffic_source": traffic_src,
                "issue": issue_roofline(args.workload, dom, per_launch_ms, clk)}
    cpu = None
    if w.get("device_gen"):
        cpu = {"value": None, "unit": UNIT, "cores": os.cpu_count(), "kind": "oracle",
               "sample": "not run in the bench: the oracle's host build of 2e9 samples alone exceeds the "
                         "bench's CPU budget; C5 parity runs on sampled roots in tests/test_gpu_c5.py"}
    elif world == 1 and not args.no_cpu_baseline:
        cpu = cpu_oracle_sample(n, s, d, lab, w, budget_s=args.cpu_seconds)
        cpu.pop("embeddings", None)
        cpu.pop("seconds", None)
    h2d = 2 * 4 * m_raw + (0 if lab is None else 4 * n)
    nres = len(w.get("ks", ())) or (len(sm_runs()) if w["kind"] == "sm" else 1)
    out = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": total_ms / args.steps, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "u32 ids / u64 counts (integer)",
        "data": "synthetic",
        "config": {"workload": w["desc"], "n": n, "m_raw": int(m_raw), "m": int(info["m"]),
                   "max_degree": info["max_degree"], "max_out_degree": info["max_out_degree"],
                   "results": results, "embeddings_per_step": emb,
                   **({"kcl_calls": "per-k gamma_kclique" if args.per_k else "one gamma_kclique_multi pass"}
                      if w["kind"] == "kcl" else {}),
                   "l2": "flushed between steps (256 MiB write)",
                   **({"host_dag_cache_mb": args.host_dag_cache_mb} if args.host_dag_cache_mb >= 0 else {}),
                   "parallelism": f"root-partition dp{world} (CSR replicated)"},
        "roofline": roof,
        "cpu_baseline": cpu,
        "e2e": {"value": e2e_value, "unit": UNIT, "h2d_bytes_per_step": int(h2d), "d2h_bytes_per_step": int(8 * nres)},
        "gpu_launches": int(agg["_total_launches"]["n"]),
        "clocks": clk,
        "kernels": {k: v for k, v in agg.items() if not k.startswith("_") and v["launches"]},
        "build_ms_per_step": statistics.median(builds),
        "timed_region": "CSR resident -> global result on host (SURVEY §8(d)); the A1 build from the raw "
                        "samples in HBM runs before each step, untimed (build_ms_per_step), then L2 is flushed; "
                        "e2e includes H2D + build",
        "step_ms": [round(x, 3) for x in times],
        **({"sm_retries_per_step": sm_retries} if sm_retries else {}),
        "step_kernel_ms": [round(x, 3) for x in kern_ms if x > 0],
        "step_host_ms": [round(x, 3) for x in host_ms],
        "rank_time_max_over_mean": imbalance,
        "e2e_step_ms": [round(x, 3) for x in e2e_times],
    }
    print(json.dumps(out))
    if world > 1:
        dist.destroy_process_group()
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="gamma", choices=["gamma", "reference"])
    ap.add_argument("--workload", default="c2", choices=sorted(WORKLOADS))
    ap.add_argument("--cpu-seconds", type=float, default=15.0)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--per-k", action="store_true", help="kCL: one gamma_kclique call per k instead of one multi-k pass")
    ap.add_argument("--sm-sequential", action="store_true",
                    help="SM: one gamma_match call per (query, labeling) instead of one gamma_match_batch")
    ap.add_argument("--no-clocks", action="store_true", help="diagnostics only: skip nvidia-smi sampling")
    ap.add_argument("--host-dag-cache-mb", type=float, default=-1,
                    help="kCL with the DAG in pinned host memory and an HBM cache of this many MiB of its "
                         "hottest pages (GAMMA_FLAG_HOST_DAG; SURVEY §8(f) rank 4); -1: DAG in HBM")
    args = ap.parse_args()
    if args.impl == "reference":
        return run_reference(args)
    return run_gamma(args)


if __name__ == "__main__":
    sys.exit(main())
