#!/usr/bin/env python
"""Benchmark of the iBFS hot path on B200 (driver contract).

  python bench.py [--gpus N --steps K --warmup W --config c5]
  python -m torch.distributed.run --nproc-per-node N ... bench.py --gpus N ...
  python bench.py --impl reference ...      (the CPU oracle as the reference arm)

Metric (BASELINE.json): aggregate GTEPS summed over the i instances,
GTEPS = sum_s m_s / time / 1e9 with m_s = sum over reached v of deg(v).
A step = one pass of the whole hot path (init, every level's expand + commit, the m_s
finalize) over one batch of sources: `--groups-per-rank` GroupBy groups of 128 sources
per rank.  Weak scaling: each rank takes its LPT share of the config's plan and cycles
through it, G groups per step.  Inputs are resident in HBM before the timed region; the
graph (8 GiB adjacency for c5) and per-group state (3 GiB) exceed the 126 MB L2, so no
flush is needed between steps (c4's graph fits in L2: it flushes by writing 256 MiB).
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import ibfs_gen  # noqa: E402  (seeded input generator shared with the oracle)

METRIC = "aggregate GTEPS (summed over i instances)"
DEFAULT_GROUPS = {"c1": 1, "c2": 1, "c3": 8, "c4": 256, "c5": 4}
PEAKS = os.path.join(ROOT, "MEASURED_PEAKS.json")
FALLBACK_HBM = 6650.0  # GB/s, B200_PROFILING.md fallback


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=8)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="c5", choices=sorted(ibfs_gen.CONFIGS))
    ap.add_argument("--groups-per-rank", type=int, default=0)
    ap.add_argument("--groups-in-flight", type=int, default=0, help="groups per launch batch (0 = library auto)")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--direction", default="auto")
    ap.add_argument("--alpha", type=float, default=4.0)
    ap.add_argument("--beta", type=float, default=24.0)
    ap.add_argument("--split-div", type=float, default=64.0)
    ap.add_argument("--group-bits", type=int, default=0, help="instances per group (0 = the config's, 128)")
    ap.add_argument("--plan-hops", type=int, default=2, help="GroupBy hub radius (1 = the literal steps, 2 = 2-hop anchors, P:L577)")
    ap.add_argument("--max-depth", type=int, default=0, help="k-hop mode (the 3-hop index of §8.7): 0 = plain BFS")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-clocks", action="store_true", help="diagnostics: no nvidia-smi sampling")
    ap.add_argument("--cpu-sample", type=int, default=0, help="oracle sources (0 = host cores)")
    ap.add_argument("--json-out", default="")
    return ap.parse_args()


def env_rank():
    return (int(os.environ.get("RANK", 0)), int(os.environ.get("WORLD_SIZE", 1)),
            int(os.environ.get("LOCAL_RANK", 0)))


def host_cores() -> int:
    try:
        return len(os.sched_getaffinity(0))
    except Exception:
        return os.cpu_count() or 1


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""
    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index: int):
        self.idx = gpu_index
        self.p = None
        self.lines = []

    def start(self):
        try:
            self.p = subprocess.Popen(["nvidia-smi", f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits",
                                       "-lms", "200", "-i", str(self.idx)],
                                      stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.p = None

    def _read(self):
        for line in self.p.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if self.p is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unavailable"], "samples": 0}
        self.p.terminate()
        try:
            self.p.wait(timeout=5)
        except Exception:
            self.p.kill()
        self.t.join(timeout=2)
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 9:
                continue
            try:
                sm.append(float(f[1]))
                mx = float(f[2])
            except ValueError:
                continue
            for nm, val in zip(names, f[5:9]):
                if val.lower() == "active":
                    reasons.add(nm)
        load = [x for x in sm if mx and x > 0.5 * mx] or sm
        return {"sm_mhz": float(np.median(load)) if load else None, "sm_max_mhz": mx,
                "reasons": sorted(reasons), "samples": len(sm)}


def peak_hbm():
    try:
        with open(PEAKS) as f:
            return float(json.load(f)["hbm_gbs"]), "measured"
    except Exception:
        return FALLBACK_HBM, "fallback"


def ncu_traffic(config: str, kernel: str):
    """dram bytes per launch of `kernel` from the committed ncu --set full summary."""
    path = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:
        with open(path) as f:
            d = json.load(f)
        e = d[config][kernel]
        return float(e["dram_bytes_per_launch"]), e.get("source", path)
    except Exception:
        return None, None


def plan_for(cfg, g, el, W, hops=1):
    src = cfg.sources(el)
    t0 = time.perf_counter()
    perm = g.plan(src, W, hops=hops)
    plan_ms = (time.perf_counter() - t0) * 1e3
    return src[perm], plan_ms


def main():
    args = parse()
    rank, world, local = env_rank()
    if args.impl == "reference":
        return run_reference(args, rank, world)
    import torch
    import torch.distributed as dist
    import paper_conf_sigmod_liuhh16_b200 as P
    from paper_conf_sigmod_liuhh16_b200 import dist as pdist

    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
    cfg = ibfs_gen.CONFIGS[args.config]
    W = args.group_bits or cfg.group_bits
    G = args.groups_per_rank or DEFAULT_GROUPS[args.config] * (cfg.group_bits // W)

    # ---- setup (untimed: timing starts with the data in GPU memory) ----------
    t0 = time.perf_counter()
    el = cfg.edges(threads=host_cores())
    gen_s = time.perf_counter() - t0
    t0 = time.perf_counter()
    g = P.Graph.from_edgelist(el, device=local)
    load_s = time.perf_counter() - t0
    s_plan, plan_ms = plan_for(cfg, g, el, W, args.plan_hops)
    n = len(s_plan)
    n_groups = (n + W - 1) // W
    deg = np.diff(g.export_csr()[0]).astype(np.int64) if cfg.scale <= 24 else None
    costs = pdist.group_costs(s_plan, deg, W) if deg is not None else None
    share = pdist.shard_groups(n_groups, world, rank, costs, "lpt" if costs is not None else "round_robin")
    if len(share) == 0:
        share = np.array([rank % n_groups])

    def step_sources(k):
        gids = [int(share[(k * G + i) % len(share)]) for i in range(G)]
        rows = pdist.rows_of_groups(np.asarray(gids), n, W)
        return s_plan[rows]

    out_dev = torch.empty((G * W, g.nv), dtype=torch.int8, device=dev)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev) if args.config in ("c1", "c2", "c4") else None
    run_kw = dict(direction=args.direction, alpha=args.alpha, beta=args.beta, groups_in_flight=args.groups_in_flight,
                  split_div=args.split_div, max_depth=(args.max_depth or None))
    stream = torch.cuda.current_stream(dev)

    def do_step(k, timing):
        s = step_sources(k)
        if flush is not None:
            flush.fill_(k & 0xff)
        return g.run(s, W, out=out_dev[: len(s)], stream=stream, timing=timing, **run_kw)[1]

    for k in range(args.warmup):
        do_step(k, True)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    sampler = ClockSampler(local)
    if not args.no_clocks:
        sampler.start()
    time.sleep(0.25)
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    ev0.record(stream)
    sts = [do_step(args.warmup + k, True) for k in range(args.steps)]
    ev1.record(stream)
    torch.cuda.synchronize()
    clocks = sampler.stop()
    if world > 1:
        dist.barrier()
    local_ms = ev0.elapsed_time(ev1)
    edges = sum(s.edges_traversed for s in sts)
    t = torch.tensor([local_ms], dtype=torch.float64, device=dev)
    e = torch.tensor([edges], dtype=torch.int64, device=dev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        dist.all_reduce(e, op=dist.ReduceOp.SUM)
    max_ms = float(t.item())
    total_edges = int(e.item())
    value = total_edges / (max_ms * 1e-3) / 1e9
    traverse_ms = sum(s.traverse_ms for s in sts)

    # ---- roofline of the dominant kernel (algorithmic bytes / CUDA-event time) -------
    peak, peak_kind = peak_hbm()
    # level_kernel = commit of level l-1 + expand of level l (one cooperative launch per
    # level); its two phases are also split by the kernel's own globaltimer stamps
    kern = {
        "level": (sum(s.expand_bytes + s.commit_bytes for s in sts), sum(s.level_ms for s in sts),
                  sum(s.level_launches for s in sts)),
        "depth": (sum(s.depth_bytes for s in sts), sum(s.depth_ms for s in sts), sum(s.depth_launches for s in sts)),
    }
    phases = {
        "level.expand": (sum(s.expand_bytes for s in sts), sum(s.expand_ms for s in sts)),
        "level.commit": (sum(s.commit_bytes for s in sts), sum(s.commit_ms for s in sts)),
    }
    dom = max(kern, key=lambda k: kern[k][1])
    b, ms, nl = kern[dom]
    achieved = b / (ms * 1e-3) / 1e9 if ms > 0 else 0.0
    traffic, _ = ncu_traffic(args.config, dom)
    roofline = {"bound": "hbm", "kernel": dom, "achieved": round(achieved, 1), "peak": peak,
                "peak_kind": peak_kind, "unit": "GB/s", "frac": round(achieved / peak, 4),
                "traffic": traffic, "algorithmic_bytes_per_launch": (b / nl if nl else None),
                "share_of_step": round(ms / local_ms, 4) if local_ms else None,
                "all_kernels": {k: {"GB/s": round(v[0] / (v[1] * 1e-3) / 1e9, 1) if v[1] else None,
                                    "ms": round(v[1], 3), "launches": v[2]} for k, v in kern.items()},
                "phases": {k: {"GB/s": round(v[0] / (v[1] * 1e-3) / 1e9, 1) if v[1] else None,
                               "ms": round(v[1], 3)} for k, v in phases.items()}}

    # ---- end to end through the public API with HOST buffers -------------------------
    e2e = None
    if not args.no_e2e:
        host_out = torch.empty((G * W, g.nv), dtype=torch.int8, pin_memory=True)
        srcs_host = [torch.from_numpy(step_sources(args.warmup + k).astype(np.int32)).pin_memory()
                     for k in range(args.steps + 1)]
        g.run(srcs_host[0], W, out=host_out[: len(srcs_host[0])], stream=stream, **run_kw)
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        e2e_edges = 0
        h2d = d2h = 0
        for k in range(args.steps):
            s = srcs_host[k + 1]
            _, st = g.run(s, W, out=host_out[: len(s)], stream=stream, **run_kw)
            e2e_edges += st.edges_traversed
            h2d += s.numel() * 4
            d2h += len(s) * g.nv + len(s) * 8  # depth rows + per-source m_s
        e1.record(stream)
        torch.cuda.synchronize()
        e_ms = e0.elapsed_time(e1)
        te = torch.tensor([e_ms], dtype=torch.float64, device=dev)
        ee = torch.tensor([e2e_edges], dtype=torch.int64, device=dev)
        if world > 1:
            dist.all_reduce(te, op=dist.ReduceOp.MAX)
            dist.all_reduce(ee, op=dist.ReduceOp.SUM)
        e2e = {"value": round(int(ee.item()) / (float(te.item()) * 1e-3) / 1e9, 2), "unit": "GTEPS",
               "h2d_bytes_per_step": h2d // args.steps, "d2h_bytes_per_step": d2h // args.steps}
        del host_out

    # ---- CPU oracle beside it (rank 0, N = 1 only) -----------------------------------
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu = cpu_baseline(el, step_sources(0), args.cpu_sample, args.max_depth or None)

    if rank == 0:
        line = {
            "metric": METRIC, "value": round(value, 2), "unit": "GTEPS", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(max_ms / args.steps, 3),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": f"u{W}",
            "data": "synthetic",
            "config": {"workload": cfg.name + (f", {args.max_depth}-hop" if args.max_depth else ""), "generator": f"R-MAT/Kronecker (A,B,C)={cfg.abc}, seed {cfg.graph_seed}",
                       "scale": cfg.scale, "edgefactor": cfg.ef, "group_bits": W,
                       "sources_per_rank_per_step": G * W, "groups_per_rank_per_step": G,
                       "planner": f"GroupBy (hops={args.plan_hops})", "direction": args.direction,
                       "groups_in_flight": args.groups_in_flight or "auto",
                       "max_depth": args.max_depth or None,
                       "l2": ("flush 256 MiB between steps" if flush is not None
                              else "inputs > L2 (adjacency + per-group state), no flush"),
                       "parallelism": f"groups sharded over {world} rank(s), graph replicated"},
            "traverse_gteps": round(edges / (traverse_ms * 1e-3) / 1e9, 2) if traverse_ms else None,
            "roofline": roofline, "cpu_baseline": cpu, "e2e": e2e,
            "timeline": {"timed_ms": round(max_ms, 3), "traverse_ms": round(traverse_ms, 3),
                         "level_gap_ms": round(sum(s.level_gap_ms for s in sts), 3),
                         "note": "traverse = device windows of the ibfs_run_ex calls; level_gap = device idle "
                                 "between consecutive level kernels (in-kernel globaltimer); the rest of "
                                 "timed_ms is between calls / batches"},
            "gpu_launches": int(sum(s.n_launches for s in sts)),
            "clocks": clocks,
            "setup": {"gen_s": round(gen_s, 2), "load_s": round(load_s, 2), "plan_ms": round(plan_ms, 2),
                      "nv": g.nv, "ne": g.ne, "n_sources": n, "n_groups": n_groups},
            "levels": {"max": max(s.max_levels for s in sts), "td_group_levels": sum(s.levels_td for s in sts),
                       "bu_group_levels": sum(s.levels_bu for s in sts),
                       "sd_td": round(sum(s.sd_fq_td for s in sts) / max(1, sum(s.sd_jfq_td for s in sts)), 3),
                       "sd_bu": round(sum(s.sd_fq_bu for s in sts) / max(1, sum(s.sd_jfq_bu for s in sts)), 3)},
        }
        txt = json.dumps(line)
        print(txt, flush=True)
        if args.json_out:
            with open(args.json_out, "w") as f:
                f.write(txt + "\n")
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


def cpu_baseline(el, sources, sample, max_depth=None):
    """The oracle as it stands, timed on the host cores on a bounded sample."""
    import oracle
    cores = host_cores()
    k = sample or cores
    s = np.asarray(sources[:k], dtype=np.uint32)
    og = oracle.OracleGraph.from_edges(el)  # adjacency build: setup, untimed
    t0 = time.perf_counter()
    r = og.bfs(s, want_depths=False, threads=cores, max_depth=max_depth)
    dt = time.perf_counter() - t0
    return {"value": round(float(r.m_s.sum()) / dt / 1e9, 4), "unit": "GTEPS", "cores": min(cores, len(s)),
            "kind": "oracle", "seconds": round(dt, 2),
            "sample": f"{len(s)} sources of step 0 (textbook BFS each, one thread per source)"}


def run_reference(args, rank, world):
    """--impl reference: the CPU oracle, on rank 0 only, each step a bounded sample."""
    if rank != 0:
        return
    import oracle
    cfg = ibfs_gen.CONFIGS[args.config]
    el = cfg.edges(threads=host_cores())
    src = cfg.sources(el)
    og = oracle.OracleGraph.from_edges(el)
    cores = host_cores()
    k = args.cpu_sample or cores
    for i in range(args.warmup):
        og.bfs(src[(i * k) % len(src):][:k], want_depths=False, threads=cores)
    t0 = time.perf_counter()
    edges = 0
    for i in range(args.steps):
        j = ((args.warmup + i) * k) % len(src)
        r = og.bfs(src[j:j + k], want_depths=False, threads=cores)
        edges += int(r.m_s.sum())
    dt = time.perf_counter() - t0
    value = edges / dt / 1e9
    line = {
        "impl": "reference", "metric": METRIC, "value": round(value, 4), "unit": "GTEPS", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(dt * 1e3 / args.steps, 2),
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "int32 (depth)",
        "data": "synthetic",
        "config": {"workload": cfg.name, "scale": cfg.scale, "edgefactor": cfg.ef,
                   "sources_per_step": k, "note": "CPU oracle (textbook BFS per source), bounded sample"},
        "cpu_baseline": {"value": round(value, 4), "unit": "GTEPS", "cores": cores, "kind": "oracle",
                         "sample": f"{k} sources per step, {args.steps} steps"},
        "e2e": {"value": round(value, 4), "unit": "GTEPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


if __name__ == "__main__":
    main()
