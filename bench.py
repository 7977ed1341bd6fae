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
REF_BUDGET_S = 150.0   # --impl reference: timed CPU work of the whole run


def parse(argv=None):
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=8)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="c5", choices=sorted(ibfs_gen.CONFIGS))
    ap.add_argument("--groups-per-rank", type=int, default=0)
    ap.add_argument("--groups-in-flight", type=int, default=0, help="groups per launch batch (0 = library auto)")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--direction", default="auto")
    ap.add_argument("--alpha", type=float, default=3.0)
    ap.add_argument("--beta", type=float, default=24.0)
    ap.add_argument("--split-div", type=float, default=512.0)
    ap.add_argument("--group-bits", type=int, default=0, help="instances per group (0 = the config's, 128)")
    ap.add_argument("--plan-hops", type=int, default=2, help="GroupBy hub radius (1 = the literal steps, 2 = 2-hop anchors, P:L577)")
    ap.add_argument("--max-depth", type=int, default=0, help="k-hop mode (the 3-hop index of §8.7): 0 = plain BFS")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-clocks", action="store_true", help="diagnostics: no nvidia-smi sampling")
    ap.add_argument("--cpu-sample", type=int, default=0, help="oracle sources (0 = host cores)")
    ap.add_argument("--json-out", default="")
    ap.add_argument("--dist-backend", default="nccl", choices=["nccl", "gloo"],
                    help="process group of a multi-rank run (gloo: the one-GPU CI test of the rank logic)")
    return ap.parse_args(argv)


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


def ncu_traffic_entry(config: str, kernel: str):
    """The committed ncu DRAM-traffic record of `kernel` (profiles/ncu_traffic.json, written
    by tools/ncu_launch_traffic.py from an ncu launch list of a bench run): bytes per live
    launch, with the file and commit it came from (not measured in this run)."""
    path = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:
        with open(path) as f:
            e = json.load(f)[config][kernel]
        return e
    except Exception:
        return None


def random_ceiling():
    """Committed B200 random-access ceilings (tools/randbench.cu -> profiles/randbench.json)."""
    try:
        with open(os.path.join(ROOT, "profiles", "randbench.json")) as f:
            return json.load(f)
    except Exception:
        return None


def make_roofline(config, sts, step_ms):
    """Roofline of the dominant kernel: ALGORITHMIC bytes per
    live launch over its average CUDA-event time (events on the launching stream, every
    launch of the timed steps).  Look-ahead level launches that find every group finished
    exit at once; bytes per launch and traffic are averaged over the live ones."""
    peak, peak_kind = peak_hbm()
    S = lambda f: sum(getattr(s, f) for s in sts)  # noqa: E731
    kern = {
        # level_kernel = commit of level l-1 + expand of level l (one cooperative launch
        # per level); the commit is counted with §8(d)'s dense-scan model
        "level": (S("expand_bytes") + S("commit_bytes"), S("level_ms"), S("level_launches_live"), S("level_launches")),
        "depth": (S("depth_bytes"), S("depth_ms"), S("depth_launches"), S("depth_launches")),
        "ms": (S("ms_bytes"), S("ms_ms"), S("ms_launches"), S("ms_launches")),
        "clean": (S("clean_bytes"), S("clean_ms"), S("clean_launches"), S("clean_launches")),
    }
    dom = max(kern, key=lambda k: kern[k][1])
    b, ms, live, nl = kern[dom]
    achieved = b / (ms * 1e-3) / 1e9 if ms > 0 else 0.0
    tr = ncu_traffic_entry(config, dom)
    gbs = lambda x, t: round(x / (t * 1e-3) / 1e9, 1) if t else None  # noqa: E731
    exp_ms, com_ms = S("expand_ms"), S("commit_ms")
    insp = S("edges_inspected")
    rl = {"bound": "hbm", "kernel": dom, "achieved": round(achieved, 1), "peak": peak, "peak_kind": peak_kind,
          "unit": "GB/s", "frac": round(achieved / peak, 4),
          "traffic": tr.get("dram_bytes_per_launch") if tr else None,
          "traffic_source": (f"{tr.get('source')} (commit {tr.get('commit', '?')}), not this run" if tr else None),
          "algorithmic_bytes_per_launch": (b / live if live else None),
          "launches": nl, "launches_live": live,
          "model": "DESIGN.md §5 = SURVEY.md §8(d): expand 8+B per frontier, 4+B per inspection, B per write; "
                   "commit 2B per vertex (dense scan; the clean ring clears each read slot once, in the m_s "
                   "pass or the clean kernel: B per vertex and loaded level) + B per new vertex; depth rows "
                   "i*|V| + B per loaded snapshot",
          "share_of_step": round(ms / step_ms, 4) if step_ms else None,
          "all_kernels": {k: {"GB/s": gbs(v[0], v[1]), "ms": round(v[1], 3), "launches": v[3], "live": v[2],
                              "bytes_per_live_launch": (v[0] / v[2] if v[2] else None)} for k, v in kern.items()},
          "phases": {"level.expand": {"GB/s": gbs(S("expand_bytes"), exp_ms), "ms": round(exp_ms, 3)},
                     "level.commit": {"GB/s": gbs(S("commit_bytes"), com_ms), "ms": round(com_ms, 3),
                                      "GB/s_moved": gbs(S("commit_bytes_moved"), com_ms),
                                      "note": "GB/s = §8(d) dense-scan model; GB/s_moved = bytes the sparse and "
                                              "dense commits actually stream (degrees and chunk map included)"}}}
    rc = random_ceiling()
    if rc and exp_ms > 0:
        rate = insp / (exp_ms * 1e-3)
        ceil = rc.get("gather16_per_s_2GiB")  # random 16-byte gathers over 2 GiB (4 c5 groups' words)
        rl["phases"]["level.expand"].update({
            "inspections_per_s": round(rate / 1e9, 3), "unit_rate": "G/s",
            "random_gather16_ceiling_per_s": round(ceil / 1e9, 3) if ceil else None,
            "frac_of_random_ceiling": round(rate / ceil, 4) if ceil else None,
            "ceiling_source": rc.get("source", "profiles/randbench.json")})
    return rl


def plan_for(cfg, g, el, W, hops=1):
    src = cfg.sources(el)
    t0 = time.perf_counter()
    perm = g.plan(src, W, hops=hops)
    plan_ms = (time.perf_counter() - t0) * 1e3
    return src[perm], plan_ms


class Workload:
    """What one rank runs: the config's sources in GroupBy order (every rank computes the
    same plan), this rank's LPT share of the groups (cost proxy from the tuple degrees),
    G groups per step (dist.GroupSchedule), and the run options.  The full-size parity
    tests build the same object, so they run exactly the launch shape bench.py times."""

    def __init__(self, args, g, el, world: int = 1, rank: int = 0):
        from paper_conf_sigmod_liuhh16_b200 import dist as pdist
        cfg = ibfs_gen.CONFIGS[args.config]
        self.W = args.group_bits or cfg.group_bits
        self.G = args.groups_per_rank or DEFAULT_GROUPS[args.config] * (cfg.group_bits // self.W)
        self.s_plan, self.plan_ms = plan_for(cfg, g, el, self.W, args.plan_hops)
        costs = pdist.group_costs(self.s_plan, pdist.tuple_degrees(el), self.W)
        self.sched = pdist.GroupSchedule.make(len(self.s_plan), self.W, world, rank, costs, "lpt", self.G)
        self.run_kw = dict(direction=args.direction, alpha=args.alpha, beta=args.beta,
                           groups_in_flight=args.groups_in_flight, split_div=args.split_div,
                           max_depth=(args.max_depth or None))

    def step_sources(self, k: int) -> np.ndarray:
        key = (k * self.sched.groups_per_step) % len(self.sched.share)
        cache = self.__dict__.setdefault("_src", {})
        if key not in cache:
            cache[key] = np.ascontiguousarray(self.s_plan[self.sched.step_rows(k)], dtype=np.uint32)
        return cache[key]


def relaunch(args) -> int:
    """`python bench.py --gpus N` (N > 1) outside torchrun: re-run this command as N ranks,
    one process per GPU (torch.distributed.run, rendezvous on 127.0.0.1)."""
    import socket
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr=127.0.0.1", f"--master-port={port}", os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd)


def main():
    args = parse()
    rank, world, local = env_rank()
    if "WORLD_SIZE" not in os.environ and args.gpus > 1:
        sys.exit(relaunch(args))
    if world != args.gpus:
        sys.exit(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world}: pass --gpus {world}, or launch "
                 f"one rank per GPU with torchrun --nproc-per-node {args.gpus}")
    if args.impl == "reference":
        return run_reference(args, rank, world)
    import torch
    import torch.distributed as dist
    import paper_conf_sigmod_liuhh16_b200 as P
    from paper_conf_sigmod_liuhh16_b200 import dist as pdist

    ndev = torch.cuda.device_count()
    dev_index = local % max(ndev, 1)  # several ranks share a GPU only in the gloo test
    torch.cuda.set_device(dev_index)
    dev = torch.device("cuda", dev_index)
    coll_dev = dev if args.dist_backend == "nccl" else torch.device("cpu")
    if world > 1:
        if args.dist_backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group("gloo")
    cfg = ibfs_gen.CONFIGS[args.config]

    # ---- setup (untimed: timing starts with the data in GPU memory) ----------
    t0 = time.perf_counter()
    el = cfg.edges(threads=host_cores())
    gen_s = time.perf_counter() - t0
    t0 = time.perf_counter()
    g = P.Graph.from_edgelist(el, device=dev_index)
    load_s = time.perf_counter() - t0
    wl = Workload(args, g, el, world, rank)
    W, G, s_plan, sched, run_kw, plan_ms = wl.W, wl.G, wl.s_plan, wl.sched, wl.run_kw, wl.plan_ms
    n = len(s_plan)
    n_groups = (n + W - 1) // W
    step_sources = wl.step_sources

    out_dev = torch.empty((G * W, g.nv), dtype=torch.int8, device=dev)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev) if args.config in ("c1", "c2", "c4") else None
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
    sampler = ClockSampler(dev_index)
    if not args.no_clocks:
        sampler.start()
    time.sleep(0.25)
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    ev0.record(stream)
    wall0 = time.perf_counter()
    sts = [do_step(args.warmup + k, True) for k in range(args.steps)]
    py_wall_ms = (time.perf_counter() - wall0) * 1e3
    ev1.record(stream)
    torch.cuda.synchronize()
    clocks = sampler.stop()
    if world > 1:
        dist.barrier()
    local_ms = ev0.elapsed_time(ev1)
    edges = sum(s.edges_traversed for s in sts)
    # end-of-run collectives (dist.gather_results): MAX of the device time over ranks
    # and every source's m_s (its first run in the timed steps); the traversed
    # edges of every step, repeats included, are SUMmed for the rate
    first_rows, first_m = [], []
    seen = set()
    for k, st_k in enumerate(sts):
        for r, m in zip(sched.step_rows(args.warmup + k), st_k.per_source_m):
            if int(r) not in seen:
                seen.add(int(r))
                first_rows.append(int(r))
                first_m.append(m)
    max_ms, m_full, _ = pdist.gather_results(n, np.asarray(first_rows, dtype=np.int64),
                                             np.asarray(first_m, dtype=np.uint64), None, local_ms, world,
                                             device=coll_dev)
    e = torch.tensor([edges], dtype=torch.int64, device=coll_dev)
    if world > 1:
        dist.all_reduce(e, op=dist.ReduceOp.SUM)
    total_edges = int(e.item())
    value = total_edges / (max_ms * 1e-3) / 1e9
    traverse_ms = sum(s.traverse_ms for s in sts)

    # ---- roofline of the dominant kernel (algorithmic bytes / CUDA-event time) -------
    roofline = make_roofline(args.config, sts, local_ms)

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
        te = torch.tensor([e_ms], dtype=torch.float64, device=coll_dev)
        ee = torch.tensor([e2e_edges], dtype=torch.int64, device=coll_dev)
        if world > 1:
            dist.all_reduce(te, op=dist.ReduceOp.MAX)
            dist.all_reduce(ee, op=dist.ReduceOp.SUM)
        e2e = {"value": round(int(ee.item()) / (float(te.item()) * 1e-3) / 1e9, 2), "unit": "GTEPS",
               "h2d_bytes_per_step": h2d // args.steps, "d2h_bytes_per_step": d2h // args.steps}
        del host_out

    # ---- the ranks' shares (every rank's groups, for the partition check) ----------
    ranks = [{"rank": rank, "groups": [int(x) for x in sched.share], "ms": round(local_ms, 3),
              "edges": int(edges)}]
    if world > 1:
        allr = [None] * world
        dist.all_gather_object(allr, ranks[0])
        ranks = allr

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
                         "host": {"setup_ms": round(sum(s.host_setup_ms for s in sts), 3),
                                  "wait_ms": round(sum(s.host_wait_ms for s in sts), 3),
                                  "in_library_ms": round(sum(s.host_total_ms for s in sts), 3),
                                  "python_wall_ms": round(py_wall_ms, 3)},
                         "note": "traverse = device windows of the ibfs_run_ex calls; level_gap = device idle "
                                 "between consecutive level kernels (in-kernel globaltimer); the rest of "
                                 "timed_ms is between calls / batches"},
            "gpu_launches": int(sum(s.n_launches for s in sts)),
            "shards": {"policy": "LPT on sum over deg>0 sources of 1+log2(1+deg) (dist.group_costs)",
                       "ranks": ranks, "sum_m_s_first_runs": int(m_full.sum()),
                       "sources_run": int((m_full > 0).sum())},
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


def cpu_model() -> str:
    try:
        with open("/proc/cpuinfo") as f:
            for ln in f:
                if ln.startswith("model name"):
                    return ln.split(":", 1)[1].strip()
    except Exception:
        pass
    return "unknown"


def cpu_baseline(el, sources, sample, max_depth=None):
    """The oracle as it stands, timed on the host cores on a bounded sample: one source per
    host core of step 0 (about 20-30 s on c5), plus a 1-thread rate on one source."""
    import oracle
    cores = host_cores()
    k = sample or cores
    og = oracle.OracleGraph.from_edges(el)  # adjacency build: setup, untimed
    while True:  # grow a too-short sample (small graphs) toward ~10 s of CPU work
        s = np.asarray(sources[:k], dtype=np.uint32)
        t0 = time.perf_counter()
        r = og.bfs(s, want_depths=False, threads=cores, max_depth=max_depth)
        dt = time.perf_counter() - t0
        if sample or dt >= 2.0 or k >= len(sources):
            break
        k = min(len(sources), k * max(2, int(10.0 / max(dt, 1e-3))))
    k1 = 1
    while True:
        t1 = time.perf_counter()
        r1 = og.bfs(s[:k1], want_depths=False, threads=1, max_depth=max_depth)
        dt1 = time.perf_counter() - t1
        if dt1 >= 2.0 or k1 >= len(s):
            break
        k1 = min(len(s), k1 * max(2, int(5.0 / max(dt1, 1e-3))))
    return {"value": round(float(r.m_s.sum()) / dt / 1e9, 4), "unit": "GTEPS", "cores": min(cores, len(s)),
            "kind": "oracle", "seconds": round(dt, 2), "cpu_model": cpu_model(),
            "one_thread": {"value": round(float(r1.m_s.sum()) / dt1 / 1e9, 4), "unit": "GTEPS",
                           "seconds": round(dt1, 2), "sample": f"the first {k1} source(s) of the sample"},
            "sample": f"{len(s)} sources of step 0 (textbook BFS each, one thread per source)"}


def run_reference(args, rank, world):
    """--impl reference: the CPU oracle as it stands, rank 0 only (the other ranks exit).

    Budget: the whole run ends within a few minutes.  One warm-up source on one thread
    measures t1 (seconds per source); each of the K timed steps is then a sample of k
    sources, k = max(1, floor(REF_BUDGET_S * cores / (K * t1))), and the K samples run as
    one pool on all host cores (one textbook BFS per source and thread)."""
    if rank != 0:
        return
    import oracle
    cfg = ibfs_gen.CONFIGS[args.config]
    el = cfg.edges(threads=host_cores())
    src = cfg.sources(el)
    og = oracle.OracleGraph.from_edges(el)
    cores = host_cores()
    t0 = time.perf_counter()
    r1 = og.bfs(src[:1], want_depths=False, threads=1, max_depth=args.max_depth or None)
    t1 = max(time.perf_counter() - t0, 1e-3)
    k = args.cpu_sample or max(1, int(REF_BUDGET_S * cores / (max(args.steps, 1) * t1)))
    k = min(k, len(src))
    pool = np.concatenate([src[((1 + i * k) + np.arange(k)) % len(src)] for i in range(args.steps)])
    t0 = time.perf_counter()
    r = og.bfs(pool, want_depths=False, threads=cores, max_depth=args.max_depth or None)
    dt = time.perf_counter() - t0
    edges = int(r.m_s.sum())
    value = edges / dt / 1e9
    line = {
        "impl": "reference", "metric": METRIC, "value": round(value, 4), "unit": "GTEPS", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(dt * 1e3 / max(args.steps, 1), 2),
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "int32 (depth)",
        "data": "synthetic",
        "config": {"workload": cfg.name + (f", {args.max_depth}-hop" if args.max_depth else ""),
                   "scale": cfg.scale, "edgefactor": cfg.ef, "sources_per_step": k,
                   "note": "CPU oracle (textbook BFS per source), bounded sample; the K steps' samples run "
                           "as one pool on all host cores"},
        "cpu_baseline": {"value": round(value, 4), "unit": "GTEPS", "cores": min(cores, len(pool)), "kind": "oracle",
                         "cpu_model": cpu_model(), "seconds": round(dt, 2),
                         "one_thread": {"value": round(float(r1.m_s.sum()) / t1 / 1e9, 4),
                                        "unit": "GTEPS", "seconds": round(t1, 2), "sample": "1 source (the warm-up)"},
                         "sample": f"{k} sources per step x {args.steps} steps; warm-up = 1 source on 1 thread"},
        "e2e": {"value": round(value, 4), "unit": "GTEPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


if __name__ == "__main__":
    main()
