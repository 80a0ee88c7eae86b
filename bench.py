#!/usr/bin/env python3
"""bench.py -- fundamental cycles balanced per second on B200 (BASELINE.json).

One *step* = the whole hot path (roots + BFS +
min-hash parents, Alg. 4 labels, Alg. 3 cycle traversal and balancing, flip
and Harary-agree accumulation) over the workload's T trees per GPU; for N > 1
ranks it also includes the NCCL all-reduce of the integer counters (L248).
Trees are sharded t -> rank (t mod N), T per GPU (weak scaling).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config c3] [--trees T]
  python bench.py --impl reference ...   # the CPU oracle as the reference arm

Prints ONE JSON line on rank 0.  Device time = CUDA events on the stream the
library launches on, barrier + synchronize on both sides, max over ranks.
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
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

PAPER_BOOKS_CYCLES_PER_S = 12_294_896 / 0.8512   # PAPER.md L27, Table 3, Table 1
METRIC = "fundamental cycles balanced/sec (device-timed)"
DEFAULT_CONFIG = "c3"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default=DEFAULT_CONFIG)
    ap.add_argument("--trees", type=int, default=0, help="trees per GPU per step (0 = config default)")
    ap.add_argument("--walk", type=int, default=0)
    ap.add_argument("--batch", type=int, default=0)
    ap.add_argument("--sub", type=int, default=0, help="trees per labelling launch (0 = auto)")
    ap.add_argument("--opt", action="append", default=[], help="library option key=value (gb_set_option)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-sample-trees", type=int, default=0)
    return ap.parse_args()


# ---------------------------------------------------------------------------
# clocks during the timed region (B200_PROFILING.md)
# ---------------------------------------------------------------------------
class ClockSampler:
    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index):
        self.idx = gpu_index
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.idx), f"--query-gpu={self.FIELDS}",
                 "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        if not self.lines:
            # timed region shorter than the sampling period: one sample right after it
            try:
                out = subprocess.run(["nvidia-smi", "-i", str(self.idx), f"--query-gpu={self.FIELDS}",
                                      "--format=csv,noheader,nounits"], capture_output=True,
                                     text=True, timeout=10).stdout.strip()
                if out:
                    self.lines.append(out.splitlines()[0])
                    self.post = True
            except Exception:
                pass
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        self.t.join(timeout=2)
        sm, smax, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            p = [x.strip() for x in ln.split(",")]
            if len(p) < 7:
                continue
            try:
                sm.append(float(p[0]))
                smax.append(float(p[1]))
            except ValueError:
                continue
            for nm, val in zip(names, p[3:7]):
                if val.lower().startswith("active"):
                    reasons.add(nm)
        out = {"sm_mhz": statistics.median(sm) if sm else None,
               "sm_max_mhz": max(smax) if smax else None,
               "reasons": sorted(reasons), "samples": len(sm)}
        if getattr(self, "post", False):
            out["note"] = "timed region shorter than 100 ms: one sample taken right after it"
        return out


# ---------------------------------------------------------------------------
# algorithmic byte model per tree (SURVEY.md §8d B_tree): the
# minimal compulsory traffic of each phase, 4-byte ids / offsets.  Batching
# (one CSR pass serving B trees) can move less than this; the ncu traffic of
# the dominant kernel is reported next to it (profiles/traffic_c3.json).
# ---------------------------------------------------------------------------
def phase_bytes(n, m, sumk, trees, batch):
    return {
        "init": 0.0,
        "bfs": 4 * (n + 1) + 8 * m + 8 * m + 8 * n,      # CSR read, one neighbour-state gather per slot, dist+parent
        "bottom_up": 16 * n,                             # read parent, RMW size
        "top_down": 16 * n,                              # read parent/size, write pre and the record
        "cycles": 8 * m + 8 * (sumk / trees),            # non-tree enumeration + one 8 B record per cycle step
        "accumulate": (m + n) / 8 + 8 * (m + n) / batch,  # flip/pi bits + amortised counter RMW
    }


def ncu_traffic(config, kernel, trees_per_launch):
    """DRAM bytes (read + write) per launch of `kernel` from the committed ncu
    --set full capture (profiles/traffic_<config>.json), scaled to the trees of
    one launch here; None if there is no capture for this config/kernel."""
    try:
        with open(os.path.join(ROOT, "profiles", f"traffic_{config}.json")) as f:
            d = json.load(f)[kernel]
        return d["dram_bytes"] / d["trees"] * trees_per_launch
    except Exception:
        return None


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


# ---------------------------------------------------------------------------
def _cpu_model():
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except Exception:
        pass
    return "unknown"


_ORACLE_SHARED = {}


def _oracle_shard(job):
    """Child of the all-cores baseline (fork): trees t_begin, t_begin+P, ...
    of the shared oracle graph."""
    og = _ORACLE_SHARED["og"]
    t0 = time.perf_counter()
    og.balance(job[1], job[2], t_begin=job[0], stride=job[3])
    return time.perf_counter() - t0


def cpu_baseline(g, seed, trees, c_nt):
    """The oracle as it stands (plain single-threaded C), on a bounded sample:
    1 core (`trees` trees), and all host cores as P = nproc independent
    processes over disjoint tree subsets (P trees, one per process; the
    graph is built once and shared copy-on-write by fork)."""
    import multiprocessing as mp
    import oracle
    og = oracle.Graph.from_csr(g)
    t0 = time.perf_counter()
    og.balance(trees, seed)
    dt = time.perf_counter() - t0
    out = {"value": trees * c_nt / dt, "unit": "cycles/s", "cores": 1, "kind": "oracle",
           "cpu_model": _cpu_model(), "host_cores": os.cpu_count(),
           "sample": f"{trees} tree(s) of the same workload (seed {seed}), {dt:.2f} s, "
                     f"single-threaded plain C (-O2)"}
    P = os.cpu_count() or 1
    if P > 1:
        try:
            _ORACLE_SHARED["og"] = og
            ctx = mp.get_context("fork")
            with ctx.Pool(P) as pool:
                t1 = time.perf_counter()
                pool.map(_oracle_shard, [(r, P, seed, P) for r in range(P)], chunksize=1)
                dt_all = time.perf_counter() - t1
            out["all_cores"] = {"value": P * c_nt / dt_all, "unit": "cycles/s", "cores": P,
                                "sample": f"{P} trees, one per process (tree-parallel oracle, "
                                          f"fork after the graph build), {dt_all:.2f} s wall"}
        except Exception as e:  # the 1-core figure stands on its own
            out["all_cores"] = {"value": None, "error": str(e)[:200]}
        finally:
            _ORACLE_SHARED.clear()
    return out


def sample_trees_for(g, requested):
    if requested:
        return requested
    # ~10-30 s of oracle work: about 2e6 edges per tree-second on the host
    return int(max(1, min(200, 4e7 / max(1, g.m))))


def run_reference(args, g, desc, T):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import oracle
    og = oracle.Graph.from_csr(g)
    c_nt = g.m - g.n + og.ncomp
    per_step = sample_trees_for(g, args.cpu_sample_trees)
    for i in range(args.warmup):
        og.balance(per_step, 1 + i, t_begin=0)
    times = []
    for s in range(args.steps):
        t0 = time.perf_counter()
        og.balance(per_step, 1000 + s)
        times.append(time.perf_counter() - t0)
    tot = sum(times)
    val = args.steps * per_step * c_nt / tot
    line = {
        "impl": "reference", "metric": METRIC, "value": val, "unit": "cycles/s",
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": 1000 * tot / args.steps, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": val / PAPER_BOOKS_CYCLES_PER_S, "dtype": "u32", "data": "synthetic",
        "config": {"workload": f"{args.config}: {desc}", "n": g.n, "m": g.m,
                   "trees_per_step": per_step, "note": "oracle = the reference arm of this tier"},
        "cpu_baseline": {"value": val, "unit": "cycles/s", "cores": 1, "kind": "oracle",
                         "sample": f"{per_step} tree(s) per step of {args.config}"},
        "e2e": {"value": val, "unit": "cycles/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def _relaunch_under_torchrun(args):
    """`bench.py --gpus N` started without torchrun: start the N ranks here
    (one process per GPU, 127.0.0.1 rendezvous) and return their exit code."""
    import socket
    sock = socket.socket()
    sock.bind(("127.0.0.1", 0))
    port = sock.getsockname()[1]
    sock.close()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd)


def main():
    args = parse()
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ and args.impl == "ours":
        sys.exit(_relaunch_under_torchrun(args))
    import graphgen
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "ours" and world != args.gpus:
        raise SystemExit(f"bench.py --gpus {args.gpus} but WORLD_SIZE={world}")
    g, T_default, desc = graphgen.config(args.config)
    T = args.trees or T_default
    if args.impl == "reference":
        return run_reference(args, g, desc, T)

    if world > 1:
        # rank counts and the NCCL transport in the log (init lines only)
        os.environ.setdefault("NCCL_DEBUG", "INFO")
        os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
        os.environ.setdefault("NCCL_DEBUG_FILE", "/dev/stderr")   # stdout carries the one JSON line
    import torch
    import torch.distributed as dist
    from paper_conf_sc_alabanditrb21_b200 import graphb
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    graphb.set_option("walk", args.walk)
    graphb.set_option("batch", args.batch)
    graphb.set_option("sub", args.sub)
    for kv in args.opt:
        k, v = kv.split("=")
        graphb.set_option(k, int(v))
    graphb.load_graph(g)
    n, m, ncomp = graphb.graph_info()
    c_nt = m - n + ncomp
    dev = torch.device("cuda", local)
    stream = torch.cuda.current_stream(dev)
    buf = graphb.counter_buffer(dev)      # [cnt (m) | agree (n)]: the all-reduce buffer, allocated once
    total_trees = T * world

    def step(seed):
        graphb.balance_range_buf(rank, total_trees, world, seed, buf, stream=stream)
        if world > 1:
            dist.all_reduce(buf)

    for i in range(args.warmup):
        step(100 + i)
    # per-phase CUDA events (library-internal, same stream) on one extra step
    graphb.set_option("timing", 1)
    step(99)
    phase = graphb.stats()
    graphb.set_option("timing", 0)
    step(98)
    launches_per_step = graphb.stats()["launches"]

    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    clk = ClockSampler(local)
    clk.start()
    evs = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps + 1)]
    evs[0].record(stream)
    for s in range(args.steps):
        step(1 + s)                       # no host synchronisation inside the timed region
        evs[s + 1].record(stream)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    clocks = clk.stop()
    ms = evs[0].elapsed_time(evs[-1])
    step_ms = [evs[s].elapsed_time(evs[s + 1]) for s in range(args.steps)]
    t = torch.tensor([ms] + step_ms, dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms_max = float(t[0].item())
    step_max = [float(x) for x in t[1:].tolist()]
    cycles_total = args.steps * total_trees * c_nt
    value = cycles_total / (ms_max / 1000.0)
    per_step_cycles = total_trees * c_nt
    steps_summary = {"best_ms": min(step_max), "median_ms": statistics.median(step_max),
                     "best_value": per_step_cycles / (min(step_max) / 1000.0),
                     "median_value": per_step_cycles / (statistics.median(step_max) / 1000.0),
                     "note": "per-step CUDA events, max over ranks; best-of and median as the paper's L327"}

    # roofline of the dominant phase (from the timed-phase step)
    ph = phase["phase_ms"]
    dom = max(ph, key=lambda k: ph[k])
    trees_in_step = phase["trees"]
    per_tree_sumk = phase["sum_cycle_len"] / max(1, trees_in_step)
    bytes_per_tree = phase_bytes(n, m, per_tree_sumk * trees_in_step, trees_in_step, phase["batch"])
    # launches per phase, from the library's own counts (gb_get_stats [6], [7], [9], [10])
    launches_of = {"bfs": max(1, phase["batches"] * -(-phase["batch"] // max(1, phase["bfs_group"]))),
                   "cycles": max(1, phase["batches"] * -(-phase["batch"] // max(1, phase["cycle_group"]))),
                   "bottom_up": max(1, phase["batches"] * -(-phase["batch"] // max(1, phase["sub"]))),
                   "top_down": max(1, phase["batches"] * -(-phase["batch"] // max(1, phase["sub"])))}
    dom_launches = launches_of.get(dom, phase["batches"])
    dom_bytes_per_launch = bytes_per_tree[dom] * trees_in_step / dom_launches
    dom_ms_per_launch = ph[dom] / dom_launches
    peak, peak_src = load_peaks()
    achieved = dom_bytes_per_launch / (dom_ms_per_launch / 1000.0) / 1e9
    bfs_kernel = "k_msbfs"
    opts = {kv.replace(" ", "").split("=")[0]: kv.replace(" ", "").split("=")[1] for kv in args.opt}
    walk_kernel = {0: "k_cycles_irec" if opts.get("jump", "1") == "1" else "k_cycles_jump",
                   1: "k_cycles_descent", 2: "k_cycles_paper", 3: "k_cycles_pclimb"}[args.walk]
    kernel_of = {"bfs": bfs_kernel, "bottom_up": "k_bottom_up", "top_down": "k_top_down",
                 "cycles": walk_kernel, "accumulate": "k_accumulate_edges", "init": "k_ms_roots"}
    traffic = ncu_traffic(args.config, kernel_of[dom], trees_in_step / dom_launches)
    path_bytes = sum(bytes_per_tree.values()) * total_trees * args.steps / world
    roofline = {"bound": "hbm", "kernel": dom, "achieved": achieved, "peak": peak, "unit": "GB/s",
                "frac": achieved / peak, "traffic": traffic, "peak_source": peak_src,
                "kernel_name": kernel_of[dom], "trees_per_launch": trees_in_step / dom_launches,
                "path_achieved": path_bytes / (ms_max / 1000.0) / 1e9,
                "path_frac": path_bytes / (ms_max / 1000.0) / 1e9 / peak,
                "bytes_per_launch": dom_bytes_per_launch, "launch_ms": dom_ms_per_launch,
                "traffic_source": "profiles/traffic_%s.json (ncu --set full, per launch)" % args.config,
                "phase_share": {k: v / max(1e-9, sum(ph.values())) for k, v in ph.items()}}
    graphb_only = (ph["bottom_up"] + ph["top_down"] + ph["cycles"]) / max(1, trees_in_step)

    # end-to-end through the public API with host buffers: gb_load_csr (H2D +
    # ingest) + gb_balance (host outputs; N > 1: graphb.balance, the sharded
    # path with its all-reduce) per step
    e2e = None
    if not args.no_e2e:
        pin = lambda a: torch.from_numpy(np.ascontiguousarray(a)).pin_memory().numpy()
        hrp, hcol, hsg = pin(g.row_ptr), pin(g.col), pin(g.sign)
        h_cnt = torch.empty(max(m, 1), dtype=torch.int32).pin_memory().numpy().view(np.uint32)
        h_agr = torch.empty(n, dtype=torch.int32).pin_memory().numpy().view(np.uint32)
        e_steps = max(1, min(args.steps, 3))

        def e2e_step(seed):
            graphb.load_csr(hrp, hcol, hsg)
            if world > 1:
                graphb.balance(total_trees, seed)
            else:
                graphb.balance_host(T, seed, out=(h_cnt, h_agr))

        e2e_step(499)            # untimed: first-call allocations of the host-output path
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        trace = os.environ.get("GB_E2E_TRACE")
        for s in range(e_steps):
            ta = time.perf_counter()
            graphb.load_csr(hrp, hcol, hsg)
            tb = time.perf_counter()
            if world > 1:
                graphb.balance(total_trees, 500 + s)
            else:
                graphb.balance_host(T, 500 + s, out=(h_cnt, h_agr))
            if trace:
                print(f"e2e step {s}: load {1e3 * (tb - ta):.1f} ms, balance+d2h "
                      f"{1e3 * (time.perf_counter() - tb):.1f} ms", file=sys.stderr, flush=True)
        el = time.perf_counter() - t0
        tt = torch.tensor([el], dtype=torch.float64, device=dev)
        if world > 1:
            dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        e2e = {"value": e_steps * total_trees * c_nt / float(tt.item()), "unit": "cycles/s",
               "h2d_bytes_per_step": int(hrp.nbytes + hcol.nbytes + hsg.nbytes),
               "d2h_bytes_per_step": int(4 * (m + n)),
               "note": "per step: gb_load_csr (H2D + ingest) + gb_balance with host outputs "
                       "(N > 1: graphb.balance = shard + NCCL all-reduce + D2H)"}

    cpu = None
    if rank == 0 and not args.no_cpu_baseline:
        if g.m > 2e8 and not args.cpu_sample_trees:
            # the single-threaded oracle needs minutes just to build a 1 B-edge graph
            cpu = {"value": None, "unit": "cycles/s", "cores": 1, "kind": "oracle",
                   "sample": "not run: m > 2e8 exceeds the bounded-sample budget "
                             "(pass --cpu-sample-trees 1 to force one tree)"}
        else:
            cpu = cpu_baseline(g, 1, sample_trees_for(g, args.cpu_sample_trees), c_nt)

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": "cycles/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_max / args.steps,
            "higher_is_better": True, "scaling": "weak",
            "vs_baseline": value / PAPER_BOOKS_CYCLES_PER_S,
            "vs_baseline_ref": "paper: 14.44M cycles/s, Amazon Books, Titan V (L27, L395) -- context",
            "dtype": "u32", "data": "synthetic",
            "config": {"workload": f"{args.config}: {desc}", "n": n, "m": m, "components": ncomp,
                       "cycles_per_tree": c_nt, "trees_per_gpu": T, "trees_total": total_trees,
                       "batch": phase["batch"], "cycle_group": phase["cycle_group"],
                       "bfs_trees_per_launch": phase["bfs_group"],
                       "walk": {0: "two-ended interval climb", 1: "alg3-descent", 2: "paper edge lists",
                                3: "pre-order climb"}[args.walk],
                       "avg_cycle_len": per_tree_sumk / max(1, c_nt),
                       "max_depth": phase["max_depth"],
                       "l2": "inputs larger than L2 (graph arrays > 126 MB)" if 16 * m > 126e6
                             else "graph fits L2; consecutive steps use new seeds (new trees)",
                       "parallelism": f"trees t mod {world}; NCCL all-reduce of counters" if world > 1
                                      else "1 GPU"},
            "gpu_launches": launches_per_step * args.steps,
            "steps_detail": steps_summary,
            "phase_ms_per_step": {k: v for k, v in ph.items()},
            "graphb_only_ms_per_tree": graphb_only,
            "roofline": roofline,
            "cpu_baseline": cpu,
            "e2e": e2e,
            "clocks": clocks,
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
    graphb.free()
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
