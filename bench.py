#!/usr/bin/env python
"""bench.py -- GTEPS of the EtaGraph hot path (BFS + SSSP + CC) on B200.

One STEP = one pass of the whole hot path (rows A1-A7 of SURVEY 8(a)) for each
algorithm on the N=1 workload, BASELINE.json configs[1] = C2 (RMAT scale 22,
edge factor 16, PaRMAT a/b/c = .45/.22/.22): one BFS and one SSSP from the same
seeded source (16 sources, rotating) and one CC on the symmetrised graph.

value = traversed edges / device time, summed over the step's three calls
(GTEPS; edges = m of the activatable subgraph for BFS/SSSP, Def. 2, and
nnz of the symmetric CSR for CC).  Inputs are resident in HBM; L2 is flushed
(256 MiB write) before every traversal call, outside the timed events.

--gpus N > 1 (torchrun, or bench.py relaunches itself under
torch.distributed.run when WORLD_SIZE is unset): the SAME workload split over
the N ranks (1-D destination partition) through the library's
communicator -- every call runs the partitioned loop with the exchange done
by the library's kernels over peer memory; "scaling": "strong", value = the
same edges / the per-call device time, max over ranks.  Ranks share a GPU when
fewer devices than ranks are visible (tests; no speed-up expected there).
--replicas keeps the older mode: N independent replicas, "scaling": "weak".

--impl reference times the CPU oracle (oracle/, the paper's definitions written
out plainly) on the host cores, on a bounded sample of the same workload.
"""
from __future__ import annotations

import argparse
import ctypes
import json
import os
import statistics
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "GTEPS (BFS/SSSP/CC) at 1/2/4/8 B200; expand-kernel HBM GB/s vs peak"
UNIT = "GTEPS"
# algorithmic bytes: per relaxed edge, per active vertex
BYTES_PER_EDGE = {"bfs": 8, "sssp": 12, "cc": 8}
BYTES_PER_VERTEX = {"bfs": 20, "sssp": 24, "cc": 24}
REASONS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap",
           0x8: "hw_slowdown", 0x10: "sync_boost", 0x20: "sw_thermal_slowdown",
           0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown",
           0x100: "display_clock_setting"}


def parse_args():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=20)
    p.add_argument("--warmup", type=int, default=5)
    p.add_argument("--impl", choices=["ours", "reference"], default="ours")
    p.add_argument("--config", default="C2")
    p.add_argument("--algs", default="bfs,sssp,cc")
    p.add_argument("--K", type=int, default=32)
    p.add_argument("--sssp-delta", default="auto",
                   help="SSSP wave schedule: vertices at distance >= a threshold that advances by this much "
                        "every iteration wait (0: the paper's schedule, every improved vertex every iteration; "
                        "auto: 6 x mean weight / mean out-degree = 12 on C2, 13 on C3, 6 on C4, each near "
                        "its measured best), DESIGN.md sec. 5")
    p.add_argument("--flags", type=int, default=0, help="extra ETG_* flags (e.g. 2 = NO_UDC)")
    p.add_argument("--sources", type=int, default=16)
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--no-profile", action="store_true")
    p.add_argument("--json-out", default=None)
    p.add_argument("--host-edges", action="store_true",
                   help="NEXT-2: keep col/w in pinned host memory (zero-copy reads by the kernels)")
    p.add_argument("--replicas", action="store_true",
                   help="N > 1: N independent replicas (own sources per rank, weak scaling) instead of "
                        "one graph partitioned over the N ranks")
    p.add_argument("--push", action="store_true",
                   help="N > 1: SSSP/CC on a SOURCE partition with the fused push exchange (NEXT-3: the "
                        "expand kernel reduces into the owners' labels over peer memory); BFS keeps the "
                        "destination partition")
    return p.parse_args()


# --------------------------------------------------------------------------- #
# distributed plumbing
# --------------------------------------------------------------------------- #
def dist_setup():
    """Rank / world from the torchrun env.  torch.distributed (gloo) is host
    plumbing only: the communicator id, barriers around the timed region and
    the max-over-ranks reduction of a few numbers; no data-path collective."""
    import torch
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    ndev = max(1, torch.cuda.device_count())
    torch.cuda.set_device(local % ndev)
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("gloo")
    return rank, world, local


def barrier(world):
    if world > 1:
        import torch.distributed as dist
        dist.barrier()


def allreduce(vals, op, world):
    if world == 1:
        return vals
    import torch
    import torch.distributed as dist
    t = torch.tensor(vals, dtype=torch.float64)
    dist.all_reduce(t, op=op)
    return t.tolist()


def relaunch(args):
    """--gpus N > 1 without a torchrun environment: run this script under
    torch.distributed.run with N ranks (127.0.0.1), pass its exit code on."""
    import socket
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd)


# --------------------------------------------------------------------------- #
# clocks during the timed region
# --------------------------------------------------------------------------- #
class ClockSampler:
    def __init__(self, index):
        self.index = index
        self.proc = None
        self.path = None
        self.t0 = self.t1 = None

    def start(self):
        fd, self.path = tempfile.mkstemp(suffix=".csv")
        os.close(fd)
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index),
                 "--query-gpu=timestamp,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active",
                 "--format=csv,noheader,nounits", "-lms", "50"],
                stdout=open(self.path, "w"), stderr=subprocess.DEVNULL)
        except OSError:
            self.proc = None

    def mark(self, which):
        setattr(self, which, time.time())

    def stop(self):
        if self.proc is None:
            return None
        time.sleep(0.12)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except subprocess.TimeoutExpired:
            self.proc.kill()
        rows = []
        for line in open(self.path):
            parts = [x.strip() for x in line.split(",")]
            if len(parts) < 5:
                continue
            try:
                ts = time.mktime(time.strptime(parts[0].split(".")[0], "%Y/%m/%d %H:%M:%S"))
                ts += float("0." + parts[0].split(".")[1]) if "." in parts[0] else 0.0
                rows.append((ts, float(parts[1]), float(parts[2]), float(parts[3]), int(parts[4], 16)))
            except (ValueError, IndexError):
                continue
        os.unlink(self.path)
        if not rows:
            return None
        inside = [r for r in rows if self.t0 - 0.06 <= r[0] <= self.t1 + 0.06] or rows
        busy = [r for r in inside if not (r[4] & 0x1)] or inside
        reasons = set()
        for r in inside:
            for bit, name in REASONS.items():
                if r[4] & bit and bit != 0x1:
                    reasons.add(name)
        return {"sm_mhz": statistics.median(r[1] for r in busy), "sm_max_mhz": max(r[2] for r in inside),
                "reasons": sorted(reasons), "samples": len(inside),
                "power_w_max": max(r[3] for r in inside)}


def measured_peak():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(path) as f:
            return float(json.load(f)["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy)"
    except (OSError, KeyError, ValueError):
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def ncu_traffic(config, algs, flags=0):
    """dram bytes per expand launch and the algorithmic bytes of the SAME launches,
    from the newest committed ncu summary of this config (profiles/r03, else r02:
    expand_traffic_*.json, tools/traffic_summary.py), if any."""
    for rnd in ("r03", "r02"):
        # engine flags change the launches (e.g. NO_UDC): their own capture, if any
        suffix = f"_flags{flags}" if flags else ""
        path = os.path.join(ROOT, "profiles", rnd, f"expand_traffic_{config}_{'+'.join(algs)}{suffix}.json")
        try:
            with open(path) as f:
                d = json.load(f)
            return d, os.path.relpath(path, ROOT)
        except (OSError, ValueError):
            continue
    return None, None


def l2_roofline(tr, tr_path, avg_launch_ms):
    """The expand's second roofline: L2 requests from the SMs per second against
    the chip's measured ceiling for random 4-byte requests (tools/gather_bench.cu,
    committed as profiles/r03/l2_ceiling.json).  Requests per launch come from the
    ncu capture of the same launches as `traffic`; the time per launch is this
    run's CUDA-event mean.  None when either input is missing."""
    if not tr or not tr.get("l2_requests_per_launch"):
        return None
    try:
        with open(os.path.join(ROOT, "profiles", "r03", "l2_ceiling.json")) as f:
            ceil = json.load(f)
    except (OSError, ValueError):
        return None
    achieved = tr["l2_requests_per_launch"] / (avg_launch_ms * 1e-3) / 1e9
    return {"unit": "G requests/s", "achieved": achieved, "ceiling": ceil["ceiling_g_per_s"],
            "frac": achieved / ceil["ceiling_g_per_s"], "requests_per_launch": tr["l2_requests_per_launch"],
            "requests_per_edge": tr.get("l2_requests_per_edge"),
            "source": f"{tr_path} (lts__t_requests_srcunit_tex.sum); ceiling: {ceil['source']}"}


# --------------------------------------------------------------------------- #
# workload
# --------------------------------------------------------------------------- #
def build_workload(cfg, device, algs):
    import graphgen as gg
    g = gg.make(cfg, device=device, weights=("sssp" in algs))
    gs = gg.make(cfg, device=device, symmetric=True, weights=False) if "cc" in algs else None
    return g, gs


class pinned_core:
    """Run the oracle pinned to one host core (single-threaded,
    one core), restoring the previous affinity afterwards."""

    def __enter__(self):
        self.old = os.sched_getaffinity(0)
        self.core = max(self.old)
        os.sched_setaffinity(0, {self.core})
        return self

    def __exit__(self, *exc):
        os.sched_setaffinity(0, self.old)


def select_sources(cands, reached, n, count):
    """SURVEY A-7 / PAPER.md L249 ("make sure the queried traversal is
    untrivial"): keep the seeded candidates (out-degree >= 1) whose traversal
    reaches at least 1 % of the vertices, in order, up to `count`.
    `reached(s)` -> (vertices reached, edges of the activatable subgraph)."""
    keep, m_reach = [], {}
    for s in cands:
        v, e = reached(s)
        if v >= 0.01 * n:
            keep.append(s)
            m_reach[s] = e
            if len(keep) == count:
                break
    if not keep:
        raise RuntimeError("no candidate source reaches 1 % of the vertices")
    return keep, m_reach


def oracle_sources(g, off, col, count, seed):
    """A-7 sources chosen with the oracle's own BFS (the reference arm never
    touches the GPU path)."""
    import numpy as np
    import graphgen as gg
    import oracle
    deg = np.diff(off.astype(np.int64))

    def reached(s):
        lab = oracle.bfs(off, col, s)
        r = lab != oracle.INF
        return int(r.sum()), int(deg[r].sum())
    return select_sources(gg.sample_sources(g, 4 * count, seed), reached, g.n, count)


def cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown CPU"


def oracle_leg(cfg, algs, nsrc, seed, budget_s=25.0, g=None, gs=None, srcs=None):
    """Time the CPU oracle on a bounded sample: the algorithms of one step, from
    as many sources as fit in ``budget_s`` (at least one).  Returns (edges, seconds, sample)."""
    import numpy as np
    import graphgen as gg
    import oracle
    if g is None:
        g, gs = build_workload(cfg, "cuda" if _has_cuda() else "cpu", algs)
    off, col, w = g.to("cpu").numpy()
    deg = np.diff(off.astype(np.int64))
    srcs, _ = oracle_sources(g, off, col, nsrc, seed) if srcs is None else (srcs, None)
    edges = 0
    secs = 0.0
    done = []
    if gs is not None:
        soff, scol, _ = gs.to("cpu").numpy()
    k = 0
    while True:
        s = srcs[k % len(srcs)]
        for a in algs:
            with pinned_core():
                t = time.perf_counter()
                if a == "bfs":
                    lab = oracle.bfs(off, col, s)
                elif a == "sssp":
                    lab = oracle.sssp(off, col, w, s)
                else:
                    lab = oracle.cc(soff, scol)
                secs += time.perf_counter() - t
            if a == "cc":
                edges += int(scol.shape[0])
            else:
                edges += int(deg[lab != oracle.INF].sum())
            done.append(a if a == "cc" else f"{a}(s={s})")
        k += 1
        if secs >= budget_s or k >= len(srcs):
            break
    return edges, secs, ", ".join(done)


def _has_cuda():
    try:
        import torch
        return torch.cuda.is_available()
    except ImportError:
        return False


def config_desc(cfg):
    import graphgen as gg
    p = gg.CONFIGS[cfg]
    if p["kind"] == "rmat":
        return f"{cfg}: RMAT scale-{p['scale']} ef{p['edge_factor']} (PaRMAT a/b/c=.45/.22/.22), seed {p['seed']}"
    return f"{cfg}: Chung-Lu n={p['n']} m~{p['m_target']} (alpha_out {p['alpha_out']}, alpha_in {p['alpha_in']})"


# --------------------------------------------------------------------------- #
# arms
# --------------------------------------------------------------------------- #
def run_reference(args):
    """The oracle as the reference arm: step i runs ONE call of the step's
    algorithm set (algs[i % len(algs)], rotating sources), so a default run
    stays within a few minutes on one host core."""
    import numpy as np
    import graphgen as gg
    import oracle
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    algs = args.algs.split(",")
    g, gs = build_workload(args.config, "cuda" if _has_cuda() else "cpu", algs)
    off, col, w = g.to("cpu").numpy()
    deg = np.diff(off.astype(np.int64))
    if gs is not None:
        soff, scol, _ = gs.to("cpu").numpy()
    srcs, _ = oracle_sources(g, off, col, args.sources, 4242)
    edges, secs, done = 0, 0.0, []
    for i in range(args.warmup + args.steps):
        a = algs[i % len(algs)]
        s = srcs[(i // len(algs)) % len(srcs)]
        if i < args.warmup and i > 0:
            continue                       # nothing to warm on the CPU beyond one call
        with pinned_core():
            t = time.perf_counter()
            if a == "bfs":
                lab = oracle.bfs(off, col, s)
            elif a == "sssp":
                lab = oracle.sssp(off, col, w, s)
            else:
                lab = oracle.cc(soff, scol)
            dt = time.perf_counter() - t
        if i < args.warmup:
            continue
        secs += dt
        edges += int(scol.shape[0]) if a == "cc" else int(deg[lab != oracle.INF].sum())
        done.append(a)
    value = edges / secs / 1e9
    counts = {a: done.count(a) for a in algs}
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": secs * 1e3 / args.steps,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u32",
        "data": "synthetic",
        "config": {"workload": config_desc(args.config) + "; " + "+".join(algs) + " per step",
                   "n": g.n, "m": g.m},
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": 1, "kind": "oracle",
                         "sample": f"one oracle call per step, rotating {'/'.join(algs)} and sources: "
                                   f"{counts} calls on {args.config}; single-threaded C oracle (gcc -O3) pinned "
                                   f"to 1 of {os.cpu_count()} host cores ({cpu_model()})"},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


def run_ours(args):
    import numpy as np
    import torch
    import torch.distributed as tdist
    import graphgen as gg
    import paper_conf_ipps_wangzlg19_b200 as etg
    from paper_conf_ipps_wangzlg19_b200 import _build

    if not torch.cuda.is_available():
        print(json.dumps({"metric": METRIC, "error": "no CUDA device (etg has no CPU fallback)"}))
        return 1
    rank, world, local = dist_setup()
    if rank == 0:
        _build.build()
    barrier(world)
    dev = torch.device("cuda", torch.cuda.current_device())
    algs = args.algs.split(",")
    g, gs = build_workload(args.config, dev, algs)

    def mk(graph, flags, sym=False):
        o, c, w, fl = etg.csr_to_device(graph.off, graph.col, graph.w, device=dev)
        if args.host_edges:
            c = c.cpu().pin_memory()
            w = None if w is None else w.cpu().pin_memory()
            fl |= etg.HOST_EDGES
        return etg.Graph(o, c, w, n=graph.n, K=args.K, flags=flags | fl | args.flags, symmetric=sym,
                         sssp_delta=args.sssp_delta)

    G = mk(g, 0)
    Gs = mk(gs, 0, sym=True) if gs is not None else None
    out = torch.empty(g.n, dtype=torch.int32, device=dev)
    # sources per SURVEY A-7 and m of their activatable subgraphs (outside the timed region)

    def reached(s):
        st = G.reach_stats(G.bfs(s, out)[0])
        return int(st.vertices_reached), int(st.edges_reached)
    sources, m_reach = select_sources(gg.sample_sources(g, 4 * args.sources, 4242 + 7919 * rank),
                                      reached, g.n, args.sources)
    m_sym = gs.m if gs is not None else 0
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    stream = torch.cuda.current_stream()

    def call(alg, s, handle_main, handle_sym):
        if alg == "bfs":
            return handle_main.bfs(s, out)[1], m_reach[s]
        if alg == "sssp":
            return handle_main.sssp(s, out)[1], m_reach[s]
        return handle_sym.cc(out)[1], m_sym

    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in algs]

    def step(i, acc):
        s = sources[i % len(sources)]
        for k, a in enumerate(algs):
            flush.zero_()
            evs[k][0].record(stream)
            st, edges = call(a, s, G, Gs)
            evs[k][1].record(stream)
            torch.cuda.synchronize()
            if acc is not None:
                ms = evs[k][0].elapsed_time(evs[k][1])
                acc[a]["ms"] += ms
                acc[a]["edges"] += edges
                acc[a]["calls"] += 1
                acc[a]["rates"].append(edges / ms / 1e6)

    for i in range(args.warmup):
        step(i, None)
    clocks = ClockSampler(torch.cuda.current_device()) if rank == 0 else None
    if clocks:
        clocks.start()
        time.sleep(0.3)
    acc = {a: {"ms": 0.0, "edges": 0, "calls": 0, "rates": []} for a in algs}
    launches0 = etg.kernel_launches()
    barrier(world)
    torch.cuda.synchronize()
    if clocks:
        clocks.mark("t0")
    for i in range(args.steps):
        step(args.warmup + i, acc)
    torch.cuda.synchronize()
    barrier(world)
    if clocks:
        clocks.mark("t1")
    launches = etg.kernel_launches() - launches0
    clk = clocks.stop() if clocks else None

    my_ms = sum(v["ms"] for v in acc.values())
    my_edges = sum(v["edges"] for v in acc.values())
    max_ms = allreduce([my_ms], tdist.ReduceOp.MAX if world > 1 else None, world)[0]
    tot_edges = allreduce([float(my_edges)], tdist.ReduceOp.SUM if world > 1 else None, world)[0]
    per_alg = {}
    for a in algs:
        ms_a = allreduce([acc[a]["ms"]], tdist.ReduceOp.MAX if world > 1 else None, world)[0]
        e_a = allreduce([float(acc[a]["edges"])], tdist.ReduceOp.SUM if world > 1 else None, world)[0]
        rates = acc[a]["rates"]
        per_alg[a] = {"gteps": e_a / ms_a / 1e6, "ms_per_call": acc[a]["ms"] / max(1, acc[a]["calls"]),
                      # per call (one source each): Graph500-style harmonic mean, min, max
                      "gteps_per_call_hmean": len(rates) / sum(1.0 / r for r in rates) if rates else None,
                      "gteps_per_call_min": min(rates) if rates else None,
                      "gteps_per_call_max": max(rates) if rates else None}
    value = tot_edges / max_ms / 1e6

    # ---- roofline pass: CUDA events around every expand launch (ETG_PROFILE) ----
    roof = None
    if not args.no_profile:
        Gp = mk(g, etg.PROFILE)
        Gsp = mk(gs, etg.PROFILE, sym=True) if gs is not None else None
        bytes_tot, exp_ms, scan_ms, call_ms, launches_p = 0, 0.0, 0.0, 0.0, 0
        per = {}
        for i in range(args.steps):
            s = sources[(args.warmup + i) % len(sources)]
            for a in algs:
                flush.zero_()
                torch.cuda.synchronize()
                st, _ = call(a, s, Gp, Gsp)
                b = BYTES_PER_EDGE[a] * st.edges_processed + BYTES_PER_VERTEX[a] * st.frontier_total
                bytes_tot += b
                exp_ms += st.expand_ms
                scan_ms += st.scan_ms
                call_ms += st.ms
                launches_p += st.expand_launches
                d = per.setdefault(a, {"bytes": 0, "expand_ms": 0.0, "launches": 0, "edges_processed": 0})
                d["bytes"] += b
                d["expand_ms"] += st.expand_ms
                d["launches"] += st.expand_launches
                d["edges_processed"] += st.edges_processed
        peak, peak_src = measured_peak()
        achieved = bytes_tot / (exp_ms * 1e-3) / 1e9
        tr, tr_path = ncu_traffic(args.config, algs, args.flags)
        roof = {"bound": "hbm", "kernel": "expand_warp_kernel", "achieved": achieved, "peak": peak,
                "unit": "GB/s", "frac": achieved / peak,
                "traffic": tr["dram_bytes_per_launch"] if tr else None,
                "traffic_note": (f"ncu dram read+write bytes per expand launch, mean over all {tr['launches']} "
                                 f"expand launches of one call per algorithm ({tr_path}); algorithmic bytes per "
                                 f"launch of those same launches: {tr['alg_bytes_per_launch']:.0f} "
                                 f"(dram/algorithmic = {tr['dram_over_alg']:.2f})") if tr else None,
                "peak_source": peak_src,
                # SURVEY 8(d)'s pass criterion is the expand kernel's achieved DRAM GB/s: the
                # ncu traffic of the same launches over their (serialised) durations
                "dram_gbs_ncu": tr["dram_gbs_under_ncu"] if tr else None,
                "dram_frac_ncu": tr["dram_gbs_under_ncu"] / peak if tr else None,
                "algorithmic_bytes_per_launch": bytes_tot / max(1, launches_p),
                "avg_launch_ms": exp_ms / max(1, launches_p),
                "expand_share_of_call": exp_ms / max(1e-9, call_ms),
                "scan_share_of_call": scan_ms / max(1e-9, call_ms),
                "bytes_model": "BFS 8 B/edge + 20 B/active vertex; SSSP 12 + 24; CC 8 + 24 (SURVEY 8(d))",
                "timing": "CUDA events on the handle stream around each expand launch (ETG_PROFILE "
                          "host-driven pass over the same steps)",
                "per_alg": {a: {"achieved_gbs": v["bytes"] / (v["expand_ms"] * 1e-3) / 1e9,
                                "launches": v["launches"],
                                "edges_processed": v["edges_processed"]} for a, v in per.items()}}
        roof["l2"] = l2_roofline(tr, tr_path, exp_ms / max(1, launches_p))
        Gp.close()
        if Gsp:
            Gsp.close()

    # ---- e2e: the same metric through the C ABI on HOST buffers ----
    e2e = None
    if not args.no_e2e:
        def pinned(graph):
            o, c, w, fl = etg.csr_to_device(graph.off, graph.col, graph.w, device="cpu")
            return (o.pin_memory(), c.pin_memory(), None if w is None else w.pin_memory())
        hg = pinned(g)
        hgs = pinned(gs) if gs is not None else None
        travs = [a for a in algs if a != "cc"]        # traversals of the directed graph, one H2D for all
        hout = torch.empty(max(1, len(travs)) * g.n, dtype=torch.int32).pin_memory()
        scratch = torch.empty(etg.host_scratch_bytes(g.n, max(g.m, m_sym), True, args.K),
                              dtype=torch.uint8, device=dev)
        ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e_ms, e_edges, h2d, d2h = 0.0, 0, 0, 0
        alg_id = {"bfs": etg.BFS, "sssp": etg.SSSP, "cc": etg.CC}
        for i in range(args.steps):
            s = sources[(args.warmup + i) % len(sources)]
            calls = []
            if travs:
                calls.append(("dir", hg, [(alg_id[a], s) for a in travs]))
            if "cc" in algs:
                calls.append(("sym", hgs, [(etg.CC, 0)]))
            for kind, (o, c, w), queries in calls:
                ww = w if (kind == "dir" and "sssp" in travs) else None
                flush.zero_()
                torch.cuda.synchronize()
                ev0.record(stream)
                etg.run_host_batch(queries, o, c, ww, hout, scratch, K=args.K, flags=args.flags,
                                   sssp_delta=args.sssp_delta, symmetric=(kind == "sym"))
                ev1.record(stream)
                torch.cuda.synchronize()
                e_ms += ev0.elapsed_time(ev1)
                e_edges += m_sym if kind == "sym" else m_reach[s] * len(queries)
                if i == 0:
                    h2d += o.numel() * o.element_size() + c.numel() * 4 + (ww.numel() * 4 if ww is not None else 0)
                    d2h += g.n * 4 * len(queries)
        e_max = allreduce([e_ms], tdist.ReduceOp.MAX if world > 1 else None, world)[0]
        e_tot = allreduce([float(e_edges)], tdist.ReduceOp.SUM if world > 1 else None, world)[0]
        e2e = {"value": e_tot / e_max / 1e6, "unit": UNIT, "h2d_bytes_per_step": h2d,
               "d2h_bytes_per_step": d2h,
               "how": "etg_run_host_batch on pinned host CSRs: per step the directed CSR (off/col/w) crosses "
                      "the host link once for BFS and SSSP (weights copied while BFS runs), the symmetric "
                      "CSR once for CC; every query's labels copied back (overlapping the next query)"}

    # ---- CPU oracle baseline (rank 0, N = 1 only) ----
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        e, secs, sample = oracle_leg(args.config, algs, args.sources, 4242, budget_s=12.0, g=g, gs=gs,
                                     srcs=sources)
        cpu = {"value": e / secs / 1e9, "unit": UNIT, "cores": 1, "kind": "oracle",
               "sample": f"{sample} on {args.config} (single-threaded C oracle, gcc -O3, pinned to 1 of "
                         f"{os.cpu_count()} host cores, {cpu_model()})"}

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": max_ms / args.steps, "higher_is_better": True,
            # N > 1 partitions this same workload (strong scaling) unless --replicas
            "scaling": "weak" if (args.replicas and world > 1) else "strong",
            "vs_baseline": None, "dtype": "u32", "data": "synthetic",
            "config": {"workload": config_desc(args.config) + "; " + "+".join(algs) + " per step",
                       "n": g.n, "m": g.m, "m_sym": m_sym, "K": args.K, "flags": args.flags,
                       "sssp_schedule": (f"wave, Delta={args.sssp_delta}" if str(args.sssp_delta) != "0"
                                         else "paper (Proc. 1)"),
                       "sources": f"{len(sources)} seeded, each reaching >= 1 % of V (SURVEY A-7)",
                       "l2": "flushed (256 MiB write) before every traversal call; col/w 4 B x m each > 126 MB L2",
                       "parallelism": f"{world} independent replica(s), own sources per rank",
                       "sha256": {g.name + "+w" if g.w is not None else g.name: g.sha256(),
                                  **({gs.name: gs.sha256()} if gs is not None else {})}},
            "per_alg": per_alg,
            "roofline": roof,
            "cpu_baseline": cpu,
            "e2e": e2e,
            "gpu_launches": launches,
            "clocks": clk,
        }
        s = json.dumps(line)
        print(s, flush=True)
        if args.json_out:
            with open(args.json_out, "w") as f:
                f.write(s + "\n")
    if world > 1:
        tdist.destroy_process_group()
    return 0


def run_partitioned(args):
    """The N=1 workload split over the N ranks: per algorithm
    one communicator handle per rank (1-D destination partition; --push: SSSP/CC
    on a source partition), every call the whole partitioned loop inside the
    library.  Strong scaling: the same traversals, sources and edges at every N."""
    import numpy as np
    import torch
    import torch.distributed as tdist
    import graphgen as gg
    import paper_conf_ipps_wangzlg19_b200 as etg
    from paper_conf_ipps_wangzlg19_b200 import _build, dist as edist

    rank, world, local = dist_setup()
    if rank == 0:
        _build.build()
    barrier(world)
    dev = torch.device("cuda", torch.cuda.current_device())
    comm = edist.comm_from_group(rank, world, device=dev.index)
    algs = args.algs.split(",")
    alg_id = {"bfs": etg.BFS, "sssp": etg.SSSP, "cc": etg.CC}
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    stream = torch.cuda.current_stream()
    res, e2e_acc = {}, {"ms": 0.0, "edges": 0, "h2d": 0, "d2h": 0}
    launches = 0
    clocks = ClockSampler(dev.index) if rank == 0 else None
    clk_started = False
    shas = {}
    # sources per SURVEY A-7, the same as the N = 1 run (seed 4242), chosen with
    # a partitioned BFS (collective: every rank takes the same decisions)
    g0 = gg.make(args.config, device=dev, weights=False)
    deg0 = g0.degrees()
    dg0 = edist.DistGraph(g0.off, g0.col, None, g0.n, comm, K=args.K, device=dev)
    out0 = torch.empty(max(1, dg0.hi - dg0.lo), dtype=torch.int32, device=dev)

    def reached(s):
        lab, _ = dg0.run(etg.BFS, s, out0)
        r = lab[:dg0.hi - dg0.lo] != -1
        v, e = allreduce([float(r.sum()), float(deg0[dg0.lo:dg0.hi][r].sum())], tdist.ReduceOp.SUM, world)
        return int(v), int(e)
    sources, m_reach_all = select_sources(gg.sample_sources(g0, 4 * args.sources, 4242), reached, g0.n,
                                          args.sources)
    dg0.close()
    del dg0, g0, deg0, out0
    torch.cuda.empty_cache()
    for a in algs:
        g = gg.make(args.config, device=dev, weights=(a == "sssp"), symmetric=(a == "cc"))
        if rank == 0:
            shas[g.name + ("+w" if g.w is not None else "")] = g.sha256()
        exchange = "push" if (args.push and a != "bfs") else "dest"
        dg = edist.DistGraph(g.off, g.col, g.w, g.n, comm, exchange=exchange, K=args.K, flags=args.flags,
                             symmetric=(a == "cc"), sssp_delta=args.sssp_delta, device=dev)
        lo, hi = dg.lo, dg.hi
        m_sym = g.m
        del g
        torch.cuda.empty_cache()
        out = torch.empty(max(1, hi - lo), dtype=torch.int32, device=dev)
        m_reach = {s: (m_sym if a == "cc" else m_reach_all[s]) for s in sources}
        # warm-up, then the timed calls: per call the library's device time, max over ranks
        ms_tot, edges_tot = 0.0, 0
        for i in range(args.warmup + args.steps):
            s = sources[i % len(sources)]
            if i == args.warmup:
                if clocks and not clk_started:
                    clocks.start()
                    time.sleep(0.3)
                    clk_started = True
                l0 = etg.kernel_launches()
                barrier(world)
                torch.cuda.synchronize()
                if clocks and clocks.t0 is None:
                    clocks.mark("t0")
            flush.zero_()
            torch.cuda.synchronize()
            _, st = dg.run(alg_id[a], s, out)
            if i >= args.warmup:
                ms_tot += st.ms
                edges_tot += m_reach[s]
        torch.cuda.synchronize()
        barrier(world)
        launches += etg.kernel_launches() - l0
        # e2e: the same calls from pinned HOST buffers -- H2D of this rank's
        # sub-CSR into the buffers the handle borrows, the call, D2H of the owned slice
        if not args.no_e2e:
            dev_bufs = [t for t in dg.graph._keep[:3] if t is not None]
            host_bufs = [t.cpu().pin_memory() for t in dev_bufs]
            hout = torch.empty(max(1, hi - lo), dtype=torch.int32).pin_memory()
            ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            for i in range(args.steps):
                s = sources[(args.warmup + i) % len(sources)]
                flush.zero_()
                barrier(world)
                torch.cuda.synchronize()
                ev0.record(stream)
                for d, h in zip(dev_bufs, host_bufs):
                    d.copy_(h, non_blocking=True)
                dg.run(alg_id[a], s, out)
                hout.copy_(out, non_blocking=True)
                ev1.record(stream)
                torch.cuda.synchronize()
                e_ms = allreduce([ev0.elapsed_time(ev1)], tdist.ReduceOp.MAX, world)[0]
                e2e_acc["ms"] += e_ms
                e2e_acc["edges"] += m_reach[s]
                if i == 0:
                    e2e_acc["h2d"] += int(allreduce([float(sum(h.numel() * 4 for h in host_bufs))],
                                                    tdist.ReduceOp.SUM, world)[0])
                    e2e_acc["d2h"] += 4 * dg.n                 # the owned slices of all ranks
            del host_bufs, dev_bufs
        res[a] = {"gteps": edges_tot / ms_tot / 1e6, "ms_per_call": ms_tot / args.steps, "edges": edges_tot,
                  "ms": ms_tot, "exchange": exchange}
        dg.close()
        del dg
        torch.cuda.empty_cache()
    if clocks:
        clocks.mark("t1")
    clk = clocks.stop() if clocks else None
    launches = int(allreduce([float(launches)], tdist.ReduceOp.SUM, world)[0])
    tot_e = sum(v["edges"] for v in res.values())
    tot_ms = sum(v["ms"] for v in res.values())
    if rank == 0:
        line = {
            "metric": METRIC, "value": tot_e / tot_ms / 1e6, "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": tot_ms / args.steps,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "u32",
            "data": "synthetic",
            "config": {"workload": config_desc(args.config) + "; " + "+".join(algs) + " per step",
                       "parallelism": (f"1-D vertex partition over {world} rank(s) "
                                       f"({'SSSP/CC source partition + fused push exchange, BFS destination' if args.push else 'destination'} "
                                       "partition), exchange by the library's kernels into the peers' device memory "
                                       "(CUDA IPC; NVLink between GPUs), host barrier per iteration; "
                                       f"{torch.cuda.device_count()} visible device(s)"),
                       "K": args.K, "flags": args.flags,
                       "sources": f"{len(sources)} seeded, each reaching >= 1 % of V (SURVEY A-7), as at N = 1",
                       "sssp_schedule": (f"wave, Delta={args.sssp_delta} (auto from the global sums)"
                                         if str(args.sssp_delta) != "0" else "paper (Proc. 1)"),
                       "l2": "flushed (256 MiB write) before every traversal call",
                       "timing": "per call: the library's CUDA-event device time, max over ranks (etg_stats.ms)",
                       "sha256": shas},
            "per_alg": {k: {"gteps": v["gteps"], "ms_per_call": v["ms_per_call"], "exchange": v["exchange"]}
                        for k, v in res.items()},
            "roofline": None,
            "cpu_baseline": None,
            "e2e": ({"value": e2e_acc["edges"] / e2e_acc["ms"] / 1e6, "unit": UNIT,
                     "h2d_bytes_per_step": e2e_acc["h2d"], "d2h_bytes_per_step": e2e_acc["d2h"],
                     "how": "per rank: H2D of its sub-CSR from pinned host memory into the handle's buffers, "
                            "the call, D2H of the owned label slice; max over ranks"}
                    if not args.no_e2e and e2e_acc["ms"] > 0 else None),
            "gpu_launches": launches,
            "clocks": clk,
        }
        out_s = json.dumps(line)
        print(out_s, flush=True)
        if args.json_out:
            with open(args.json_out, "w") as f:
                f.write(out_s + "\n")
    comm.close()
    if tdist.is_initialized():
        tdist.destroy_process_group()
    return 0


def main():
    args = parse_args()
    world = int(os.environ.get("WORLD_SIZE", "0"))
    if args.impl == "reference":
        return run_reference(args)
    if args.gpus > 1 and world == 0:
        return relaunch(args)                  # no torchrun around us: become N ranks
    if world > 1 and not args.replicas:
        return run_partitioned(args)
    return run_ours(args)


if __name__ == "__main__":
    sys.exit(main())
