#!/usr/bin/env python
"""TempGraph on B200 -- benchmark harness (one JSON line on rank 0).

Metric (BASELINE.json): EAT queries/s & temporal-edges/s at 1/2/4/8 B200, HBM GB/s
against the peak.  The metric's 1/2/4/8-GPU wording is quoted on configs[3] ("C4"),
which is the default workload: R-MAT 2^24 vertices / 536,870,912 temporal edges,
t ~ U[0, 2^16), duration ~ U[1, 16], ONE 1024-source earliest-arrival batch, full
window, sharded by source across the ranks (1024/N sources per rank: strong scaling,
no data-path collective).  `--config C2|C3|C5` selects the other configs.

A step is one pass of the whole hot path over the step's
input: tg_graph_create from the device-resident edge arrays (validate),
tg_build_chains (sort, departure nodes, hubs, chains, shortcuts, occurrence index;
+ the LD mirror when the config has LD), then tg_query for every problem of the
config over this rank's sources (activation, chain relaxation, rounds, extraction
into device-resident outputs), then destroy.
`value` = (queries answered by all ranks per step) / (max-over-ranks ms/step).

--impl reference: the oracle (oracle/, the paper's one-pass scans) on the box's host
cores, one query per thread, same metric / unit / config.
"""
from __future__ import annotations

import argparse
import json
import os
import platform
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

HBM_FALLBACK_GBS = 6650.0  # B200_PROFILING.md fallback, used only without MEASURED_PEAKS.json
METRIC = "temporal-path queries/s (EAT; plus LD/FP/SP where the config lists them)"
UNIT = "queries/s"
RELAX_KERNELS = ("k_eat_rounds", "k_spfp_rounds", "k_eat_activate", "k_eat_big", "k_eat_chain", "k_reach_scan", "k_reach_big", "k_spfp_activate",
                 "k_spfp_wait", "k_spfp_big")


def parse_args(argv=None):
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--config", default="C4")
    ap.add_argument("--k", type=int, default=None,
                    help="sources per problem of the WHOLE job (default: the config's batch)")
    ap.add_argument("--scaling", choices=["strong", "weak"], default="strong",
                    help="strong: the job's batch is split across ranks; weak: every rank answers k sources")
    ap.add_argument("--sub-batch", type=int, default=0)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-profile", action="store_true", help="do not bracket kernels with CUDA events")
    ap.add_argument("--profile-all", action="store_true",
                    help="bracket every kernel with CUDA events (default: only the relaxation kernels)")
    ap.add_argument("--query-only", action="store_true", help="time only tg_query (graph built once)")
    ap.add_argument("--mode", choices=["replicate", "vertex"], default="replicate",
                    help="multi-GPU mode: replicate = source sharding; vertex = one batch partitioned by "
                         "vertex range with per-round ncclAllReduce(min)")
    ap.add_argument("--partitions", type=int, default=1, help="logical vertex-range partitions per GPU")
    ap.add_argument("--exchange", type=int, default=0, help="vertex mode: cross-rank exchange algorithm")
    ap.add_argument("--cpu-threads", type=int, default=0, help="oracle threads (0 = all host cores)")
    ap.add_argument("--problems", default=None, help="comma list overriding the config's problems (e.g. reach)")
    ap.add_argument("--reach-bits", action="store_true", help="TG_REACH on the bit-lane engine (option reach_bits)")
    ap.add_argument("--stream-blocks", type=int, default=0,
                    help="out-of-memory mode: the graph streamed from host memory in this many time blocks")
    return ap.parse_args(argv)


# --------------------------------------------------------------------------- helpers
def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy kernel read+write bytes)"
    return HBM_FALLBACK_GBS, "fallback (B200_PROFILING.md)"


def host_facts():
    cpu = platform.processor() or ""
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                cpu = line.split(":", 1)[1].strip()
                break
    except OSError:
        pass
    ram = None
    try:
        for line in open("/proc/meminfo"):
            if line.startswith("MemTotal"):
                ram = round(int(line.split()[1]) / 2**20, 1)
                break
    except OSError:
        pass
    return {"cpu_model": cpu, "host_cores": os.cpu_count(), "ram_GiB": ram}


class ClockSampler:
    """NVML sampling of SM clock and throttle reasons during the timed region."""

    REASONS = {
        0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap", 0x8: "hw_slowdown",
        0x10: "sync_boost", 0x20: "sw_thermal_slowdown", 0x40: "hw_thermal_slowdown",
        0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting",
    }

    def __init__(self, device_index):
        self.interval = float(os.environ.get("BENCH_CLOCK_INTERVAL", "0.02"))
        self.samples = []
        self.reasons = set()
        self.max_mhz = None
        self.ok = False
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(device_index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception as e:  # pragma: no cover - no NVML on CPU boxes
            self.err = str(e)
        self._stop = threading.Event()

    def _run(self):
        while not self._stop.is_set():
            try:
                mhz = self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM)
                r = self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                self.samples.append(mhz)
                for bit, name in self.REASONS.items():
                    if r & bit and name not in ("gpu_idle",):
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(self.interval)

    def start(self):
        if self.ok:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()

    def stop(self):
        if self.ok:
            self._stop.set()
            self.t.join()
        return {"sm_mhz": (statistics.median(self.samples) if self.samples else None),
                "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons), "samples": len(self.samples)}


# --------------------------------------------------------------------------- workload
def plan_sources(job_sources, rank, world, scaling, mode):
    """This rank's sources.  strong: the job's batch split into contiguous rank blocks;
    weak: rank r answers its own block of len(job_sources) sources (the caller passes a
    job list world times longer); vertex mode: every rank answers the whole batch."""
    from paper_conf_asplos_0003wh0dhwy0lyl25_b200.distributed import shard_sources
    if mode == "vertex":
        return list(job_sources)
    return shard_sources(job_sources, rank, world)


def workload(cfg_name, k_job, rank, world, device, mode="replicate", scaling="strong"):
    import tgsynth
    cfg = tgsynth.CONFIGS[cfg_name]
    ge = tgsynth.make_graph(cfg_name, device=device)
    k = k_job if k_job else cfg["k"]
    want = k * (world if (scaling == "weak" and mode == "replicate") else 1)
    job = tgsynth.config_sources(cfg_name, ge, k=want)
    if len(job) < want:  # single-source configs asked for more: cycle
        job = (job * (want // max(1, len(job)) + 1))[:want]
    mine = plan_sources(job, rank, world, scaling, mode)
    problems = list(cfg["problems"]) or ["eat"]
    if getattr(workload, "problems", None):
        problems = list(workload.problems)
    win = cfg["windows"][0]
    weighted = cfg["kind"] == "wikitalk"
    return ge, job, mine, problems, win, weighted, cfg


def describe(cfg_name, ge, k_job, problems, win, world, scaling, mode):
    """Workload line of the JSON config (starts with the config name)."""
    share = ("every rank answers the whole batch cooperatively (vertex range)" if mode == "vertex" else
             (f"{k_job}/{world} per rank" if scaling == "strong" else f"{k_job} per rank"))
    return (f"{cfg_name}: {ge.meta.get('config')} n={ge.n} m={ge.m}; one {k_job}-source batch per problem "
            f"({'+'.join(problems)}; {share}), window [{win[0]}, {win[1]}]")


ORACLE_FN = {"eat": "eat", "ld": "ld", "fp": "fp", "fastest": "fp", "sp": "sp", "shortest": "sp",
             "reach": "reach"}


def oracle_call(og, problem, x, win):
    import oracle
    return getattr(oracle, ORACLE_FN[problem])(og, x, *win)


def oracle_allcore(og, problems, sources, win, threads):
    """One oracle query per host thread (ctypes drops the GIL inside the C scans).
    Returns (wall seconds, per-query seconds list)."""
    from concurrent.futures import ThreadPoolExecutor
    tasks = [(p, x) for x in sources for p in problems]
    per = [0.0] * len(tasks)

    def run(i):
        p, x = tasks[i]
        t0 = time.perf_counter()
        oracle_call(og, p, x, win)
        per[i] = time.perf_counter() - t0

    t0 = time.perf_counter()
    with ThreadPoolExecutor(max_workers=threads) as ex:
        list(ex.map(run, range(len(tasks))))
    return time.perf_counter() - t0, per


# --------------------------------------------------------------------------- our arm
def run_ours(a, rank, world, local_rank):
    import torch
    import torch.distributed as dist

    import paper_conf_asplos_0003wh0dhwy0lyl25_b200 as tg

    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
    ge, job, mine, problems, win, weighted, cfg = workload(a.config, a.k, rank, world, dev, a.mode, a.scaling)
    if not weighted:
        ge.w = None  # weights are not part of this workload (w = duration, reading A7)
    torch.cuda.synchronize()
    torch.cuda.empty_cache()  # generator temporaries: give them back before the library allocates
    k = len(mine)
    k_job = len(job)
    n, m = ge.n, ge.m
    w_arg = ge.w if weighted else None
    outs = {p: torch.empty((k, n), dtype=torch.int32, device=dev) for p in problems}
    torch.cuda.synchronize()
    host_edges = None
    if a.stream_blocks:  # out-of-memory mode: the library takes HOST arrays and streams time blocks
        host_edges = [x.cpu() for x in (ge.u, ge.v, ge.t, ge.dur)] + [ge.w.cpu() if weighted else None]
    comm = None
    if a.mode == "vertex":
        from paper_conf_asplos_0003wh0dhwy0lyl25_b200.distributed import make_comm
        comm = make_comm(rank, world, local_rank, bcast_device=dev)

    def make_graph():
        if host_edges is not None:
            g = tg.Graph(n, *host_edges, device=local_rank, block_edges=m // a.stream_blocks + 1)
            return g.build()
        g = tg.Graph(n, ge.u, ge.v, ge.t, ge.dur, w_arg, device=local_rank)
        if a.sub_batch:
            g.set_option("sub_batch", a.sub_batch)
        if "ld" not in problems:
            g.set_option("mirror", 0)
        if a.partitions > 1:
            g.set_option("partitions", a.partitions)
        if a.exchange:
            g.set_option("exchange", 1)
        if a.reach_bits:
            g.set_option("reach_bits", 1)
        if comm is not None:
            tg.tg_graph_attach_comm(g.h, comm, 1)
        return g.build()

    persistent = make_graph() if a.query_only else None

    def step():
        g = persistent or make_graph()
        for p in problems:
            g.query(p, mine, win, out=outs[p])
        if persistent is None:
            g.close()

    def barrier():
        if world > 1:
            dist.barrier()

    # warm-up: exactly W steps (with the in-library event profiling on when it will be on
    # in the timed region: the event pool then already holds the events it records)
    plevel = 0 if a.no_profile else (1 if a.profile_all else 2)
    if plevel:
        tg.tg_profile_enable(plevel)
    for _ in range(max(a.warmup, 0)):
        step()
    torch.cuda.synchronize()
    tg.tg_profile_enable(False)
    tg.tg_profile_report()  # recycle the warm-up's events into the pool

    # work counts (untimed): W per query from the engine's first-touch counter (== oracle W, tested)
    gstat = persistent or make_graph()
    gstat.set_option("stats", 1)
    W_by_problem, Wu_by_problem, SPFP = {}, {}, {}
    for p in problems:
        if p == "reach" and a.reach_bits:
            # the bit-lane engine's usable edges are the EAT union of the same batch
            gstat.query("eat", mine, win, out=outs[p])
            Wu_by_problem[p] = int(gstat.last_stats(k)["slots_union"])
            continue
        if p in ("sp", "fp", "lds"):
            # node-state engine: chain-slot relaxations and wait-edge steps
            gstat.query(p, mine, win, out=outs[p])
            st = gstat.last_stats(k)
            SPFP[p] = (int(st["slots_relaxed"]), int(st["slots_union"]))
            continue
        if p not in ("eat", "ld", "reach"):
            continue  # the first-touch work counters cover the EAT-family engine
        gstat.query(p, mine, win, out=outs[p])
        st = gstat.last_stats(k)
        W_by_problem[p] = int(st["per_query_relax"].sum())
        Wu_by_problem[p] = int(st["slots_union"])
    gstat.set_option("stats", 0)
    rounds = {}
    for p in problems:
        gstat.query(p, mine, win, out=outs[p])
        rounds[p] = gstat.last_stats()["rounds"]
    info = gstat.info()
    if persistent is None:
        gstat.close()
    torch.cuda.synchronize()
    W_local = sum(W_by_problem.values())
    W_global = float(W_local)
    if world > 1:
        t = torch.tensor([W_global], dtype=torch.float64, device=dev)
        dist.all_reduce(t)  # every rank's own sources (vertex mode: its own partition's relaxations)
        W_global = float(t.item())

    # timed region: EXACTLY a.steps steps between barrier + synchronize on both sides, CUDA
    # events on the stream all our kernels run on (the legacy default stream), NVML clocks
    # sampled during the region
    prof = plevel != 0
    sampler = ClockSampler(local_rank)
    if prof:
        tg.tg_profile_report()  # clear
        tg.tg_profile_enable(plevel)
    launches0 = tg.tg_kernel_launch_count()
    barrier()
    torch.cuda.synchronize()
    sampler.start()
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    e0.record()
    marks = []
    for _ in range(a.steps):
        step()
        ev = torch.cuda.Event(enable_timing=True)
        ev.record()
        marks.append(ev)
    e1.record()
    torch.cuda.synchronize()
    barrier()
    clocks = sampler.stop()
    step_ms = [round(e0.elapsed_time(marks[0]), 3)] + [round(marks[i - 1].elapsed_time(marks[i]), 3)
                                                       for i in range(1, len(marks))]
    launches = tg.tg_kernel_launch_count() - launches0
    kprof = tg.tg_profile_report() if prof else {}
    tg.tg_profile_enable(False)
    ms = e0.elapsed_time(e1) / a.steps
    if world > 1:
        t = torch.tensor([ms], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())

    queries_per_step = k_job * len(problems)  # the whole job: every rank's share (or the shared batch)
    value = queries_per_step / (ms / 1e3)

    # roofline of the dominant kernel group: the relax phase (this rank's launches)
    peak, peak_src = peaks()
    roof = None
    if kprof:
        # concurrent query lanes: the round-loop graphs overlap in time, so the relax phase
        # counts their union (the wall time some lane's round loop ran), not their sum
        union = kprof.pop("k_eat_rounds_union", None)
        relax_names = [x for x in kprof if x.startswith(RELAX_KERNELS)]
        relax_ms = sum(kprof[x][1] for x in relax_names if not (union and x.startswith("k_eat_rounds")))
        relax_ms += union[1] if union else 0.0
        relax_launches = sum(kprof[x][0] for x in relax_names)
        dom = max(kprof.items(), key=lambda kv: kv[1][1])
        if union:  # overlapping lanes: the round loops' wall time, not their summed durations
            dom = ("k_eat_rounds (graph loops of the query lanes, union of their intervals)", union)
        # SURVEY 8(d), batched with source lanes, at the state width the timed path moves
        # (u32 arrivals: pred = NULL): every slot relaxed by some query of a sub-batch is read
        # once (16 B slot + 4 B occurrence), every relaxation touches 4 B of state:
        # B = 20 B x W_union + 4 B x sum_q W_q.  (The survey's packed 8-B word is reported too.)
        # bit-lane reach (f2): per usable edge one 16-B occurrence record, the 8-B head word
        # and the 8-B tail-node word (64 sources per word); per sub-batch the vertex words
        W_steps = W_local * a.steps
        bits = "reach" in problems and a.reach_bits
        Wu_eat = sum(v for p, v in Wu_by_problem.items() if not (p == "reach" and bits)) * a.steps
        Wu_reach = Wu_by_problem.get("reach", 0) * a.steps if bits else 0
        reach_bytes = (32 * Wu_reach + 8 * n * (-(-k // 64)) * a.steps) if bits else 0
        # SP / FP / LDS: per chain-slot relaxation the 16-B slot, the 4-B tail
        # node id and weight, the 4-B node state and the 4-B vertex output; per wait step the
        # 4-B departure time and the 4-B node state
        spfp_bytes = sum(32 * r + 8 * wst for r, wst in SPFP.values()) * a.steps
        relax_bytes = 20 * Wu_eat + 4 * W_steps + reach_bytes + spfp_bytes
        relax_bytes_pk = 20 * Wu_eat + 8 * W_steps + reach_bytes + spfp_bytes
        Wu_steps = Wu_eat + Wu_reach
        traffic = None
        tf = os.path.join(ROOT, "profiles", "round2", f"relax_traffic_{a.config}.json")
        if os.path.exists(tf) and a.mode == "replicate" and a.partitions == 1 and world == 1 and not a.k:
            traffic = json.load(open(tf))  # ncu on this code for this workload (see the file)
        ach = relax_bytes / (relax_ms / 1e3) / 1e9 if relax_ms else None
        roof = {
            "bound": "hbm",
            "kernel": "relax phase (" + " + ".join(sorted({x.split("<")[0] for x in relax_names})) + ")",
            "achieved": ach,
            "peak": peak,
            "unit": "GB/s",
            "frac": ach / peak if ach else None,
            "traffic": (traffic["dram_bytes_per_step"] if traffic else None),
            "traffic_source": (os.path.relpath(tf, ROOT) + ": " + traffic["source"]) if traffic else None,
            "traffic_vs_algorithmic": (traffic["dram_bytes_per_step"] / (relax_bytes / a.steps)) if traffic else None,
            "ncu_dram_GBps": traffic.get("ncu_GBps") if traffic else None,
            "peak_source": peak_src,
            "algorithmic_bytes_per_step": relax_bytes / a.steps,
            "algorithmic_bytes_formula": ("20 B x W_union + 4 B x sum_q W_q (SURVEY 8(d) batched source lanes, "
                                          "u32 state as timed)") if not ("reach" in problems and a.reach_bits) else
                                         "32 B x W_union + 8 B x n per 64-source word (bit-lane reach, DESIGN 5.5)",
            "algorithmic_bytes_formula_spfp": "32 B x chain-slot relaxations + 8 B x wait steps (SP/FP/LDS)",
            "achieved_packed_8B_formula": relax_bytes_pk / (relax_ms / 1e3) / 1e9 if relax_ms else None,
            "spfp_relax_and_wait_steps_per_step": {p: list(v) for p, v in SPFP.items()},
            "W_union_per_step": Wu_steps / a.steps,
            "W_sum_per_step": W_steps / a.steps,
            "relax_ms_per_step": relax_ms / a.steps,
            "relax_ms_is_union_of_lanes": bool(union),
            "relax_launches_per_step": relax_launches / a.steps,
            "relax_share_of_step": relax_ms / a.steps / ms,
            "dominant_single_kernel": dom[0],
            "dominant_single_kernel_share_of_step": dom[1][1] / a.steps / ms,
            "profiled_kernels": "all" if plevel == 1 else "relaxation kernels only (CUDA events per launch)",
            "kernels_ms_per_step": {x: round(v[1] / a.steps, 4) for x, v in
                                    sorted(kprof.items(), key=lambda kv: -kv[1][1])[:12]},
            "kernels_ms_note": ("summed per-launch durations; the query lanes' round loops overlap, so their sum "
                                "exceeds the step" if union else "summed per-launch durations"),
        }

    if persistent is not None:
        persistent.close()
        persistent = None
    del outs
    torch.cuda.synchronize()
    torch.cuda.empty_cache()
    e2e = None
    if not a.no_e2e and comm is None and not a.stream_blocks:
        e2e = run_e2e(a, tg, ge, mine, k_job, problems, win, weighted, world, dev)

    cpu = None
    if rank == 0 and world == 1 and not a.no_cpu_baseline:
        cpu = cpu_baseline(ge, job, problems, win, weighted, a.cpu_threads)

    res = {
        "metric": METRIC,
        "value": value,
        "unit": UNIT,
        "n_gpus": world,
        "steps": a.steps,
        "warmup": a.warmup,
        "ms_per_step": ms,
        "higher_is_better": True,
        "scaling": ("strong" if (a.scaling == "strong" or a.mode == "vertex") else "weak"),
        "vs_baseline": None,
        "dtype": "u32",
        "data": "synthetic",
        "config": {
            "workload": describe(a.config, ge, k_job, problems, win, world, a.scaling, a.mode),
            "parallelism": ((f"source-sharded x{world} (replicated graph, no data-path collective)"
                             if a.mode == "replicate" else
                             f"vertex-range x{world} (one batch; per-round ncclAllReduce(min) of states)")
                            + (f"; {a.partitions} logical vertex-range partitions per GPU" if a.partitions > 1
                               else "")),
            "step": (("" if a.query_only else
                      "create+validate, build_chains (" + ("fwd+mirror" if "ld" in problems else "fwd") + "), ")
                     + " + ".join(f"{p} x{k}" for p in problems) + " per rank"),
            "query_only": a.query_only,
            "streamed_blocks": info.get("n_blocks", 0) if a.stream_blocks else 0,
            "l2": "inputs larger than L2 (edge list %.0f MB, chain structure %.0f MB > 126 MB)" % (
                m * (20 if weighted else 16) / 1e6, info["device_bytes"] / 1e6),
            "sub_batch": a.sub_batch or "auto",
        },
        "teps_graph": value * m,  # queries/s x |E|: the paper-comparable |E|-normalised rate
        "teps_work": W_global / (ms / 1e3),
        "W_per_query": {p: W_by_problem[p] / k for p in W_by_problem},
        "W_union": Wu_by_problem,
        "rounds": rounds,
        "graph": {"n": n, "m": m, "nodes": info["n_nodes"], "chains": info["n_chains"],
                  "long_chains": info["n_long_chains"], "max_chain_len": info["max_chain_len"],
                  "device_bytes": info["device_bytes"], "build_ms": info["build_ms"]},
        "roofline": roof,
        "cpu_baseline": cpu,
        "e2e": e2e,
        "gpu_launches": launches,
        "clocks": clocks,
        "step_ms": step_ms,
    }
    if comm is not None:
        tg.tg_comm_destroy(comm)
    if world > 1:
        dist.destroy_process_group()
    return res if rank == 0 else None


def run_e2e(a, tg, ge, mine, k_job, problems, win, weighted, world, dev):
    """Same metric through the public C-ABI with HOST buffers: pinned host edge arrays
    -> tg_graph_create (H2D inside) -> build -> tg_query into pinned host outputs (the
    library copies each sub-batch's rows out on a copy stream while the next one runs)."""
    import torch
    n, m = ge.n, ge.m
    k = len(mine)
    hu, hv, ht, hd = (x.cpu().pin_memory() for x in (ge.u, ge.v, ge.t, ge.dur))
    hw = ge.w.cpu().pin_memory() if weighted else None
    houts = {p: torch.empty((k, n), dtype=torch.int32, pin_memory=True) for p in problems}

    def step():
        g = tg.Graph(n, hu, hv, ht, hd, hw, device=dev.index)
        if a.sub_batch:
            g.set_option("sub_batch", a.sub_batch)
        if "ld" not in problems:
            g.set_option("mirror", 0)
        g.build()
        for p in problems:
            tg.tg_query(g.h, tg.PROBLEMS[p], mine, win, houts[p])
        g.close()

    warm = max(1, min(a.warmup, 2))
    for _ in range(warm):
        step()
    torch.cuda.synchronize()
    if world > 1:
        torch.distributed.barrier()
    steps = max(1, min(a.steps, 3))
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(steps):
        step()
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / steps
    if world > 1:
        t = torch.tensor([ms], dtype=torch.float64, device=dev)
        torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
        ms = float(t.item())
    h2d = m * (20 if weighted else 16) + k * 4 * len(problems)
    d2h = len(problems) * k * n * 4
    del houts
    return {"value": k_job * len(problems) / (ms / 1e3), "unit": UNIT, "ms_per_step": ms,
            "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h, "steps": steps, "warmup": warm}


# --------------------------------------------------------------------------- oracle (CPU) legs
def _oracle_graph(ge, weighted):
    import oracle
    n, u, v, t, d, w = ge.numpy()
    return oracle.Graph(n, u, v, t, d, w if weighted else None)


def _oracle_preprocess_seconds(og):
    """The oracle's own preprocessing: the stable time sort its one-pass scans need."""
    t0 = time.perf_counter()
    _ = og.order
    return time.perf_counter() - t0


def cpu_baseline(ge, job, problems, win, weighted, threads=0):
    """The oracle as it stands on the host: its time sort once, then one query per
    problem on ONE core, then one query per core on all cores concurrently (a bounded
    sample of the job's sources); the job's queries/s is extrapolated from the all-core
    throughput plus the sort."""
    og = _oracle_graph(ge, weighted)
    t_sort = _oracle_preprocess_seconds(og)
    cores = threads or os.cpu_count() or 1
    one = {}
    for p in problems:
        t0 = time.perf_counter()
        oracle_call(og, p, job[0], win)
        one[p] = time.perf_counter() - t0
    sample = job[1:1 + max(1, cores // len(problems))] or job[:1]
    wall, per = oracle_allcore(og, problems, sample, win, cores)
    q_allcore = len(per) / wall
    k_job = len(job) * len(problems)
    value = k_job / (t_sort + k_job / q_allcore)
    return {"value": value, "unit": UNIT, "cores": cores, "kind": "oracle",
            "sample": (f"oracle time sort once ({t_sort:.2f} s); 1 query per problem on 1 core "
                       f"({', '.join(f'{p} {one[p]:.3f} s' for p in problems)}); {len(per)} queries "
                       f"({len(sample)} sources x {'+'.join(problems)}) on {cores} threads in {wall:.2f} s "
                       f"= {q_allcore:.3f} q/s; value = the job's {k_job} queries / (sort + queries at "
                       f"the all-core rate)"),
            "per_query_1core_s": one, "allcore_queries_per_s": q_allcore, "sort_s": t_sort,
            **host_facts()}


def run_reference(a, rank, world):
    """--impl reference: the oracle on the host cores, each step one oracle query (one
    source x every problem of the config) run one per thread; W warm-up steps, then K
    timed steps; value = K x problems / wall of the timed steps, extrapolated to the
    job with the oracle's own time sort (as in cpu_baseline)."""
    if rank != 0:
        return None
    import torch
    dev = "cuda" if torch.cuda.is_available() else "cpu"
    ge, job, mine, problems, win, weighted, cfg = workload(a.config, a.k, 0, 1, dev, "replicate", a.scaling)
    og = _oracle_graph(ge, weighted)
    wl = describe(a.config, ge, len(job), problems, win, 1, a.scaling, "replicate")
    del ge
    t_sort = _oracle_preprocess_seconds(og)
    cores = a.cpu_threads or os.cpu_count() or 1
    # the K timed steps are spread over the threads in whole waves (at least one query per
    # thread, so every core works); the warm-up is one wave of min(W, cores) queries
    n_timed = -(-max(a.steps, cores) // cores) * cores
    n_warm = min(a.warmup, cores)
    srcs = [job[i % len(job)] for i in range(n_warm + n_timed)]
    if n_warm:
        oracle_allcore(og, problems, srcs[:n_warm], win, cores)
    wall, per = oracle_allcore(og, problems, srcs[n_warm:], win, cores)
    q = len(per) / wall
    k_job = len(job) * len(problems)
    value = k_job / (t_sort + k_job / q)
    sample = (f"{n_timed} timed oracle queries ({a.steps} steps rounded up to whole waves of {cores} threads; "
              f"+{n_warm} warm-up), each one source x ({'+'.join(problems)}) scans, one per thread: "
              f"{wall:.2f} s = {q:.3f} q/s; time sort "
              f"{t_sort:.2f} s once; value = the job's {k_job} queries / (sort + queries at that rate)")
    return {"impl": "reference", "metric": METRIC, "value": value, "unit": UNIT,
            "n_gpus": world, "steps": a.steps, "warmup": a.warmup, "ms_per_step": wall / n_timed * 1e3,
            "higher_is_better": True, "scaling": "strong" if a.scaling == "strong" else "weak",
            "vs_baseline": None, "dtype": "u32", "data": "synthetic",
            "config": {"workload": wl},
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": cores, "kind": "oracle", "sample": sample,
                             "per_query_s_mean": statistics.mean(per), "sort_s": t_sort, **host_facts()},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}


def main():
    os.environ.setdefault("NCCL_DEBUG", "WARN")  # keep NCCL's version banner off stdout (one JSON line)
    a = parse_args()
    if a.problems:
        workload.problems = a.problems.split(",")
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if world == 1 and a.gpus > 1:
        print(json.dumps({"error": "use torchrun --nproc-per-node N for --gpus N > 1"}))
        return 2
    # stdout carries exactly one JSON line: native libraries (NCCL's version banner, ...)
    # print to fd 1, so fd 1 points at stderr while the benchmark runs
    sys.stdout.flush()
    saved = os.dup(1)
    os.dup2(2, 1)
    try:
        res = run_reference(a, rank, world) if a.impl == "reference" else run_ours(a, rank, world, local_rank)
    finally:
        sys.stdout.flush()
        os.dup2(saved, 1)
        os.close(saved)
    if res is not None:
        print(json.dumps(res), flush=True)
    return 0


if __name__ == "__main__":
    sys.exit(main())
