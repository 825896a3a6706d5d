#!/usr/bin/env python
"""Throughput of the Core Graph 2Phase hot path on B200 (BASELINE.json metric:
"queries/s and GTEPS (CG-2Phase vs full graph) at 1/2/4/8 B200; %HBM peak").

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config c2] [--batch B]
    python -m torch.distributed.run --nproc-per-node N --master-addr 127.0.0.1 bench.py --gpus N
    python bench.py --impl reference      # the CPU oracle arm (no reference code exists)

A step = one pass of the query hot path (init, phase 1 on the
Core Graph, impacted-set seeding, phase 2 on G, values written) for a batch of B sources of
EACH of the six kinds on the config's synthetic graph (configs[1] = LiveJournal-shaped RMAT
by default).  The graph and its Core Graphs are built once before timing (a1-a7, reported as
build_ms); the paper builds the CG once for "all future queries".
Multi-GPU: sources are sharded (each rank its own batch, graph replicated, weak scaling);
with --gather (default when N > 1) every step's values are gathered to rank 0 over NCCL.
Prints ONE JSON line on rank 0.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import tempfile
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

KINDS = ("sssp", "sswp", "ssnp", "viterbi", "bfs", "reach")
INIT = {"sssp": 0xFFFFFFFF, "sswp": 0, "ssnp": 0xFFFFFFFF, "viterbi": 0, "bfs": 0xFFFFFFFF, "reach": 0}
METRIC = "queries/s (CG-2Phase, all six kinds)"


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=10)
    p.add_argument("--warmup", type=int, default=3)
    p.add_argument("--config", default="c2")
    p.add_argument("--batch", type=int, default=32, help="sources per kind per step (per GPU)")
    p.add_argument("--K", type=int, default=20, help="Core Graph hubs")
    p.add_argument("--kinds", default=",".join(KINDS))
    p.add_argument("--impl", default="native", choices=["native", "reference"])
    p.add_argument("--gather", type=int, default=-1, help="gather values to rank 0 (default: on when N>1)")
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--cpu-sample", type=int, default=0, help="oracle queries in the cpu_baseline sample")
    return p.parse_args()


# ---------------------------------------------------------------------------- helpers
def load_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy test)"
    except Exception:  # noqa: BLE001
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def load_traffic(config):
    """dram bytes per launch of the query kernel from the committed ncu summary, if any."""
    path = os.path.join(ROOT, "profiles", "ncu_query_kernel.json")
    try:
        with open(path) as f:
            d = json.load(f)
        return d.get(config)
    except Exception:  # noqa: BLE001
        return None


class ClockSampler:
    """nvidia-smi sampling DURING the timed region (B200_PROFILING.md clocks line)."""
    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")
    NAMES = ("hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.proc = None
        self.file = None

    def start(self):
        try:
            self.file = tempfile.NamedTemporaryFile("w+", delete=False, suffix=".csv")
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=self.file, stderr=subprocess.DEVNULL)
            time.sleep(0.3)
        except Exception:  # noqa: BLE001
            self.proc = None

    def stop(self):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        self.proc.wait()
        self.file.close()
        rows = []
        with open(self.file.name) as f:
            for line in f:
                parts = [x.strip() for x in line.split(",")]
                if len(parts) == 7:
                    rows.append(parts)
        os.unlink(self.file.name)
        sm = [float(r[0]) for r in rows if r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in rows if r[1].replace(".", "").isdigit()]
        reasons = sorted({self.NAMES[i] for r in rows for i in range(4) if r[3 + i].lower() == "active"})
        load = [x for x in sm if x > 500] or sm
        return {"sm_mhz": statistics.median(load) if load else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(rows)}


def dist_setup():
    import torch
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if ws > 1:
        import torch.distributed as dist
        torch.cuda.set_device(local)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    return rank, ws, local




def host_edges(cfg):
    import gen
    return gen.rmat(cfg.n, cfg.m, cfg.abcd, cfg.w_max, cfg.seed)


def sources_for(cand, kind_idx, count, rank, world=1):
    """Rank's contiguous shard of the kind's global seeded source list (count per rank: weak
    scaling over independent vertex queries).  cand = gen.source_candidates(...)."""
    import gen
    from paper_conf_eurosys_0002a0a024_b200 import multi
    allsrc = gen.sample_from(cand, count * world, seed=1000 + 17 * kind_idx)
    a, b = multi.shard(len(allsrc), rank, world)
    return allsrc[a:b]


def device_candidates(n, src_d, dst_d):
    """gen.source_candidates computed on the device twin's (bit-identical) raw edge list."""
    import torch
    has = torch.zeros(n, dtype=torch.bool, device=src_d.device)
    keep = src_d.view(torch.int32) != dst_d.view(torch.int32)
    has[src_d.view(torch.int32)[keep].to(torch.int64)] = True
    return torch.nonzero(has).flatten().to(torch.int64).cpu().numpy().astype(np.uint32)


# ---------------------------------------------------------------------------- CPU oracle arm
def oracle_inputs(cfg, src_h, dst_h, w_h):
    """The oracle's canonical CSR and the source candidates, from the HOST generator's edges."""
    import gen
    import oracle
    t0 = time.time()
    og = oracle.canonical_csr(cfg.n, src_h, dst_h, w_h)
    cand = gen.source_candidates(cfg.n, src_h, dst_h)
    return og, cand, time.time() - t0


def cpu_oracle_run(cfg, src_h, dst_h, w_h, kinds, per_kind, rank=0, prepared=None):
    """Time the oracle (as it stands: label-setting Dijkstra per kind, one source per OpenMP
    thread) on a bounded sample of the same workload.  Returns (queries/s, cores, sample, seconds)."""
    import oracle
    og, cand, build_s = prepared or oracle_inputs(cfg, src_h, dst_h, w_h)
    cores = os.cpu_count() or 1
    total_q, total_t = 0, 0.0
    for kind in kinds:
        srcs = sources_for(cand, KINDS.index(kind), per_kind, rank)
        t0 = time.perf_counter()
        oracle.query_batch(kind, og, srcs, nthreads=cores)
        total_t += time.perf_counter() - t0
        total_q += len(srcs)
    sample = (f"{per_kind} sources x {len(kinds)} kinds ({total_q} queries) of {cfg.name}, oracle Dijkstra, "
              f"{cores} OpenMP threads, one source per thread; oracle CSR build {build_s:.1f}s untimed")
    return total_q / total_t, cores, sample, total_t


def workload_config(cfg, m_canonical, kinds, batch, K, ws, gather, l2):
    """The `config` object of both arms' JSON lines."""
    return {"workload": cfg.name, "n": cfg.n, "m_generated": cfg.m, "m_canonical": m_canonical,
            "rmat_abcd": list(cfg.abcd), "w_max": cfg.w_max, "seed": cfg.seed, "kinds": kinds,
            "batch_per_kind_per_gpu": batch, "K_hubs": K, "hub_policy": "topdeg", "l2": l2,
            "parallelism": f"source-sharded x{ws}, graph replicated", "gather": gather}


def run_reference(args):
    """The reference arm: there is no reference implementation (the reference is the paper), so
    this times the oracle as it stands on the host cores — W untimed warm-up steps, then exactly
    K timed steps, each a bounded sample (per-kind sources) of the workload; rank 0 alone."""
    import gen
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    cfg = gen.CONFIGS[args.config]
    kinds = [k for k in args.kinds.split(",") if k]
    src_h, dst_h, w_h = host_edges(cfg)
    prepared = oracle_inputs(cfg, src_h, dst_h, w_h)
    del src_h, dst_h, w_h
    cores = os.cpu_count() or 1
    per_kind = args.cpu_sample or max(1, min(cores, 16) // 2)  # as the native arm's cpu_baseline
    for _ in range(args.warmup):
        cpu_oracle_run(cfg, None, None, None, kinds, per_kind, rank, prepared)
    total_t, total_q, sample = 0.0, 0, ""
    for _ in range(args.steps):
        qps, cores, sample, t = cpu_oracle_run(cfg, None, None, None, kinds, per_kind, rank, prepared)
        total_t += t
        total_q += per_kind * len(kinds)
    v = total_q / total_t
    gws = max(1, args.gpus)
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": "queries/s", "n_gpus": gws,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1000.0 * total_t / args.steps,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u32 (f32 Viterbi)",
            "data": "synthetic",
            "config": workload_config(cfg, prepared[0].m, kinds, args.batch, args.K, gws, False,
                                      "host oracle (no GPU); CSR %.0f MB" % (8 * prepared[0].m / 1e6)),
            "cpu_baseline": {"value": v, "unit": "queries/s", "cores": cores, "kind": "oracle",
                             "sample": sample + f"; per step, {args.steps} timed steps after {args.warmup} warm-up"},
            "e2e": {"value": v, "unit": "queries/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


# ---------------------------------------------------------------------------- native arm
def main():
    args = parse()
    if args.impl == "reference":
        return run_reference(args)
    import torch

    import gen
    from paper_conf_eurosys_0002a0a024_b200 import Graph, kernel_launches, multi, rmat_device

    rank, ws, local = dist_setup()
    dev = torch.device("cuda", local)
    torch.cuda.set_device(dev)
    cfg = gen.CONFIGS[args.config]
    kinds = [k for k in args.kinds.split(",") if k]
    B = args.batch
    gather = (ws > 1) if args.gather < 0 else bool(args.gather)
    if args.warmup < 3:
        args.warmup = 3  # timing rule: >= 3 warm-up steps

    # ---- inputs (untimed): the device twin of the generator for the graph and the source
    # candidates; host edges only for the oracle's cpu_baseline (rank 0, N = 1)
    t0 = time.time()
    need_host = rank == 0 and ws == 1 and not args.no_cpu_baseline
    src_h = dst_h = w_h = None
    if need_host:
        src_h, dst_h, w_h = host_edges(cfg)
    src_d, dst_d, w_d = rmat_device(cfg.n, cfg.m, cfg.abcd, cfg.w_max, cfg.seed, True, dev)
    cand = device_candidates(cfg.n, src_d, dst_d)
    g = Graph(cfg.n, src_d, dst_d, w_d, device=dev)
    del src_d, dst_d, w_d
    torch.cuda.synchronize()
    graph_s = time.time() - t0
    build = {}
    for kind in kinds:
        if kind == "bfs" and "reach" in build:
            build["bfs"] = dict(build["reach"])
            continue
        build[kind] = g.build(kind, K=args.K)
    ptr = g.export(ptr_only=True)[0]
    outdeg = (ptr[1:] - ptr[:-1]).to(torch.int64)
    del ptr
    srcs = {k: torch.from_numpy(sources_for(cand, KINDS.index(k), B, rank, ws).astype(np.int64))
            .to(torch.uint32).to(dev) for k in kinds}
    nbuf = 2 if gather else 1
    outs = [{k: torch.empty((B, cfg.n), dtype=torch.uint32, device=dev) for k in kinds} for _ in range(nbuf)]
    stream = torch.cuda.current_stream(dev)

    def barrier():
        if ws > 1:
            import torch.distributed as dist
            dist.barrier()
        torch.cuda.synchronize(dev)

    gathered = None
    if gather and rank == 0:
        gathered = {k: [torch.empty((B, cfg.n), dtype=torch.uint32, device=dev) for _ in range(ws)] for k in kinds}

    resident_bytes = 4 * g.m + 64 * cfg.n  # packed CSR + one batch's value rows
    flush = torch.empty(64 << 20, dtype=torch.int32, device=dev) if resident_bytes < 126e6 else None

    def run_step(mode, slot, events=None, works=None):
        o = outs[slot]
        for k in kinds:
            if events is not None:
                events[k][0].record(stream)
            g.query(k, srcs[k], mode=mode, out=o[k])
            if events is not None:
                events[k][1].record(stream)
        if gather and works is not None:
            for k in kinds:
                _, wk = multi.gather_rows(o[k], rank, ws, gathered[k] if rank == 0 else None, async_op=True)
                works.append(wk)

    def timed(mode, steps, with_events=True):
        for i in range(args.warmup):
            run_step(mode, i % nbuf, works=[] if gather else None)
        barrier()
        evs = [{k: (torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for k in kinds}
               for _ in range(steps)] if with_events else [None] * steps
        start, end = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        l0 = kernel_launches()
        works = [] if gather else None
        if flush is not None:
            # L2-resident config: flush L2 between timed steps (a 256 MB write outside the
            # step's events) and sum the per-step device times
            sev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(steps)]
            for i in range(steps):
                flush.fill_(i)
                sev[i][0].record(stream)
                run_step(mode, i % nbuf, evs[i], works)
                sev[i][1].record(stream)
            if works:
                for wk in works:
                    wk.wait()
            barrier()
            launches = kernel_launches() - l0
            ms = multi.max_over_ranks(sum(a.elapsed_time(b) for a, b in sev), dev)
            per_kind_ms = {k: [e[k][0].elapsed_time(e[k][1]) for e in evs] for k in kinds} if with_events else None
            return ms, per_kind_ms, launches
        start.record(stream)
        for i in range(steps):
            run_step(mode, i % nbuf, evs[i], works)
        if works:
            for wk in works:
                wk.wait()
        end.record(stream)
        barrier()
        launches = kernel_launches() - l0
        ms = multi.max_over_ranks(start.elapsed_time(end), dev)
        per_kind_ms = {k: [e[k][0].elapsed_time(e[k][1]) for e in evs] for k in kinds} if with_events else None
        return ms, per_kind_ms, launches

    # ---- 2Phase (headline), with clocks sampled during the timed region
    clk = ClockSampler(local)
    clk.start()
    ms2, kms2, launches = timed("2phase", args.steps)
    clocks = clk.stop()
    q_step = B * len(kinds)
    qps2 = ws * q_step * args.steps / (ms2 / 1000.0)
    # ---- FULL baseline on the same batch
    msf, kmsf, _ = timed("full", args.steps)
    qpsf = ws * q_step * args.steps / (msf / 1000.0)

    # ---- GTEPS numerator (Graph500: edges whose tail is reachable), results of the last step
    m_reach = 0
    for k in kinds:
        o = outs[(args.steps - 1) % nbuf][k]
        init_i32 = int(np.array([INIT[k]], dtype=np.uint32).view(np.int32)[0])
        mask = (o.view(torch.int32) != init_i32).to(torch.int64)
        m_reach += int((mask * outdeg.unsqueeze(0)).sum().item())
    gteps2 = ws * m_reach * args.steps / (ms2 / 1000.0) / 1e9
    gtepsf = ws * m_reach * args.steps / (msf / 1000.0) / 1e9

    # ---- per-query counters (untimed): algorithmic bytes, EDGES-RED, p1 precision
    per_kind = {}
    alg_bytes_2p = {}
    eb = 4 if (int(cfg.n - 1).bit_length() + int(cfg.w_max - 1).bit_length()) <= 32 else 8  # packed edge word?
    for k in kinds:
        _, p1, st2 = g.query(k, srcs[k], mode="2phase", p1=True, stats=True)
        del p1
        _, stf = g.query(k, srcs[k], mode="full", stats=True)
        e2 = sum(s["edges_p1"] + s["edges_p2"] for s in st2)
        ef = sum(s["edges_p2"] for s in stf)
        reached = sum(s["reached"] for s in st2)
        precise = sum(s["precise_p1"] for s in st2)

        def bytes_of(sts, two_phase):
            # algorithmic bytes of the batched query kernel, per pass of Qb queries
            # with RB-byte value rows (cg_stats.batch_queries / row_bytes): rows initialised
            # (n RB) and masks cleared (4 n); per union-frontier vertex 8 B of row offsets + its
            # RB row + 3x4 B list entry written and read; per union edge one edge word (4 B packed
            # / 8 B wide) + v's RB row; per EdgeFunction a 4 B atomic; the impacted scan (2Phase,
            # n RB); the transpose out (n RB read + 4 n per query written)
            tot, i = 0, 0
            while i < len(sts):
                qb, rb = max(1, sts[i]["batch_queries"]), sts[i]["row_bytes"]
                grp = sts[i:i + qb]
                i += qb
                fr = grp[0]["frontier_p1"] + grp[0]["frontier_p2"]  # union frontier (same for the batch)
                sc = sum(s["scanned_p1"] + s["scanned_p2"] for s in grp)
                up = sum(s["updates_p1"] + s["updates_p2"] for s in grp)
                tot += cfg.n * rb + 4 * cfg.n + fr * (8 + rb + 24) + sc * (eb + rb) + 4 * up
                tot += (cfg.n * rb if two_phase else 0) + cfg.n * rb + 4 * cfg.n * len(grp)
            return tot
        alg_bytes_2p[k] = bytes_of(st2, True)
        mean2 = statistics.mean(kms2[k])
        meanf = statistics.mean(kmsf[k])
        per_kind[k] = {
            "qps_2phase": B / (mean2 / 1000.0), "qps_full": B / (meanf / 1000.0),
            "speedup": meanf / mean2, "ms_2phase": mean2, "ms_full": meanf,
            "edges_2phase_per_q": e2 / B, "edges_full_per_q": ef / B,
            "edges_red_pct": 100.0 * (1 - e2 / ef) if ef else None,
            "p1_precision_pct": 100.0 * precise / reached if reached else None,
            "cg_edge_pct": 100.0 * build[k]["edge_fraction"], "cg_build_ms": build[k]["build_ms"],
            "iters_p1": statistics.mean(s["iters_p1"] for s in st2),
            "iters_p2": statistics.mean(s["iters_p2"] for s in st2),
            "iters_full": statistics.mean(s["iters_p2"] for s in stf),
            "alg_GBps": alg_bytes_2p[k] / (mean2 / 1000.0) / 1e9,
        }

    # ---- roofline of the dominant kernel (the persistent query kernel; one launch per kind)
    peak, peak_src = load_peaks()
    tot_bytes = sum(alg_bytes_2p.values())
    tot_ms = sum(statistics.mean(kms2[k]) for k in kinds)
    achieved = tot_bytes / (tot_ms / 1000.0) / 1e9
    tr = load_traffic(cfg.name)
    # ncu dram bytes of one query_kernel launch of this bench (B queries), from the committed
    # per-query figure (profiles/ncu_query_kernel.json); None when no capture exists
    traffic = tr["dram_bytes_per_query"] * B if tr else None
    roofline = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                "traffic": traffic, "kernel": "batch_kernel<KIND,packed,lanes> (one launch per kind per step)",
                "peak_source": peak_src,
                "alg_bytes_per_launch": tot_bytes / len(kinds),
                "achieved_how": "algorithmic bytes (cg_stats counters, DESIGN.md §7) summed over the kinds' "
                                "launches / their summed CUDA-event durations on the launching stream",
                "traffic_how": (tr["how"] + " (" + tr["report"] + ")") if tr else None}

    # ---- NEXT-3 WCC (a whole-graph query, reported beside the six-kind headline): 2Phase on
    # REACH's general CG vs FULL, device-timed, same warm-up rule
    wcc = None
    if "reach" in build:
        wout = torch.empty((1, cfg.n), dtype=torch.uint32, device=dev)
        wms = {}
        for mode in ("2phase", "full"):
            for _ in range(args.warmup):
                g.query("wcc", None, mode=mode, out=wout)
            barrier()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            for _ in range(args.steps):
                g.query("wcc", None, mode=mode, out=wout)
            e1.record(stream)
            barrier()
            wms[mode] = multi.max_over_ranks(e0.elapsed_time(e1), dev) / args.steps
        _, wp1, wst = g.query("wcc", None, mode="2phase", p1=True, stats=True)
        n_comp = int(torch.unique(wout[0].to(torch.int64)).numel())
        wcc = {"ms_2phase": wms["2phase"], "ms_full": wms["full"], "speedup": wms["full"] / wms["2phase"],
               "components": n_comp, "iters_p1": wst[0]["iters_p1"], "iters_p2": wst[0]["iters_p2"],
               "p1_precision_pct": 100.0 * wst[0]["precise_p1"] / max(1, wst[0]["reached"])}
        del wp1

    # ---- e2e through the public API with HOST buffers (pinned), copies inside the timed region
    e2e = None
    if not args.no_e2e:
        import torch as _t
        hsrc = {k: srcs[k].to(_t.int64).cpu() for k in kinds}
        hout = {k: _t.empty((B, cfg.n), dtype=_t.uint32, pin_memory=True) for k in kinds}
        for _ in range(1):
            for k in kinds:
                g.query_host(k, hsrc[k], mode="2phase", out=hout[k])
        barrier()
        t0 = time.perf_counter()
        steps_e2e = max(1, min(args.steps, 5))
        for _ in range(steps_e2e):
            for k in kinds:
                g.query_host(k, hsrc[k], mode="2phase", out=hout[k])
        barrier()
        el = multi.max_over_ranks(time.perf_counter() - t0, dev)
        e2e = {"value": ws * q_step * steps_e2e / el, "unit": "queries/s", "h2d_bytes_per_step": 4 * q_step,
               "d2h_bytes_per_step": 4 * q_step * cfg.n, "api": "cg_query_host (pinned host buffers)",
               "steps": steps_e2e}

    # ---- CPU baseline: the oracle on the host cores, bounded sample (rank 0, N=1 only)
    cpu = None
    if rank == 0 and ws == 1 and not args.no_cpu_baseline:
        cores = os.cpu_count() or 1
        per_kind_n = args.cpu_sample or max(1, min(cores, 16) // 2)
        v, cores, sample, _ = cpu_oracle_run(cfg, src_h, dst_h, w_h, kinds, per_kind_n)
        cpu = {"value": v, "unit": "queries/s", "cores": cores, "kind": "oracle", "sample": sample}

    if rank == 0:
        line = {
            "metric": METRIC, "value": qps2, "unit": "queries/s", "n_gpus": ws, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms2 / args.steps, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "u32 (f32 Viterbi)", "data": "synthetic",
            "config": workload_config(cfg, g.m, kinds, B, args.K, ws, gather,
                                      ("inputs larger than L2 (packed CSR + value rows %.0f MB > 126 MB L2)"
                                       % (resident_bytes / 1e6) if flush is None else
                                       "L2 flushed between timed steps (256 MB write outside the step events; "
                                       "inputs %.0f MB)" % (resident_bytes / 1e6))),
            "gteps": gteps2, "full": {"value": qpsf, "unit": "queries/s", "gteps": gtepsf, "ms_per_step": msf / args.steps},
            "speedup_2phase_vs_full": qpsf and qps2 / qpsf,
            "per_kind": per_kind, "wcc": wcc, "roofline": roofline, "cpu_baseline": cpu, "e2e": e2e,
            "gpu_launches": launches, "clocks": clocks,
            "build_ms": {k: build[k]["build_ms"] for k in build}, "graph_build_s": graph_s,
        }
        print(json.dumps(line), flush=True)
    if ws > 1:
        import torch.distributed as dist
        dist.barrier()
        dist.destroy_process_group()
    g.close()
    return 0


if __name__ == "__main__":
    sys.exit(main())
