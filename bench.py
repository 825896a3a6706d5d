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

Multi-GPU (vertex queries are independent): `--gpus N` without a
torchrun environment re-launches itself under torch.distributed.run with N ranks.  Every rank
holds a replica of the graph and its Core Graphs.  Headline: each rank evaluates its own B
sources per kind (weak scaling) and, for N > 1, every step's value rows are gathered to rank 0
over NCCL (the path's single exchange; narrow wire format).  `c3_strong`: configs[2]'s fixed
batch of 64 SSSP + 64 SSWP sources on the Twitter-shaped graph, sharded over the N ranks
(strong scaling), gathered to rank 0.  `c1_single`: configs[0], one SSSP query from vertex 0
(µs/query, FULL vs 2PHASE; rank 0, N = 1).  Rank 0 prints ONE JSON line.
"""
from __future__ import annotations

import argparse
import json
import os
import socket
import statistics
import subprocess
import sys
import tempfile
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

KINDS = ("sssp", "sswp", "ssnp", "viterbi", "bfs", "reach")
INIT = {"sssp": 0xFFFFFFFF, "sswp": 0, "ssnp": 0xFFFFFFFF, "viterbi": 0, "bfs": 0xFFFFFFFF, "reach": 0}
METRIC = "queries/s (CG-2Phase, all six kinds)"
# value rows written by the timed queries (cg_out_format): the narrow wire format keeps every
# value exactly (u16 for the integer kinds whose values fit, 1 bit for REACH), u32 for Viterbi
NARROW = {"sssp": "u16", "sswp": "u16", "ssnp": "u16", "viterbi": "u32", "bfs": "u16", "reach": "bits"}
# value lanes the engine computes in (reading N3; results are bit-identical to u32 lanes)
LANES = ("binary16 lanes for SSSP/SSWP/SSNP/BFS (exact integers < 2048, u32 re-run on overflow), "
         "1-bit lanes for REACH, u32 lanes holding binary32 for Viterbi")


def parse(argv=None):
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
    p.add_argument("--out", default="narrow", choices=["narrow", "u32"], help="output rows of the timed queries")
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--no-c3", action="store_true", help="skip the configs[2] strong-scaling leg")
    p.add_argument("--no-c1", action="store_true", help="skip the configs[0] single-query leg")
    p.add_argument("--c3-steps", type=int, default=0, help="timed steps of the c3_strong leg (default min(K, 5))")
    p.add_argument("--cpu-sample", type=int, default=0, help="oracle queries per kind in the cpu_baseline sample")
    return p.parse_args(argv)


# ---------------------------------------------------------------------------- launch
def _free_port() -> int:
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def torchrun_cmd(argv, n: int, port: int) -> list:
    """The command that runs this bench with n ranks on one node (the driver's launch line)."""
    return [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
            "--master-addr=127.0.0.1", f"--master-port={port}", os.path.abspath(__file__), *argv]


def launch_plan(gpus: int, env) -> str:
    """'run' (this process is the rank set), 'relaunch' (spawn N ranks under torchrun) or an error
    message when a torchrun environment disagrees with --gpus."""
    ws = env.get("WORLD_SIZE")
    if ws is None:
        return "relaunch" if gpus > 1 else "run"
    if int(ws) != gpus:
        return f"WORLD_SIZE={ws} but --gpus {gpus}: launch {gpus} ranks or pass --gpus {ws}"
    return "run"


# ---------------------------------------------------------------------------- helpers
def load_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy test)"
    except Exception:  # noqa: BLE001
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def load_ncu(config):
    """Per-kind ncu DRAM bytes / durations of the batch kernel from the committed capture of
    this code (profiles/ncu_kinds.json), if any."""
    try:
        with open(os.path.join(ROOT, "profiles", "ncu_kinds.json")) as f:
            return json.load(f).get(config)
    except Exception:  # noqa: BLE001
        return None


def cpu_model() -> str:
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for line in out.splitlines():
            if line.startswith("Model name:"):
                return line.split(":", 1)[1].strip()
    except Exception:  # noqa: BLE001
        pass
    return "unknown"


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
    sample = (f"the first {per_kind} of each kind's bench sources x {len(kinds)} kinds ({total_q} queries) of "
              f"{cfg.name}, oracle Dijkstra, {cores} OpenMP threads (one source per thread) on {cpu_model()}; "
              f"oracle CSR build {build_s:.1f}s untimed")
    return total_q / total_t, cores, sample, total_t


def workload_config(cfg, m_canonical, kinds, batch, K, ws, gather, l2, out="narrow"):
    """The `config` object of both arms' JSON lines."""
    return {"workload": cfg.name, "n": cfg.n, "m_generated": cfg.m, "m_canonical": m_canonical,
            "rmat_abcd": list(cfg.abcd), "w_max": cfg.w_max, "seed": cfg.seed, "kinds": kinds,
            "batch_per_kind_per_gpu": batch, "K_hubs": K, "hub_policy": "topdeg", "l2": l2,
            "parallelism": f"source-sharded x{ws}, graph replicated", "gather": gather,
            "out_rows": ({k: NARROW[k] for k in kinds} if out == "narrow" else "u32")}


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
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
            "dtype": "u32 / binary32 (the oracle's Table 6 value words)", "data": "synthetic",
            "config": workload_config(cfg, prepared[0].m, kinds, args.batch, args.K, gws, gws > 1,
                                      "host oracle (no GPU); CSR %.0f MB" % (8 * prepared[0].m / 1e6), args.out),
            "cpu_baseline": {"value": v, "unit": "queries/s", "cores": cores, "kind": "oracle",
                             "sample": sample + f"; per step, {args.steps} timed steps after {args.warmup} warm-up"},
            "e2e": {"value": v, "unit": "queries/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


# ---------------------------------------------------------------------------- native arm
class Ctx:
    """Per-process state of the native arm."""

    def __init__(self, args, rank, ws, dev):
        import torch
        self.args, self.rank, self.ws, self.dev = args, rank, ws, dev
        self.stream = torch.cuda.current_stream(dev)

    def barrier(self):
        import torch
        if self.ws > 1:
            import torch.distributed as dist
            dist.barrier()
        torch.cuda.synchronize(self.dev)

    def max_ms(self, ms):
        from paper_conf_eurosys_0002a0a024_b200 import multi
        return multi.max_over_ranks(ms, self.dev)


def timed_steps(ctx, step, steps, warmup, flush=None, per_key=None, finish=None):
    """W untimed warm-up steps, then exactly `steps` timed steps bracketed by barrier + device
    sync; device time on the launching stream (CUDA events), max over ranks.  step(i, evs) runs
    step i (evs: per-key (start, end) events to record inside, or None).  With `flush`, L2 is
    flushed before every timed step (a write larger than L2, outside the step's events) and the
    per-step times are summed.  finish() (e.g. waiting for the last gathers) runs inside the timed
    region after the last step.  Returns (ms total, {key: [ms per step]}, kernel launches)."""
    import torch
    from paper_conf_eurosys_0002a0a024_b200 import kernel_launches
    for i in range(warmup):
        step(i, None)
    if finish is not None:
        finish()
    ctx.barrier()
    mk = lambda: (torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))  # noqa: E731
    evs = [({k: mk() for k in per_key} if per_key else None) for _ in range(steps)]
    sev = [mk() for _ in range(steps)]
    l0 = kernel_launches()
    start, end = mk()
    start.record(ctx.stream)
    for i in range(steps):
        if flush is not None:
            flush.fill_(i)
        sev[i][0].record(ctx.stream)
        step(warmup + i, evs[i])
        if finish is not None and i == steps - 1:
            finish()
        sev[i][1].record(ctx.stream)
    end.record(ctx.stream)
    ctx.barrier()
    launches = kernel_launches() - l0
    total = sum(a.elapsed_time(b) for a, b in sev) if flush is not None else start.elapsed_time(end)
    per = {k: [e[k][0].elapsed_time(e[k][1]) for e in evs] for k in per_key} if per_key else None
    return ctx.max_ms(total), per, launches


def alg_bytes(cfg, sts, two_phase, eb):
    """Algorithmic bytes of the batched query kernel for one call, per pass of Qb
    queries with RB-byte value rows (cg_stats.batch_queries / row_bytes): rows initialised (n RB)
    and masks cleared (4 n); per union-frontier vertex 8 B of row offsets + its RB row + 3 x 4 B
    list entry written and read; per union edge one edge word (eb) + v's RB row; per
    EdgeFunction a 4 B atomic; the impacted scan (2Phase, n RB); the transpose out (n RB read +
    the output row written, 4 B per value in u32 rows)."""
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


def build_graph(cfg, dev):
    """The config's graph from the device twin of the generator (untimed) and its source
    candidates."""
    import torch
    from paper_conf_eurosys_0002a0a024_b200 import Graph, rmat_device
    src_d, dst_d, w_d = rmat_device(cfg.n, cfg.m, cfg.abcd, cfg.w_max, cfg.seed, True, dev)
    cand = device_candidates(cfg.n, src_d, dst_d)
    g = Graph(cfg.n, src_d, dst_d, w_d, device=dev)
    del src_d, dst_d, w_d
    torch.cuda.synchronize()
    torch.cuda.empty_cache()
    return g, cand


def run_c1_single(ctx):
    """BASELINE configs[0]: RMAT scale-16, one SSSP query from vertex 0 with the K = 20 SSSP Core
    Graph — µs per query, FULL vs 2PHASE (the single-query engine; graph L2-resident, L2
    flushed before every timed query)."""
    import torch
    import gen
    cfg = gen.CONFIGS["c1"]
    g, _ = build_graph(cfg, ctx.dev)
    g.build("sssp", K=20)
    v0 = gen.generator_vertex(cfg, 0)  # reading N10: the generator's vertex 0 (the top hub)
    src = torch.full((1,), v0, dtype=torch.int64).to(torch.uint32).to(ctx.dev)
    out = torch.empty((1, cfg.n), dtype=torch.uint32, device=ctx.dev)
    flush = torch.empty(64 << 20, dtype=torch.int32, device=ctx.dev)
    res = {"workload": cfg.name, "query": f"SSSP from the generator's vertex 0 (id {v0}, reading N10)", "K_hubs": 20,
           "l2": "flushed before every timed query (256 MB write outside the events)"}
    steps = 200
    for mode in ("2phase", "full"):
        ms, _, _ = timed_steps(ctx, lambda i, e: g.query("sssp", src, mode=mode, out=out), steps, 20, flush=flush)
        res[f"us_{mode}"] = 1000.0 * ms / steps
    _, st = g.query("sssp", src, mode="2phase", stats=True)
    _, stf = g.query("sssp", src, mode="full", stats=True)
    res.update({"speedup": res["us_full"] / res["us_2phase"], "iters_p1": st[0]["iters_p1"],
                "iters_p2": st[0]["iters_p2"], "iters_full": stf[0]["iters_p2"],
                "edges_2phase": st[0]["edges_p1"] + st[0]["edges_p2"], "edges_full": stf[0]["edges_p2"],
                "cg_edge_pct": 100.0 * g.core_info("sssp")["edge_fraction"]})
    g.close()
    return res


def run_c3_strong(ctx, steps, warmup):
    """BASELINE configs[2]: the Twitter-shaped RMAT (41.7 M vertices, 1.47 B edges), a FIXED
    batch of 64 SSSP + 64 SSWP sources sharded over the N ranks (strong scaling), CG-2Phase and
    FULL, every step's value rows (narrow format) gathered to rank 0."""
    import torch
    import gen
    from paper_conf_eurosys_0002a0a024_b200 import multi
    cfg = gen.CONFIGS["c3"]
    t0 = time.time()
    g, cand = build_graph(cfg, ctx.dev)
    kinds = ("sssp", "sswp")
    build = {k: g.build(k, K=20)["build_ms"] for k in kinds}
    graph_s = time.time() - t0
    srcs, outs = {}, []
    for k in kinds:
        allsrc = gen.sample_from(cand, 64, seed=42 + KINDS.index(k))
        a, b = multi.shard(64, ctx.rank, ctx.ws)
        srcs[k] = torch.from_numpy(allsrc[a:b].astype(np.int64)).to(torch.uint32).to(ctx.dev)
    for _ in range(2):
        outs.append({k: torch.empty((srcs[k].numel(), cfg.n), dtype=torch.uint16, device=ctx.dev) for k in kinds})
    ring = multi.GatherRing(ctx.rank, ctx.ws)
    res = {"workload": cfg.name, "n": cfg.n, "m_canonical": g.m, "queries_per_step": 128,
           "kinds": list(kinds), "scaling": "strong", "n_gpus": ctx.ws, "gather": ctx.ws > 1,
           "out_rows": "u16", "build_ms": build, "graph_build_s": graph_s,
           "l2": "inputs larger than L2 (1.47 B edges)"}
    for mode in ("2phase", "full"):
        def step(i, evs):
            slot = i % 2
            ring.acquire(slot)
            for k in kinds:
                if srcs[k].numel():
                    g.query(k, srcs[k], mode=mode, out=outs[slot][k], fmt="u16")
                ring.submit(slot, k, outs[slot][k])
        ms, _, _ = timed_steps(ctx, step, steps, warmup, finish=ring.drain)
        res[f"ms_per_step_{mode}"] = ms / steps
        res[f"qps_{mode}"] = 128 * steps / (ms / 1000.0)
    g.status()
    res["value"] = res["qps_2phase"]
    res["speedup_2phase_vs_full"] = res["qps_2phase"] / res["qps_full"]
    g.close()
    del outs
    torch.cuda.empty_cache()
    return res


def main(argv=None):
    args = parse(argv)
    if args.impl == "reference":
        return run_reference(args)
    plan = launch_plan(args.gpus, os.environ)
    if plan == "relaunch":
        argv = sys.argv[1:] if argv is None else argv
        return subprocess.call(torchrun_cmd(argv, args.gpus, _free_port()))
    if plan != "run":
        print(f"bench.py: {plan}", file=sys.stderr)
        return 2
    import torch

    import gen
    from paper_conf_eurosys_0002a0a024_b200 import multi

    rank, ws, local = dist_setup()
    dev = torch.device("cuda", local)
    torch.cuda.set_device(dev)
    ctx = Ctx(args, rank, ws, dev)
    cfg = gen.CONFIGS[args.config]
    kinds = [k for k in args.kinds.split(",") if k]
    B = args.batch
    gather = (ws > 1) if args.gather < 0 else bool(args.gather)
    if args.warmup < 3:
        args.warmup = 3  # timing rule: >= 3 warm-up steps
    fmt = {k: (NARROW[k] if args.out == "narrow" else "u32") for k in kinds}

    # ---- inputs (untimed): the device twin of the generator for the graph and the source
    # candidates; host edges only for the oracle's cpu_baseline (rank 0, N = 1)
    t0 = time.time()
    need_host = rank == 0 and ws == 1 and not args.no_cpu_baseline
    src_h = dst_h = w_h = None
    if need_host:
        src_h, dst_h, w_h = host_edges(cfg)
    g, cand = build_graph(cfg, dev)
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

    def alloc_outs(f):
        return {k: torch.empty((B,) + (g.row_shape(f[k])[0],), dtype=g.row_shape(f[k])[1], device=dev) for k in kinds}
    outs = [alloc_outs(fmt), alloc_outs(fmt)]
    ring = multi.GatherRing(rank, ws)
    resident_bytes = 4 * g.m + 64 * cfg.n  # packed CSR + one batch's value rows
    flush = torch.empty(64 << 20, dtype=torch.int32, device=dev) if resident_bytes < 126e6 else None

    def make_step(mode, f, o):
        def step(i, evs):
            slot = i % 2
            if gather:
                ring.acquire(slot)  # step i-2's gather of this slot is done
            for k in kinds:
                if evs is not None:
                    evs[k][0].record(ctx.stream)
                g.query(k, srcs[k], mode=mode, out=o[slot][k], fmt=f[k])
                if evs is not None:
                    evs[k][1].record(ctx.stream)
                if gather:
                    ring.submit(slot, k, o[slot][k])
        return step

    def timed(mode, f=fmt, o=outs):
        # the gathers are inside the timed region: the end event waits for the last ones
        return timed_steps(ctx, make_step(mode, f, o), args.steps, args.warmup, flush, kinds,
                           ring.drain if gather else None)

    # ---- 2Phase (headline), with clocks sampled during the timed region
    clk = ClockSampler(local)
    clk.start()
    ms2, kms2, launches = timed("2phase")
    clocks = clk.stop()
    q_step = B * len(kinds)
    qps2 = ws * q_step * args.steps / (ms2 / 1000.0)
    # ---- FULL baseline on the same batch
    msf, kmsf, _ = timed("full")
    qpsf = ws * q_step * args.steps / (msf / 1000.0)
    g.status()  # no sticky device error (narrow-format overflow, bad source) in the timed runs
    # ---- the same step with the ABI's u32 rows (cg_query's format), for reference
    u32 = None
    if args.out == "narrow":
        f32 = {k: "u32" for k in kinds}
        o32 = [alloc_outs(f32), alloc_outs(f32)]
        ms32, _, _ = timed("2phase", f32, o32)
        u32 = {"value": ws * q_step * args.steps / (ms32 / 1000.0), "ms_per_step": ms32 / args.steps,
               "out_rows": "u32"}
        del o32

    # ---- GTEPS numerator (Graph500: edges whose tail is reachable), one untimed u32 run
    m_reach = 0
    for k in kinds:
        o = g.query(k, srcs[k], mode="2phase")
        init_i32 = int(np.array([INIT[k]], dtype=np.uint32).view(np.int32)[0])
        mask = (o.view(torch.int32) != init_i32).to(torch.int64)
        m_reach += int((mask * outdeg.unsqueeze(0)).sum().item())
        del o, mask
    m_reach = int(multi.max_over_ranks(float(m_reach), dev)) if ws > 1 else m_reach
    gteps2 = ws * m_reach * args.steps / (ms2 / 1000.0) / 1e9
    gtepsf = ws * m_reach * args.steps / (msf / 1000.0) / 1e9

    # ---- per-query counters (untimed): algorithmic bytes, EDGES-RED, p1 precision, phase times
    per_kind, alg_b = {}, {}
    eb = 4 if (int(cfg.n - 1).bit_length() + int(cfg.w_max - 1).bit_length()) <= 32 else 8  # packed edge word?
    for k in kinds:
        _, p1, st2 = g.query(k, srcs[k], mode="2phase", p1=True, stats=True)
        del p1
        _, stf = g.query(k, srcs[k], mode="full", stats=True)
        e2 = sum(s["edges_p1"] + s["edges_p2"] for s in st2)
        ef = sum(s["edges_p2"] for s in stf)
        reached = sum(s["reached"] for s in st2)
        precise = sum(s["precise_p1"] for s in st2)
        alg_b[k] = alg_bytes(cfg, st2, True, eb)
        mean2, meanf = statistics.mean(kms2[k]), statistics.mean(kmsf[k])
        passes = {}
        for s in st2:  # distinct passes: their phase times
            passes.setdefault((s["ms_p1"], s["ms_p2"]), None)
        per_kind[k] = {
            "qps_2phase": B / (mean2 / 1000.0), "qps_full": B / (meanf / 1000.0),
            "speedup": meanf / mean2, "ms_2phase": mean2, "ms_full": meanf,
            "ms_phase1": sum(a for a, _ in passes), "ms_phase2": sum(b for _, b in passes),
            "edges_2phase_per_q": e2 / B, "edges_full_per_q": ef / B,
            "edges_red_pct": 100.0 * (1 - e2 / ef) if ef else None,
            "p1_precision_pct": 100.0 * precise / reached if reached else None,
            "cg_edge_pct": 100.0 * build[k]["edge_fraction"], "cg_build_ms": build[k]["build_ms"],
            "iters_p1": statistics.mean(s["iters_p1"] for s in st2),
            "iters_p2": statistics.mean(s["iters_p2"] for s in st2),
            "iters_full": statistics.mean(s["iters_p2"] for s in stf),
            "alg_bytes": alg_b[k], "alg_GBps": alg_b[k] / (mean2 / 1000.0) / 1e9,
            "lanes": ("u32" if st2[0]["batch_queries"] == 16 else "1-bit" if st2[0]["row_bytes"] == 4 else "binary16"),
            "out_rows": fmt[k],
        }

    # ---- roofline of the dominant kernel (the batch kernel of the kind with the largest share)
    peak, peak_src = load_peaks()
    dom = max(kinds, key=lambda k: per_kind[k]["ms_2phase"])
    d_ms = per_kind[dom]["ms_2phase"]
    achieved = alg_b[dom] / (d_ms / 1000.0) / 1e9
    nc = load_ncu(cfg.name)
    traffic = None
    ncu_kinds = {}
    if nc:
        for k, v in nc.get("kinds", {}).items():
            gbs = v["dram_bytes"] / (v["ms"] / 1000.0) / 1e9
            ncu_kinds[k] = {"dram_GBps": gbs, "dram_frac": gbs / peak, "dram_frac_vs_8TBps": gbs / 8000.0,
                            "ms_ncu": v["ms"], "dram_bytes": v["dram_bytes"]}
        traffic = nc.get("kinds", {}).get(dom, {}).get("dram_bytes")
    roofline = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                "traffic": traffic, "kernel": f"batch_kernel<{dom.upper()}> (one launch per kind per step; "
                                              f"the kind with the largest share of the step)",
                "peak_source": peak_src, "alg_bytes_per_launch": alg_b[dom],
                "achieved_how": "ALGORITHMIC bytes of the launch (cg_stats counters x DESIGN.md §7 per-unit "
                                "bytes; every 64 B row gather counted in full, although about half hit L2) / "
                                "its mean CUDA-event duration on the launching stream",
                "frac_vs_8TBps": achieved / 8000.0,
                "per_kind_alg": {k: {"GBps": per_kind[k]["alg_GBps"], "frac": per_kind[k]["alg_GBps"] / peak}
                                 for k in kinds},
                "per_kind_ncu_dram": ncu_kinds or None,
                "traffic_how": (nc.get("how") if nc else None)}

    # ---- NEXT-3 WCC (a whole-graph query, reported beside the six-kind headline)
    wcc = None
    if "reach" in build:
        wout = torch.empty((1, cfg.n), dtype=torch.uint32, device=dev)
        wms = {}
        for mode in ("2phase", "full"):
            ms, _, _ = timed_steps(ctx, lambda i, e: g.query("wcc", None, mode=mode, out=wout), args.steps,
                                   args.warmup)
            wms[mode] = ms / args.steps
        _, wp1, wst = g.query("wcc", None, mode="2phase", p1=True, stats=True)
        n_comp = int(torch.unique(wout[0].to(torch.int64)).numel())
        wcc = {"ms_2phase": wms["2phase"], "ms_full": wms["full"], "speedup": wms["full"] / wms["2phase"],
               "components": n_comp, "iters_p1": wst[0]["iters_p1"], "iters_p2": wst[0]["iters_p2"],
               "p1_precision_pct": 100.0 * wst[0]["precise_p1"] / max(1, wst[0]["reached"])}
        del wp1

    # ---- e2e through the public API with HOST buffers (pinned), copies inside the timed region
    e2e = None
    if not args.no_e2e:
        hsrc = {k: srcs[k].to(torch.int64).cpu() for k in kinds}
        hout = {k: torch.empty((B, g.row_shape(fmt[k])[0]), dtype=g.row_shape(fmt[k])[1], pin_memory=True)
                for k in kinds}
        # one step = every kind's query_host call (asynchronous: kind k's rows drain to the host
        # while kind k + 1 computes), then the step's results are read: a stream synchronisation
        def e2e_step():
            for k in kinds:
                g.query_host(k, hsrc[k], mode="2phase", out=hout[k], fmt=fmt[k], sync=False)
            g.status()  # cg_graph_status: the stream and the graph's copy stream drained, errors returned
        e2e_step()
        ctx.barrier()
        t0 = time.perf_counter()
        steps_e2e = max(1, min(args.steps, 5))
        for _ in range(steps_e2e):
            e2e_step()
        ctx.barrier()
        el = ctx.max_ms(time.perf_counter() - t0)
        d2h = sum(hout[k].numel() * hout[k].element_size() for k in kinds)
        e2e = {"value": ws * q_step * steps_e2e / el, "unit": "queries/s", "h2d_bytes_per_step": 4 * q_step,
               "d2h_bytes_per_step": d2h, "api": "cg_query_host_async per kind + one cg_graph_status per step (pinned host buffers, out rows as `config.out_rows`)",
               "steps": steps_e2e}
        del hout

    # ---- CPU baseline: the oracle on the host cores, bounded sample (rank 0, N=1 only)
    cpu = None
    if rank == 0 and ws == 1 and not args.no_cpu_baseline:
        cores = os.cpu_count() or 1
        per_kind_n = args.cpu_sample or max(1, min(cores, 16) // 2)
        v, cores, sample, _ = cpu_oracle_run(cfg, src_h, dst_h, w_h, kinds, per_kind_n)
        cpu = {"value": v, "unit": "queries/s", "cores": cores, "kind": "oracle", "sample": sample,
               "cpu_model": cpu_model()}
    del src_h, dst_h, w_h
    g_m = g.m
    g.close()
    del outs
    torch.cuda.empty_cache()

    # ---- configs[0] (one GPU) and configs[2] (strong scaling over the N ranks)
    c1 = None
    if not args.no_c1 and ws == 1:
        c1 = run_c1_single(ctx)
    c3 = None
    if not args.no_c3 and args.config == "c2":
        c3 = run_c3_strong(ctx, args.c3_steps or min(args.steps, 5), 3)

    if rank == 0:
        line = {
            "metric": METRIC, "value": qps2, "unit": "queries/s", "n_gpus": ws, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms2 / args.steps, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None,
            "dtype": "integer / binary32 arithmetic: " + LANES + "; out rows " + (
                "narrow (u16 SSSP/SSWP/SSNP/BFS, bits REACH, u32 Viterbi; exact)" if args.out == "narrow" else "u32"),
            "data": "synthetic",
            "config": workload_config(cfg, g_m, kinds, B, args.K, ws, gather,
                                      ("inputs larger than L2 (packed CSR + value rows %.0f MB > 126 MB L2)"
                                       % (resident_bytes / 1e6) if flush is None else
                                       "L2 flushed between timed steps (256 MB write outside the step events; "
                                       "inputs %.0f MB)" % (resident_bytes / 1e6)), args.out),
            "gteps": gteps2, "full": {"value": qpsf, "unit": "queries/s", "gteps": gtepsf, "ms_per_step": msf / args.steps},
            "speedup_2phase_vs_full": qpsf and qps2 / qpsf, "u32_out": u32,
            "per_kind": per_kind, "wcc": wcc, "roofline": roofline, "cpu_baseline": cpu, "e2e": e2e,
            "c1_single": c1, "c3_strong": c3,
            "gpu_launches": launches, "clocks": clocks,
            "build_ms": {k: build[k]["build_ms"] for k in build}, "graph_build_s": graph_s,
        }
        print(json.dumps(line), flush=True)
    if ws > 1:
        import torch.distributed as dist
        dist.barrier()
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
