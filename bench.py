#!/usr/bin/env python
"""Benchmark: 8x8 Reversi playouts/s on B200 (BASELINE.json metric, configs[1]).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl reference]

One "step" = one pass of the playout hot path over one
batch of BASELINE configs[1]: 4096 synthetic mid-game positions x 256 random
playouts, inputs resident in HBM, launched through mcts_playouts_async. N>1:
one process per GPU (torchrun), every rank runs its own batch with distinct
playout streams (leaf_id_base = rank * 4096): weak scaling, no collective on
the data path. The block-parallel search (configs[2] shape, a1-a11 incl. the
NCCL root-stats allreduce at N>1), the leaf-parallel comparison (configs[3])
and the NEXT-4 shared tree (1184 workers x 128 threads on one tree) are reported
in the "search" / "leaf_search" / "tree_search" objects of the same line
(device-timed from a spin kernel's end, so host-side enqueue time stays out),
the paper's CPU-managed trees in "hosted_search". "e2e" is the same batch
through mcts_playouts with pinned host buffers, one synchronous call per step;
"e2e.pipelined" the same steps through mcts_playouts_host_async, enqueued
back to back with one synchronisation.

Prints ONE JSON line on rank 0. See DESIGN.md §8 for every field.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
STATS_LEN = 202  # include/mcts.h MCTS_STATS_LEN
sys.path.insert(0, ROOT)

N_LEAVES, N_PER_LEAF, GEN_SEED, LMIN, LMAX = 4096, 256, 2, 20, 40
OPEN_LMIN, OPEN_LMAX = 0, 8  # the opening-phase batch
PLAYOUT_SEED = 2
SEARCH_GATE_CYCLES = 500_000_000  # ~250 ms at the 1965 MHz SM clock (torch.cuda._sleep)
SEARCH_TREES, SEARCH_THREADS, SEARCH_MS = 1184, 128, 500.0
LEAF_THREADS = 16384
# (n_trees, threads_per_tree) of each scheme's searcher; for "tree" n_trees is
# the number of worker CTAs sharing one tree (NEXT-4)
SCHEME_SHAPE = {"block": (SEARCH_TREES, SEARCH_THREADS), "leaf": (1, LEAF_THREADS),
                "tree": (SEARCH_TREES, SEARCH_THREADS)}
SCHEME_DESC = {"block": "configs[2] block-parallel", "leaf": "configs[3] leaf-parallel",
               "tree": "NEXT-4 tree-parallel (one shared tree)"}
METRIC = "8x8 Reversi playouts/sec at 1/2/4/8 B200; win% vs CPU-oracle MCTS"
# SURVEY.md §8(d)'s a-priori estimate of 32-bit integer operations per ply of a
# shift-mask implementation (movegen 2x8x24, flip 8x26, pick 30, Philox 96/4,
# loop 8). The shipped loop needs far fewer, so the roofline's numerator is the
# per-ply instruction count measured by ncu on the shipped kernel;
# this figure is reported next to it as `survey_model` and is the fallback when
# no capture is committed.
ALG_OPS_PER_PLY = 440


def kernel_source_hash() -> str:
    """sha256 (16 hex) of the sources and flags the playout kernel is built from;
    stored with each committed ncu capture so a stale capture is detected."""
    import hashlib
    from paper_conf_ipps_rockis11_b200 import _build
    h = hashlib.sha256()
    for name in ("reversi_device.cuh", "playouts.cuh"):
        h.update(open(os.path.join(_build.CSRC, name), "rb").read())
    h.update(" ".join(_build.NVCC_FLAGS).encode())
    return h.hexdigest()[:16]


def ops_per_ply(kernel="playouts", plies_per_launch=None):
    """(thread-instructions per ply, basis) for the executed-instruction
    roofline: ncu smsp__thread_inst_executed (= inst_executed x lanes active) of
    the committed --set full capture of this kernel (profiles/latest_ncu.json),
    divided by the plies of one launch of the same workload. If the capture was
    taken from other kernel sources (source hash mismatch) or is missing, the
    SURVEY.md 8(d) model is used and the basis says so (with a warning)."""
    try:
        prof = json.load(open(os.path.join(ROOT, "profiles", "latest_ncu.json")))[kernel]
        if prof.get("source_hash") != kernel_source_hash():
            print(f"[bench] warning: profiles/latest_ncu.json {kernel} capture is stale "
                  f"(source hash {prof.get('source_hash')} != {kernel_source_hash()}); "
                  "using the SURVEY 8(d) model", file=sys.stderr)
            return ALG_OPS_PER_PLY, "model: SURVEY.md 8(d) estimate (committed capture is stale)"
        plies = plies_per_launch or prof["plies_per_launch"]
        return prof["thread_inst"] / plies, ("measured: ncu smsp__thread_inst_executed.sum / plies, "
                                             f"committed capture of {kernel}_kernel (profiles/latest_ncu.json, "
                                             f"source hash {prof['source_hash']})")
    except Exception:
        return ALG_OPS_PER_PLY, "model: SURVEY.md 8(d) estimate (no committed capture)"


def headline(playouts_total, plies_total, t_ms_max, steps):
    """The line's throughput numbers from whole-job counts and the max-over-ranks
    device time of the `steps` timed steps."""
    s = t_ms_max / 1e3
    return {"value": playouts_total / s, "plies_per_s": plies_total / s, "ms_per_step": t_ms_max / steps}


def roofline(plies_per_launch, kern_s, peak_ops, ops_exec, ops_basis, alu_peak, peak_basis):
    """The integer roofline of the playout kernel, both ways:
    frac = SURVEY.md 8(d)'s algorithmic ops per ply (ALG_OPS_PER_PLY) x plies per
    launch / launch time / peak (the contract's ALGORITHMIC numerator; > 1 means
    the kernel needs fewer instructions than the model); frac_executed = the
    executed thread-instructions per ply (ncu) x plies / time / peak, i.e. the
    share of the chip's integer issue rate the kernel keeps busy."""
    alg = plies_per_launch * ALG_OPS_PER_PLY / kern_s
    exe = plies_per_launch * ops_exec / kern_s
    return {"bound": "alu", "achieved": alg / 1e9, "peak": peak_ops / 1e9, "unit": "Gop/s",
            "frac": alg / peak_ops, "frac_basis": f"algorithmic: SURVEY.md 8(d) {ALG_OPS_PER_PLY} int ops per ply",
            "achieved_executed": exe / 1e9, "frac_executed": exe / peak_ops, "ops_per_ply_executed": ops_exec,
            "ops_basis": ops_basis, "plies_per_launch": plies_per_launch, "peak_basis": peak_basis,
            "alu_pipe_peak": alu_peak / 1e9}


def clocks_sampler(path):
    try:
        f = open(path, "w")
        p = subprocess.Popen(
            ["nvidia-smi", "--query-gpu=index,clocks.sm,clocks.max.sm,power.draw,"
             "clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
             "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
             "clocks_event_reasons.sw_power_cap", "--format=csv,noheader,nounits", "-lms", "100"],
            stdout=f, stderr=subprocess.DEVNULL)
        return p, f
    except Exception:
        return None, None


def clocks_summary(path, gpu_index):
    rows = []
    try:
        for line in open(path):
            parts = [x.strip() for x in line.split(",")]
            if len(parts) >= 9 and parts[0] == str(gpu_index):
                rows.append(parts)
    except Exception:
        pass
    if not rows:
        return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unavailable"], "samples": 0}
    sm = sorted(float(r[1]) for r in rows)
    names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
    reasons = sorted({n for r in rows for n, v in zip(names, r[5:9]) if v.lower() == "active"})
    return {"sm_mhz": sm[len(sm) // 2], "sm_max_mhz": float(rows[0][2]), "reasons": reasons,
            "samples": len(rows)}


def integer_peak():
    """Integer roofline denominator: the measured B200 rate of an
    alternating LOP3/IMAD stream (both integer pipes, i.e. the issue limit) from
    tools/int_peaks.cu (profiles/int_peaks.json), else the issue-slot count
    148 SM x 4 SMSP x 32 lanes x sm_max_mhz. Also returns the ALU-pipe-only rate."""
    try:
        ip = json.load(open(os.path.join(ROOT, "profiles", "int_peaks.json")))
        return (ip["lop3_imad_mixed"], "measured: alternating LOP3/IMAD stream, all SMs "
                "(tools/int_peaks.cu -> profiles/int_peaks.json)", ip["lop3_alu"])
    except Exception:
        sm_max = measured_peaks().get("sm_max_mhz", 1965.0)
        return (148 * 4 * 32 * sm_max * 1e6, f"derived: 148 SM x 4 SMSP x 32 lanes x {sm_max:.0f} MHz",
                148 * 4 * 16 * sm_max * 1e6)


def measured_peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return {}


def reference_arm(args, rank):
    """--impl reference: the CPU oracle as it stands, on this box's host cores."""
    if rank != 0:
        return
    import oracle
    cores = len(os.sched_getaffinity(0))
    leaves = oracle.gen_positions(GEN_SEED, N_LEAVES, LMIN, LMAX)
    chunk = 64  # leaves per step: a bounded sample of the configs[1] batch

    def step(i):
        a = (i * chunk) % N_LEAVES
        return oracle.playouts(leaves[a:a + chunk], N_PER_LEAF, PLAYOUT_SEED, leaf_id_base=a,
                               nthreads=cores)

    for i in range(args.warmup):
        step(i)
    t0 = time.perf_counter()
    for i in range(args.steps):
        step(args.warmup + i)
    dt = time.perf_counter() - t0
    value = args.steps * chunk * N_PER_LEAF / dt
    sample = f"{chunk} leaves x {N_PER_LEAF} playouts of configs[1] per step"
    print(json.dumps({
        "impl": "reference", "metric": METRIC, "value": value, "unit": "playouts/s",
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": dt * 1e3 / args.steps, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "u64", "data": "synthetic",
        "config": {"workload": "configs[1]: 4096 mid-game positions x 256 playouts (sampled)",
                   "sample": sample},
        "cpu_baseline": {"value": value, "unit": "playouts/s", "cores": cores, "kind": "oracle",
                         "sample": sample},
        "e2e": {"value": value, "unit": "playouts/s", "h2d_bytes_per_step": 0,
                "d2h_bytes_per_step": 0},
    }), flush=True)


def cpu_baseline(budget_s=12.0, single_budget_s=4.0):
    """The oracle timed on the host cores on a bounded sample of configs[1]:
    all cores (the reported value) and one core (`single_core`)."""
    import oracle
    cores = len(os.sched_getaffinity(0))
    leaves = oracle.gen_positions(GEN_SEED, N_LEAVES, LMIN, LMAX)
    done, t0 = 0, time.perf_counter()
    while done < N_LEAVES and time.perf_counter() - t0 < budget_s:
        oracle.playouts(leaves[done:done + 128], N_PER_LEAF, PLAYOUT_SEED, leaf_id_base=done,
                        nthreads=cores)
        done += 128
    dt = time.perf_counter() - t0
    one, t1 = 0, time.perf_counter()
    while one < N_LEAVES and time.perf_counter() - t1 < single_budget_s:
        oracle.playouts(leaves[one:one + 2], N_PER_LEAF, PLAYOUT_SEED, leaf_id_base=one, nthreads=1)
        one += 2
    d1 = time.perf_counter() - t1
    return {"value": done * N_PER_LEAF / dt, "unit": "playouts/s", "cores": cores, "kind": "oracle",
            "sample": f"leaves 0..{done - 1} of configs[1] x {N_PER_LEAF} playouts ({dt:.1f} s)",
            "single_core": {"value": one * N_PER_LEAF / d1, "cores": 1,
                            "sample": f"leaves 0..{one - 1} of configs[1] x {N_PER_LEAF} playouts ({d1:.1f} s)"}}


def sweep_leg(args, local):
    """Fig. 5 analog (NEXT-2): search playouts/s vs total GPU
    threads for leaf parallelism, block parallelism with 32- and 128-thread
    blocks and the NEXT-4 shared tree with 128-thread workers ("trees" =
    workers, "iterations_per_tree" = per worker), time mode from the opening.
    One JSON line, rank 0 only."""
    import torch
    import paper_conf_ipps_rockis11_b200 as pkg
    torch.cuda.set_device(local)
    stream = torch.cuda.current_stream()
    root = pkg.position(*pkg.OPENING)
    st = torch.zeros(STATS_LEN, dtype=torch.int64, device="cuda")
    handles = {"block": pkg.Mcts(scheme="block", device=local), "leaf": pkg.Mcts(scheme="leaf", device=local),
               "tree": pkg.Mcts(scheme="tree", device=local)}
    points = []
    for total in [128, 512, 2048, 8192, 16384, 37888, 75776, 151552]:
        for scheme, bs in [("leaf", 128), ("block", 32), ("block", 128), ("tree", 128)]:
            if scheme == "leaf" and total > 65536:
                continue
            n_trees, threads = (1, total) if scheme == "leaf" else (total // bs, bs)
            h = handles[scheme]
            try:
                h.search_async(root, 0, 10.0, n_trees, threads, 7, 0, st.data_ptr(), stream)  # warm-up
            except pkg.MctsError as e:  # time mode needs every tree co-resident (trees beyond would idle)
                points.append({"scheme": scheme, "block": bs, "gpu_threads": total, "trees": n_trees,
                               "skipped": str(e)})
                continue
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            h.search_async(root, 0, args.sweep_ms, n_trees, threads, 7, 0, st.data_ptr(), stream)
            e1.record(stream)
            torch.cuda.synchronize()
            ms = e0.elapsed_time(e1)
            s = st.cpu().numpy()
            points.append({"scheme": scheme, "block": bs, "gpu_threads": total, "trees": n_trees,
                           "playouts_per_s": float(s[195]) / (ms / 1e3),
                           "iterations_per_tree": float(s[196]) / n_trees, "ms": ms,
                           "plies_per_s": float(s[197]) / (ms / 1e3)})
            if args.sweep_games and total in (512, 2048, 16384, 151552):
                def gpu_move(black, white, to_move, seed, h=h, n_trees=n_trees, threads=threads):
                    h.search_async(pkg.position(black, white, to_move), 0, args.move_ms, n_trees, threads,
                                   seed, 0, st.data_ptr(), stream)
                    torch.cuda.synchronize()
                    x = st.cpu().numpy()
                    return pkg.best_move(x), int(x[195])
                r = play_match(gpu_move, 1, args.sweep_games, args.move_ms, tag=f"{scheme}{bs}/{total}")
                points[-1]["vs_1core"] = {k: r[k] for k in ("win_pct", "ci95_wilson", "results",
                                                            "mean_disc_diff", "gpu_playouts_per_move",
                                                            "cpu_playouts_per_move")}
            log(points[-1])
    print(json.dumps({"metric": "search playouts/s vs GPU threads (Fig. 5 analog); win% vs 1 CPU core "
                                "(Fig. 6 analog, points with vs_1core)", "unit": "playouts/s",
                      "config": {"root": "opening", "time_ms": args.sweep_ms, "C": 1.0,
                                 "games_per_point": args.sweep_games, "move_ms": args.move_ms},
                      "points": points}), flush=True)


def play_match(gpu_move, cpu_threads, games, move_ms, seed_base=1000, tag="", opp_move=None, cpu_c=1.0):
    """Games of the B200 searcher (gpu_move(black, white, to_move, seed) ->
    (move, playouts)) against the oracle's root-parallel CPU MCTS on
    `cpu_threads` host threads, alternating colours, equal time per move; the
    oracle's rules referee. Returns W/D/L, disc differences and the per-game-step
    disc difference (GPU minus CPU, the paper's "point difference")."""
    import numpy as np
    import oracle
    res = {"W": 0, "D": 0, "L": 0}
    diffs, gpu_po, cpu_po, steps = [], [], [], []
    depth = {"gpu": {}, "opp": {}}  # game step -> mean tree depths (searchers that report one)
    pool = {"refused": 0, "max_fill": 0.0}  # node-pool saturation of the GPU searcher over all moves
    t_start = time.time()
    for g in range(games):
        gpu_color = g % 2
        black, white, to_move = oracle.OPENING_BLACK, oracle.OPENING_WHITE, 0
        ply, curve = 0, []
        while True:
            own, opp = (black, white) if to_move == 0 else (white, black)
            legal = oracle.legal(own, opp)
            if legal == 0:
                if oracle.legal(opp, own) == 0:
                    break
                to_move ^= 1
                continue
            seed = seed_base + 1000 * g + ply
            if to_move == gpu_color:
                mv, po, *dp = gpu_move(black, white, to_move, seed)
                gpu_po.append(po)
                if dp:
                    depth["gpu"].setdefault(ply, []).append(dp[0])
                if len(dp) > 1:  # (refused expansions, slots used, slot capacity) of this move's search
                    pool["refused"] += dp[1][0]
                    pool["max_fill"] = max(pool["max_fill"], dp[1][1] / max(dp[1][2], 1))
            elif opp_move is not None:  # another device searcher (--h2h)
                mv, po, *dp = opp_move(black, white, to_move, seed + 500)
                cpu_po.append(po)
                if dp:
                    depth["opp"].setdefault(ply, []).append(dp[0])
            else:
                st, mv = oracle.mcts_timed(oracle.position(black, white, to_move), cpu_threads, move_ms, seed,
                                           C=cpu_c)
                cpu_po.append(int(st[195]))
            assert 0 <= mv < 64 and (legal >> mv) & 1, (mv, hex(legal))
            f = oracle.flips(own, opp, mv)
            own, opp = own | f | (1 << mv), opp & ~f
            black, white = (own, opp) if to_move == 0 else (opp, own)
            to_move ^= 1
            ply += 1
            nb, nw = bin(black).count("1"), bin(white).count("1")
            curve.append((nb - nw) if gpu_color == 0 else (nw - nb))
        d = curve[-1] if curve else 0
        diffs.append(d)
        steps.append(curve)
        res["W" if d > 0 else "D" if d == 0 else "L"] += 1
        log(f"{tag} game {g}: gpu={'black' if gpu_color == 0 else 'white'} diff {d:+d} {res}")
    n = max(games, 1)
    p = (res["W"] + 0.5 * res["D"]) / n
    z = 1.96  # Wilson score interval
    centre = (p + z * z / (2 * n)) / (1 + z * z / n)
    half = z * float(np.sqrt(p * (1 - p) / n + z * z / (4 * n * n))) / (1 + z * z / n)
    L = max((len(c) for c in steps), default=0)
    per_step = [float(np.mean([c[i] if i < len(c) else c[-1] for c in steps])) for i in range(L)]
    return {"win_pct": 100 * p, "ci95_wilson": [100 * (centre - half), 100 * (centre + half)],
            "results": res, "games": games, "mean_disc_diff": float(np.mean(diffs)) if diffs else None,
            "point_diff_per_step": per_step,
            "gpu_playouts_per_move": float(np.mean(gpu_po)) if gpu_po else None,
            "cpu_playouts_per_move": float(np.mean(cpu_po)) if cpu_po else None,
            # mean depth of the simulated node per game step (the paper's Fig. 8 "Depth")
            "gpu_depth_per_step": {int(k): float(np.mean(v)) for k, v in sorted(depth["gpu"].items())},
            "opp_depth_per_step": {int(k): float(np.mean(v)) for k, v in sorted(depth["opp"].items())},
            "gpu_refused_expansions": pool["refused"], "gpu_pool_max_fill": pool["max_fill"],
            "wall_s": time.time() - t_start}


def h2h_leg(args, local):
    """Head-to-head of two device searchers on the same GPU at equal wall time
    per move, alternating colours (--h2h-schemes A,B; "gpu" in the result = A).
    Default block,leaf = SURVEY.md 8(d) c3: the block-parallel searcher
    (configs[2], 1184 trees x 128 threads) against the paper's leaf-parallel
    scheme (1 tree x 16384 threads per leaf batch); tree,block pits the NEXT-4
    shared tree (1184 workers x 128 threads) against configs[2]."""
    import torch
    import paper_conf_ipps_rockis11_b200 as pkg
    torch.cuda.set_device(local)
    stream = torch.cuda.current_stream()
    st = torch.zeros(STATS_LEN, dtype=torch.int64, device="cuda")
    a, b = args.h2h_schemes.split(",")
    base = {"hosted": "block", "hosted-hybrid": "block"}
    ha = pkg.Mcts(c_uct=args.c_uct, scheme=base.get(a, a), device=local)
    hb = pkg.Mcts(c_uct=args.c_uct, scheme=base.get(b, b), device=local)
    cores = len(os.sched_getaffinity(0))

    def mover(h, n_trees, threads, name):
        def move(black, white, to_move, seed):
            if name in base:  # NEXT-1: CPU-managed trees (+ CPU iterations on them for hosted-hybrid)
                r = h.search_hosted(pkg.position(black, white, to_move), time_ms=args.move_ms, n_trees=n_trees,
                                    threads_per_tree=threads, seed=seed,
                                    cpu_iters=1 if name == "hosted-hybrid" else 0, cpu_threads=cores)
                return (r["best_move"], r["root_visits"], r["depth_sum"] / max(r["iterations"], 1))
            h.search_async(pkg.position(black, white, to_move), 0, args.move_ms, n_trees, threads, seed, 0,
                           st.data_ptr(), stream)
            torch.cuda.synchronize()
            x = st.cpu().numpy()
            return (pkg.best_move(x), int(x[195]), float(x[198]) / max(int(x[196]), 1),
                    (int(x[199]), int(x[200]), int(x[201])))
        return move

    r = play_match(mover(ha, *SCHEME_SHAPE[base.get(a, a)], a), 0, args.selfplay, args.move_ms, tag="h2h",
                   opp_move=mover(hb, *SCHEME_SHAPE[base.get(b, b)], b))
    r[f"{a}_playouts_per_move"] = r.pop("gpu_playouts_per_move")
    r[f"{b}_playouts_per_move"] = r.pop("cpu_playouts_per_move")
    r[f"{a}_depth_per_step"] = r.pop("gpu_depth_per_step")
    r[f"{b}_depth_per_step"] = r.pop("opp_depth_per_step")
    names = {"block": "block parallelism", "leaf": "leaf parallelism", "tree": "tree parallelism",
             "hosted": "CPU-managed block parallelism", "hosted-hybrid": "CPU-managed block parallelism + CPU iterations"}
    shape = {k: f"{SCHEME_DESC[k]}: {v[0]} {'workers' if k == 'tree' else 'trees'} x {v[1]} threads"
             for k, v in SCHEME_SHAPE.items()}
    for k in base:
        shape[k] = f"NEXT-1 {k} (DESIGN.md §14): {SEARCH_TREES} trees x {SEARCH_THREADS} GPU threads, {cores} host threads"
    print(json.dumps({"metric": f"win% of {names[a]} vs {names[b]} (equal wall time per move)",
                      "value": r["win_pct"], "unit": "%", "n_gpus": 1,
                      "config": {a: shape[a], b: shape[b], "move_ms": args.move_ms, "colours": "alternating",
                                 "C": args.c_uct}, **r}),
          flush=True)


def selfplay_leg(args, world, rank, local):
    """Win% of the B200 searcher vs the multi-threaded CPU oracle MCTS at equal
    wall time per move (BASELINE.json metric, configs[2]-[4]). Rank 0 referees
    with the oracle's rules and plays the CPU side on all host cores; every rank
    searches its own trees (tree_id_base = rank * n_trees) and the root stats
    are merged by one allreduce per move, so all ranks agree on the move.
    --fig7 instead sweeps the CPU side over 1, 2, 4, ... host threads and reports
    the point difference per game step (Fig. 7 analog)."""
    import torch
    import torch.distributed as dist
    import paper_conf_ipps_rockis11_b200 as pkg
    from paper_conf_ipps_rockis11_b200.distributed import merge_root_stats

    torch.cuda.set_device(local)
    if world > 1:
        init_dist(dist, torch, local)
    hybrid = args.sp_scheme in ("hybrid", "hybrid-tree")
    hosted = args.sp_scheme in ("hosted", "hosted-hybrid")
    if (hybrid or hosted) and world > 1:
        raise SystemExit("--sp-scheme hybrid / hosted is single-GPU")
    scheme = {"leaf": "leaf", "tree": "tree", "hybrid-tree": "tree"}.get(args.sp_scheme, "block")
    n_trees, threads = SCHEME_SHAPE[scheme]
    m = pkg.Mcts(c_uct=args.c_uct, scheme=scheme, device=local)
    stream = torch.cuda.current_stream()
    stats = torch.zeros(STATS_LEN, dtype=torch.int64, device="cuda")
    msg = torch.zeros(4, dtype=torch.int64, device="cuda")  # black, white, to_move, seed/-1

    def search(black, white, to_move, seed):
        pos = pkg.position(black, white, to_move)
        if hosted:  # NEXT-1: CPU-managed trees, GPU playouts per step (+ CPU iterations meanwhile)
            r = m.search_hosted(pos, time_ms=args.move_ms, n_trees=n_trees, threads_per_tree=threads, seed=seed,
                                cpu_iters=1 if args.sp_scheme == "hosted-hybrid" else 0,
                                cpu_threads=len(os.sched_getaffinity(0)))
            return r["best_move"], r["root_visits"], r["depth_sum"] / max(r["iterations"], 1)  # host pools: unbounded
        if hybrid:  # NEXT-1: GPU trees + one host tree per host core, root sums merged
            r = m.search_hybrid(pos, time_ms=args.move_ms, n_trees=n_trees, threads_per_tree=threads,
                                seed=seed, cpu_threads=len(os.sched_getaffinity(0)))
            return (r["best_move"], r["root_visits"], r["depth_sum"] / max(r["iterations"], 1),
                    (r["refused_expansions"], r["slots_used"], r["slot_capacity"]))
        m.search_async(pos, 0, args.move_ms, n_trees, threads, seed, rank * n_trees,
                       stats.data_ptr(), stream)
        with torch.cuda.stream(stream):
            merge_root_stats(stats)
        torch.cuda.synchronize()
        st = stats.cpu().numpy()
        return (pkg.best_move(st), int(st[195]), float(st[198]) / max(int(st[196]), 1),
                (int(st[199]), int(st[200]), int(st[201])))

    if rank != 0:  # follower ranks: search whatever position rank 0 broadcasts
        while True:
            dist.broadcast(msg, 0)
            b, w, t, seed = (int(x) for x in msg.cpu().numpy())
            if seed < 0:
                break
            search(b & ((1 << 64) - 1), w & ((1 << 64) - 1), t, seed)
        dist.destroy_process_group()
        return

    def to_i64(x):
        return x - (1 << 64) if x >= (1 << 63) else x

    def gpu_move(black, white, to_move, seed):
        if world > 1:
            msg.copy_(torch.tensor([to_i64(black), to_i64(white), to_move, seed]))
            dist.broadcast(msg, 0)
        return search(black, white, to_move, seed)

    cores = len(os.sched_getaffinity(0))
    cpu_c = args.c_uct if args.cpu_c is None else args.cpu_c
    workload = (f"{SCHEME_DESC[scheme]} searcher ({n_trees} {'workers' if scheme == 'tree' else 'trees'} x "
                f"{threads} threads per GPU, {args.sp_scheme}, {world} GPU(s))")
    if args.fig7:
        curves = []
        t = 1
        while t <= cores:
            r = play_match(gpu_move, t, args.selfplay, args.move_ms, tag=f"cpu{t}", cpu_c=cpu_c)
            curves.append({"cpu_threads": t, **r})
            t *= 2
        out = {"metric": "point difference per game step vs root-parallel CPU MCTS on 1..N host threads "
                         "(Fig. 7 analog)", "unit": "discs", "n_gpus": world,
               "config": {"workload": workload, "move_ms": args.move_ms, "games_per_point": args.selfplay,
                          "C": args.c_uct, "C_cpu": cpu_c}, "curves": curves}
    else:
        r = play_match(gpu_move, cores, args.selfplay, args.move_ms, seed_base=args.sp_seed_base, cpu_c=cpu_c)
        out = {"metric": "win% vs CPU-oracle MCTS (equal wall time per move)", "value": r["win_pct"],
               "unit": "%", "n_gpus": world,
               "config": {"workload": workload + f" vs root-parallel CPU oracle MCTS on {cores} host threads",
                          "move_ms": args.move_ms, "colours": "alternating", "C": args.c_uct, "C_cpu": cpu_c,
                          "seed_base": args.sp_seed_base}, **r}
    if world > 1:
        msg.copy_(torch.tensor([0, 0, 0, -1]))
        dist.broadcast(msg, 0)
    print(json.dumps(out), flush=True)
    if world > 1:
        dist.destroy_process_group()


def self_launch_cmd(gpus, argv, env):
    """`python bench.py --gpus N` outside torchrun: the torchrun command that runs
    this script as N ranks (one per GPU, rendezvous on 127.0.0.1), or None when
    already under torchrun or N == 1. Under torchrun WORLD_SIZE must equal N."""
    if "WORLD_SIZE" in env:
        if int(env["WORLD_SIZE"]) != gpus:
            raise SystemExit(f"bench.py: --gpus {gpus} but WORLD_SIZE={env['WORLD_SIZE']}")
        return None
    if gpus <= 1:
        return None
    import socket
    with socket.socket() as sk:  # a free rendezvous port
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    return [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={gpus}",
            "--master-addr", "127.0.0.1", f"--master-port={port}", os.path.abspath(__file__), *argv]


def init_dist(dist, torch, local):
    """One process per GPU over NCCL (BENCH_BACKEND=gloo is a single-GPU test hook).
    Logs the communicator (backend, rank, world size, device) on stderr."""
    backend = os.environ.get("BENCH_BACKEND", "nccl")
    if backend == "nccl":
        dist.init_process_group("nccl", device_id=torch.device(f"cuda:{local}"))
    else:
        dist.init_process_group(backend)
    print(f"[bench] process group: backend={dist.get_backend()} rank={dist.get_rank()} "
          f"world={dist.get_world_size()} device=cuda:{local}", file=sys.stderr, flush=True)


def hosted_leg(m, ms):
    """The paper's block parallelism as it built it: CPU-managed trees, one GPU
    playout kernel per step, without and with the hybrid CPU
    iterations on the same trees while the kernel runs (Fig. 4);
    configs[2] shape from the opening, time mode. Reports playouts/s, the
    sequential host share of a step and the CPU's share of the
    iterations, nodes and root visits."""
    cores = len(os.sched_getaffinity(0))
    out = {"workload": f"NEXT-1 CPU-managed trees: {SEARCH_TREES} trees x {SEARCH_THREADS} GPU threads, "
                       f"{ms:.0f} ms, opening root, C=1.0, {cores} host threads"}
    for name, cpu_iters in (("gpu_only", 0), ("hybrid", 1)):
        kw = dict(time_ms=ms, n_trees=SEARCH_TREES, threads_per_tree=SEARCH_THREADS, seed=1000,
                  cpu_iters=cpu_iters, cpu_threads=cores)
        m.search_hosted(pkg_opening(), **kw)  # warm-up (pinned buffers, ln table)
        t0 = time.perf_counter()
        r = m.search_hosted(pkg_opening(), **kw)
        dt = time.perf_counter() - t0
        st, inf = r["stats"], r["info"]
        step_ms = inf["select_ms"] + inf["gpu_ms"] + inf["backprop_ms"]
        out[name] = {"playouts_per_s": float(st[195]) / dt, "ms": dt * 1e3, "steps": inf["steps"],
                     "mean_depth": float(st[198]) / max(float(st[196]), 1.0),
                     "host_select_share": inf["select_ms"] / max(step_ms, 1e-9),
                     "host_backprop_share": inf["backprop_ms"] / max(step_ms, 1e-9),
                     "cpu_iteration_share": inf["cpu_iterations"] / max(float(st[196]), 1.0),
                     "cpu_node_share": inf["cpu_nodes"] / max(inf["cpu_nodes"] + inf["gpu_nodes"], 1),
                     "cpu_root_visit_share": inf["cpu_iterations"] / max(float(st[195]), 1.0),
                     "cpu_mean_depth": inf["cpu_depth_sum"] / max(inf["cpu_iterations"], 1),
                     "best_move": int(r["best_move"])}
    return out


def pkg_opening():
    import paper_conf_ipps_rockis11_b200 as pkg
    return pkg.opening()


def pool_info(st) -> dict:
    """Node-pool saturation of a search (stats [199]-[201], include/mcts.h)."""
    return {"refused_expansions": int(st[199]), "pool_slots_used": int(st[200]),
            "pool_slot_capacity": int(st[201])}


def log(*a):
    if os.environ.get("BENCH_DEBUG"):
        print("[bench]", *a, file=sys.stderr, flush=True)


def main():
    if os.environ.get("BENCH_DEBUG"):
        import faulthandler
        faulthandler.dump_traceback_later(90, repeat=True)
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="b200", choices=["b200", "reference"])
    ap.add_argument("--no-search", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--search-ms", type=float, default=SEARCH_MS)
    ap.add_argument("--selfplay", type=int, default=0,
                    help="play N games vs the CPU oracle MCTS and print the win%% line instead")
    ap.add_argument("--move-ms", type=float, default=SEARCH_MS, help="self-play time per move")
    ap.add_argument("--sp-scheme", default="block",
                    choices=["block", "leaf", "hybrid", "tree", "hybrid-tree", "hosted", "hosted-hybrid"])
    ap.add_argument("--c-uct", type=float, default=0.25,
                    help="UCB constant C of the GPU searcher (0.25: best of {0.25, 0.5, 1, 2} "
                         "in 10-game self-play at 100 ms per move, profiles/r01_selfplay_c*.json)")
    ap.add_argument("--sp-seed-base", type=int, default=1000,
                    help="self-play seed base (game g, ply p uses seed_base + 1000 g + p): a new base gives "
                         "an independent game set to pool with earlier ones")
    ap.add_argument("--cpu-c", type=float, default=None,
                    help="UCB constant of the CPU oracle opponent (default: the same as --c-uct)")
    ap.add_argument("--h2h", action="store_true",
                    help="with --selfplay: head-to-head of two device searchers on one GPU (--h2h-schemes)")
    ap.add_argument("--h2h-schemes", default="block,leaf",
                    help="A,B of block|leaf|tree|hosted|hosted-hybrid (default block,leaf = configs[2] vs configs[3])")
    ap.add_argument("--fig7", action="store_true", help="with --selfplay: CPU side on 1, 2, 4, ... threads")
    ap.add_argument("--sweep", action="store_true", help="Fig. 5 analog: playouts/s vs GPU threads")
    ap.add_argument("--sweep-games", type=int, default=0,
                    help="with --sweep: also play N games per point vs 1-core CPU MCTS (Fig. 6 analog)")
    ap.add_argument("--sweep-ms", type=float, default=200.0)
    ap.add_argument("--search-iters", type=int, default=0,
                    help="iteration-mode search legs (profiling); default: time mode")
    args = ap.parse_args()

    cmd = self_launch_cmd(args.gpus, sys.argv[1:], os.environ)
    if cmd is not None:  # --gpus N without torchrun: one process per GPU, launched here
        sys.exit(subprocess.call(cmd))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if os.environ.get("BENCH_SAME_DEVICE"):  # test hook: all ranks on GPU 0 (with BENCH_BACKEND=gloo)
        local = 0
    if args.impl == "reference":
        return reference_arm(args, rank)
    if args.selfplay and args.h2h:
        return h2h_leg(args, local) if rank == 0 else None
    if args.selfplay:
        return selfplay_leg(args, world, rank, local)
    if args.sweep:
        return sweep_leg(args, local) if rank == 0 else None
    if args.warmup < 3:
        args.warmup = 3

    import torch
    import torch.distributed as dist
    import paper_conf_ipps_rockis11_b200 as pkg
    from paper_conf_ipps_rockis11_b200 import device as dev
    from paper_conf_ipps_rockis11_b200.distributed import merge_root_stats

    torch.cuda.set_device(local)
    if world > 1:
        init_dist(dist, torch, local)

    def barrier():
        if world > 1:
            dist.barrier()

    def max_over_ranks(x: float) -> float:
        if world == 1:
            return x
        t = torch.tensor([x], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    def sum_over_ranks(x: int) -> int:
        if world == 1:
            return x
        t = torch.tensor([x], dtype=torch.int64, device="cuda")
        dist.all_reduce(t)
        return int(t.item())

    m = pkg.Mcts(c_uct=1.0, scheme="block", device=local)
    stream = torch.cuda.current_stream()
    leaf_base = rank * N_LEAVES
    d_leaves = dev.gen_positions(m, GEN_SEED, N_LEAVES, LMIN, LMAX)
    d_out = dev.empty_wdl(N_LEAVES)
    d_plies = torch.zeros(1, dtype=torch.int64, device="cuda")
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")  # > 126 MB L2

    def step():
        m.playouts_async(d_leaves.data_ptr(), N_LEAVES, N_PER_LEAF, PLAYOUT_SEED, leaf_base,
                         d_out.data_ptr(), d_plies.data_ptr(), stream)

    log('for _ in range(args.warmup):\n ')
    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    d_plies.zero_()

    clk_path = os.path.join(tempfile.gettempdir(), f"bench_clocks_{os.getpid()}.csv")
    sampler, sampler_f = clocks_sampler(clk_path)
    time.sleep(0.3)
    starts = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    ends = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    barrier()
    torch.cuda.synchronize()
    for i in range(args.steps):
        flush.zero_()  # L2 flush outside the timed events
        starts[i].record(stream)
        step()
        ends[i].record(stream)
    torch.cuda.synchronize()
    barrier()
    kernel_ms = sum(s.elapsed_time(e) for s, e in zip(starts, ends))
    plies_local = int(d_plies.item())
    t_ms = max_over_ranks(kernel_ms)
    plies_total = sum_over_ranks(plies_local)
    playouts_total = world * args.steps * N_LEAVES * N_PER_LEAF
    head = headline(playouts_total, plies_total, t_ms, args.steps)

    log('# ---- end to end')
    # ---- end to end through the C ABI with host buffers (H2D + kernel + D2H)
    h_leaves = torch.empty((N_LEAVES, 3), dtype=torch.int64).pin_memory()
    h_leaves.copy_(d_leaves.cpu())
    h_out = torch.empty((N_LEAVES, 3), dtype=torch.int32).pin_memory()
    e2e_steps = max(3, args.steps // 2)
    for _ in range(2):
        m.playouts_host_ptr(h_leaves.data_ptr(), N_LEAVES, N_PER_LEAF, PLAYOUT_SEED, h_out.data_ptr())
    barrier()
    t0 = time.perf_counter()
    for _ in range(e2e_steps):
        m.playouts_host_ptr(h_leaves.data_ptr(), N_LEAVES, N_PER_LEAF, PLAYOUT_SEED, h_out.data_ptr())
    e2e_s = max_over_ranks(time.perf_counter() - t0)
    barrier()
    e2e_value = world * e2e_steps * N_LEAVES * N_PER_LEAF / e2e_s
    # ---- the same steps pipelined through mcts_playouts_host_async (step i+1's
    # copies and launch are enqueued while step i runs; every step still copies
    # its leaves in and its counts and ply count out through pinned host memory)
    h_outs = [torch.empty((N_LEAVES, 3), dtype=torch.int32).pin_memory() for _ in range(2)]
    h_plies = torch.zeros(2, dtype=torch.int64).pin_memory()
    for i in range(8):  # one call per staging slot (MCTS_HOST_ASYNC_SLOTS): allocation outside the timing
        m.playouts_host_async(h_leaves.data_ptr(), N_LEAVES, N_PER_LEAF, PLAYOUT_SEED, h_outs[i % 2].data_ptr(),
                              h_plies.data_ptr() + 8 * (i % 2), stream)
    stream.synchronize()
    barrier()
    t0 = time.perf_counter()
    for i in range(e2e_steps):
        m.playouts_host_async(h_leaves.data_ptr(), N_LEAVES, N_PER_LEAF, PLAYOUT_SEED, h_outs[i % 2].data_ptr(),
                              h_plies.data_ptr() + 8 * (i % 2), stream)
    stream.synchronize()
    e2e_pipe_s = max_over_ranks(time.perf_counter() - t0)
    barrier()
    e2e_pipe_value = world * e2e_steps * N_LEAVES * N_PER_LEAF / e2e_pipe_s
    if not torch.equal(h_outs[0], h_out):
        raise RuntimeError("mcts_playouts_host_async and mcts_playouts disagree")

    log('# ---- opening-phase batch')
    # ---- the same kernel on an opening-phase batch (L in [0, 8] random plies:
    # the ~60-ply regime of playouts near the root), device-timed the same way
    d_open = dev.gen_positions(m, GEN_SEED, N_LEAVES, OPEN_LMIN, OPEN_LMAX)
    d_plies.zero_()
    open_steps = max(3, args.steps // 4)
    m.playouts_async(d_open.data_ptr(), N_LEAVES, N_PER_LEAF, PLAYOUT_SEED, leaf_base,
                     d_out.data_ptr(), 0, stream)
    torch.cuda.synchronize()
    barrier()
    o_ms = 0.0
    for _ in range(open_steps):
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        m.playouts_async(d_open.data_ptr(), N_LEAVES, N_PER_LEAF, PLAYOUT_SEED, leaf_base,
                         d_out.data_ptr(), d_plies.data_ptr(), stream)
        e1.record(stream)
        torch.cuda.synchronize()
        o_ms += e0.elapsed_time(e1)
    o_ms = max_over_ranks(o_ms)
    o_plies = sum_over_ranks(int(d_plies.item()))
    opening_batch = {
        "workload": f"{N_LEAVES} synthetic opening-phase positions (seed {GEN_SEED}, "
                    f"{OPEN_LMIN}-{OPEN_LMAX} random plies) x {N_PER_LEAF} playouts per GPU",
        "playouts_per_s": world * open_steps * N_LEAVES * N_PER_LEAF / (o_ms / 1e3),
        "plies_per_s": o_plies / (o_ms / 1e3), "ms_per_step": o_ms / open_steps,
    }

    log('# ---- block-parallel search')
    # ---- block-parallel search (configs[2] shape) and leaf-parallel comparison
    # (configs[3]), time mode (or --search-iters for profiling), + root allreduce
    search = None
    leaf_search = None
    tree_search = None
    hosted_search = None
    launches = args.steps  # one playouts_kernel per timed step (the headline region)

    def run_search(handle, n_trees, threads, id_base, it_scale=1):
        # it_scale: the shared tree's iteration budget is a total over its workers
        root = pkg.position(*pkg.OPENING)
        st = torch.zeros(STATS_LEN, dtype=torch.int64, device="cuda")
        it, ms = (args.search_iters * it_scale, 0.0) if args.search_iters else (0, args.search_ms)
        # warm-up with the same budget: the time-sized node pool and the ln table
        # are allocated here, not inside the timed search
        handle.search_async(root, it, ms, n_trees, threads, 999, id_base, st.data_ptr(), stream)
        torch.cuda.synchronize()
        barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        # a ~250 ms spin kernel ahead of e0 holds the stream while the host
        # validates and enqueues the search, so the events bracket device work
        # only (r2x / r2zb / r2zp saw 12 / 49 / 35 ms host-side gaps inside the
        # window, r2zp behind a 50 ms gate: host CUDA calls stalled while the
        # nvidia-smi clock sampler ran)
        with torch.cuda.stream(stream):
            torch.cuda._sleep(SEARCH_GATE_CYCLES)
        e0.record(stream)
        handle.search_async(root, it, ms, n_trees, threads, 1000, id_base, st.data_ptr(), stream)
        with torch.cuda.stream(stream):
            merge_root_stats(st)  # the single cross-GPU collective (no-op at N=1)
        e1.record(stream)
        torch.cuda.synchronize()
        t_ms = max_over_ranks(e0.elapsed_time(e1))
        return st.cpu().numpy(), t_ms

    if not args.no_search:
        mode = (f"{args.search_iters} iterations" if args.search_iters else
                f"{args.search_ms:.0f} ms time mode")
        st, s_ms = run_search(m, SEARCH_TREES, SEARCH_THREADS, rank * SEARCH_TREES)
        search = {
            "workload": f"configs[2] shape: {SEARCH_TREES} trees x {SEARCH_THREADS} threads per GPU, "
                        f"{mode}, opening root, C=1.0",
            "playouts_per_s": float(st[195]) / (s_ms / 1e3), "ms": s_ms,
            "iterations_per_tree": float(st[196]) / (SEARCH_TREES * world),
            "plies_per_s": float(st[197]) / (s_ms / 1e3),
            "best_move": int(pkg.best_move(st)), "allreduce": world > 1,
            "mean_depth": float(st[198]) / max(float(st[196]), 1.0), **pool_info(st),
            # the playout kernel's measured instructions per ply (the search
            # kernel's playouts run the same loop), per GPU
            "roofline_frac": float(st[197]) / world / (s_ms / 1e3) * ops_per_ply("playouts")[0]
                             / integer_peak()[0],
        }
        log('ml = pkg.Mcts(')
        ml = pkg.Mcts(c_uct=1.0, scheme="leaf", device=local)
        lt, l_ms = run_search(ml, 1, LEAF_THREADS, rank)
        leaf_search = {
            "workload": f"configs[3]: 1 tree x {LEAF_THREADS} threads per leaf batch per GPU, {mode}",
            "playouts_per_s": float(lt[195]) / (l_ms / 1e3), "ms": l_ms,
            "iterations": float(lt[196]) / world, "plies_per_s": float(lt[197]) / (l_ms / 1e3),
            "best_move": int(pkg.best_move(lt)), "mean_depth": float(lt[198]) / max(float(lt[196]), 1.0),
            **pool_info(lt),
        }
        ml.close()
        log('mt = pkg.Mcts(')
        mt = pkg.Mcts(c_uct=1.0, scheme="tree", device=local)
        tt, tree_ms = run_search(mt, SEARCH_TREES, SEARCH_THREADS, rank, it_scale=SEARCH_TREES)
        tree_search = {
            "workload": f"NEXT-4 tree parallelism: one shared tree, {SEARCH_TREES} workers x {SEARCH_THREADS} "
                        f"threads per GPU, {mode}, opening root, C=1.0",
            "playouts_per_s": float(tt[195]) / (tree_ms / 1e3), "ms": tree_ms,
            "iterations": float(tt[196]) / world, "plies_per_s": float(tt[197]) / (tree_ms / 1e3),
            "best_move": int(pkg.best_move(tt)), "mean_depth": float(tt[198]) / max(float(tt[196]), 1.0),
            **pool_info(tt),
        }
        mt.close()
        if rank == 0:  # NEXT-1: the paper's CPU-managed trees + hybrid CPU work (single GPU)
            hosted_search = hosted_leg(m, args.search_ms)

    log('if sampler is not None:')
    if sampler is not None:
        sampler.terminate()
        sampler.wait()
        sampler_f.close()
    clocks = clocks_summary(clk_path, local)

    if rank != 0:
        if world > 1:
            dist.destroy_process_group()
        return

    peak_ops, peak_basis, alu_peak = integer_peak()
    kern_s = kernel_ms / 1e3 / args.steps
    plies_per_launch = plies_local / args.steps
    opp, opp_basis = ops_per_ply("playouts", plies_per_launch)
    roof = roofline(plies_per_launch, kern_s, peak_ops, opp, opp_basis, alu_peak, peak_basis)
    traffic, ncu = None, None
    try:  # from the committed ncu --set full capture of this kernel (profiles/latest_ncu.json)
        prof = json.load(open(os.path.join(ROOT, "profiles", "latest_ncu.json")))["playouts"]
        if prof.get("source_hash") == kernel_source_hash():
            traffic = prof["dram_bytes_per_launch"]
            ncu = {k: prof.get(k) for k in ("alu_pipe_pct", "fmaheavy_pipe_pct", "issue_active_pct",
                                            "lanes_active_per_inst", "thread_inst", "duration_us",
                                            "source_hash", "capture")}
    except Exception:
        pass
    roof["traffic"] = traffic
    roof["ncu"] = ncu
    line = {
        "metric": METRIC, "value": head["value"], "unit": "playouts/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": head["ms_per_step"],
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u64",
        "data": "synthetic",
        "config": {"workload": "configs[1]: 4096 synthetic mid-game positions (seed 2, 20-40 random "
                               "plies) x 256 random playouts per GPU",
                   "global_batch": world * N_LEAVES * N_PER_LEAF,
                   "parallelism": f"leaf-range x{world} (weak)",
                   "l2": "flushed between steps (256 MiB write outside the timed events)"},
        "plies_per_s": head["plies_per_s"],
        "roofline": roof,
        "e2e": {"value": e2e_value, "unit": "playouts/s",
                "h2d_bytes_per_step": N_LEAVES * 24, "d2h_bytes_per_step": N_LEAVES * 12 + 8,
                "api": "mcts_playouts (host buffers, pinned; synchronous per step)",
                "pipelined": {"value": e2e_pipe_value, "unit": "playouts/s",
                              "api": "mcts_playouts_host_async (host buffers, pinned; steps enqueued back "
                                     "to back on one stream, one synchronisation at the end)"}},
        "gpu_launches": launches,
        "clocks": clocks,
        "opening_batch": opening_batch, "search": search, "leaf_search": leaf_search,
        "tree_search": tree_search, "hosted_search": hosted_search,
    }
    log('if not args.no_cpu and world =')
    if not args.no_cpu and world == 1:
        try:
            line["cpu_baseline"] = cpu_baseline()
        except Exception as e:  # the oracle is optional on the bench path
            line["cpu_baseline"] = {"error": str(e)}
    print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
