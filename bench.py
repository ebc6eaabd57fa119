#!/usr/bin/env python
"""Benchmark: one IMM run (eim_imm_run: theta estimation + RRR sampling +
greedy NodeSelection, every row of SURVEY §8(a)) per step on the BASELINE
configs[1] workload (LiveJournal-shaped R-MAT, IC weighted cascade, k=50,
eps=0.5, ell=1), graph resident in HBM.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl eim|reference] [--config C2]

Prints ONE JSON line on rank 0.  `value` = RRR sets per second of whole IMM
runs (theta / IMM seconds, all ranks together); traversed edges/s and IMM
seconds ride along.  See DESIGN.md §7 for every field.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

LT_STEP_BYTES = 24.0  # LT walk step on the walk store: 16-B entry + 8-B table key
METRIC = "RRR sets/s, traversed edges/s, end-to-end IMM s (k=50, eps=0.5) at 1/2/4/8 B200"
UNIT = "RRR sets/s"
GRAPH_SEED = 1
RUN_SEED = 1
# ALU roofline of the IC sampler: every examined in-edge costs
# one Philox4x32-10 word; the roof is the Philox word rate of this GPU,
# measured live by tools/philox_roof (wide multiplies run at a quarter of the
# issue rate; the sampler's form hoists the sample-constant work of rounds
# 0-1: 18 instead of 20 per call), the best form counts.  Fallback: the
# committed measurement in profiles/philox_roof.json.
PHILOX_PROBE = os.path.join(ROOT, "tools", "philox_roof", "philox_roof")


def philox_roof_gwords():
    """(peak Gwords/s, source, probe lines): the probe output rides along in
    the bench line (roofline.peak_probe), so the peak used is on record."""
    try:
        out = subprocess.run([PHILOX_PROBE], capture_output=True, text=True, timeout=60).stdout
        lines = [json.loads(l) for l in out.splitlines() if l.startswith("{")]
        if lines:
            return max(l["words_per_s"] for l in lines) / 1e9, "measured live (tools/philox_roof)", lines
    except Exception:
        pass
    try:
        with open(os.path.join(ROOT, "profiles", "philox_roof.json")) as f:
            return json.load(f)["roof_words_per_s"] / 1e9, "profiles/philox_roof.json (earlier measurement)", []
    except Exception:
        return 1630.0, "fallback constant", []


GATHER_PROBE = os.path.join(ROOT, "tools", "gather_roof", "gather_roof")


def gather_roof(walkers):
    """(steps/s, probe line) of tools/gather_roof --cas at the LT round's
    concurrency: random dependent 16-B loads over a walk-store-sized buffer
    plus one table CAS per step -- the roof of a walk step."""
    try:
        out = subprocess.run([GATHER_PROBE, "--cas"], capture_output=True, text=True, timeout=120).stdout
        lines = [json.loads(l) for l in out.splitlines() if l.startswith("{")]
        best = min(lines, key=lambda l: abs(l["walkers"] - walkers))
        return best["steps_per_s"], lines
    except Exception:
        return None, []


def ncu_traffic(model):
    """DRAM bytes per launch of the dominant kernel from the newest committed
    `ncu --set full` summary of this round (profiles/r02_*), else round 1's."""
    names = (["r02_ncu_ic_kernel.json", "ncu_sampler.json"] if model == "IC" else
             ["r02_ncu_lt_aug_kernel.json", "ncu_sampler_lt.json"])
    for nm in names:
        path = os.path.join(ROOT, "profiles", nm)
        if not os.path.exists(path):
            continue
        try:
            ls = [l for l in json.load(open(path))["launches"] if "dram_bytes" in l]
            if ls:
                return sum(l["dram_bytes"] for l in ls) / len(ls), f"profiles/{nm}"
        except Exception:
            continue
    return None, None


def _peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return json.load(f)
    except Exception:
        return {}


def workload_desc(cfg_name):
    import inputs
    c = inputs.CONFIGS[cfg_name]
    return (f"{cfg_name} {c['name']} R-MAT n={c['n']} m={c['m']} (a,b,c)=(0.57,0.19,0.19) graph seed {GRAPH_SEED}, "
            f"{c['model']}-WC, k={c['k']}, eps={c['eps']}, ell={c['ell']}, run seed {RUN_SEED}")


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled every 200 ms during the timed region."""

    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, device):
        self.device = device
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.device), f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                 "-lms", "200"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.proc = None
        return self

    def __exit__(self, *a):
        self.out = ""
        if self.proc:
            time.sleep(0.25)
            self.proc.terminate()
            try:
                self.out, _ = self.proc.communicate(timeout=5)
            except Exception:
                self.proc.kill()

    def summary(self):
        rows = []
        for line in (getattr(self, "out", "") or "").strip().splitlines():
            p = [x.strip() for x in line.split(",")]
            if len(p) >= 9:
                rows.append(p)
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unavailable"], "samples": 0}
        sm = [float(r[1]) for r in rows if r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in rows if r[2].replace(".", "").isdigit()]
        reasons = set()
        for r in rows:
            for name, val in zip(("hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"), r[5:9]):
                if val.lower().startswith("active"):
                    reasons.add(name)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(rows)}


def run_reference(args):
    """The reference arm: the CPU oracle as it stands, one full IMM of the same
    workload per step (same metric: theta / IMM seconds).  Warm-up steps only
    page the graph in (a 64-id oracle sample each): the oracle keeps no state
    between calls, so a warm-up IMM would measure nothing new."""
    import inputs
    import oracle
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    c = inputs.CONFIGS[args.config]
    off, nbr = inputs.config_graph(args.config, seed=GRAPH_SEED)
    cores = max(1, min(64, os.cpu_count() or 1))
    for w in range(args.warmup):
        oracle.sample(off, nbr, c["model"], RUN_SEED, w * 64, 64, nthreads=cores)
    times, theta = [], None
    for _ in range(args.steps):
        t0 = time.perf_counter()
        r = oracle.imm(off, nbr, c["k"], c["eps"], c["ell"], c["model"], RUN_SEED, nthreads=cores)
        times.append(time.perf_counter() - t0)
        theta = r["theta"]
    dt = sum(times)
    v = args.steps * theta / dt
    line = {
        "impl": "reference", "metric": METRIC, "value": v, "unit": UNIT, "n_gpus": args.gpus, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": dt * 1e3 / args.steps, "higher_is_better": True, "scaling": "strong",
        "vs_baseline": None, "dtype": "u32", "data": "synthetic",
        "config": {"workload": workload_desc(args.config), "theta": theta},
        "imm_s": dt / args.steps,
        "cpu_baseline": {"value": v, "unit": UNIT, "cores": cores, "kind": "oracle",
                         "sample": f"per step: one full oracle IMM run of the workload (theta={theta}; sampling on "
                                   f"{cores} threads, greedy single-threaded), the same work as the GPU arm's step"},
        "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def cpu_baseline(args, off, nbr):
    import inputs
    import oracle
    c = inputs.CONFIGS[args.config]
    cores = max(1, min(64, os.cpu_count() or 1))
    t0 = time.perf_counter()
    r = oracle.imm(off, nbr, c["k"], c["eps"], c["ell"], c["model"], RUN_SEED, nthreads=cores)
    dt = time.perf_counter() - t0
    return {"value": r["theta"] / dt, "unit": UNIT, "cores": cores, "kind": "oracle",
            "sample": f"one full oracle IMM run of the workload ({dt:.1f} s wall; sampling on {cores} threads, "
                      f"greedy single-threaded); theta={r['theta']}", "seconds": dt,
            "seeds_match": None, "_seeds": r["seeds"].tolist(), "_theta": r["theta"]}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="eim", choices=["eim", "reference"])
    ap.add_argument("--config", default="C2")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--budget-ids", type=int, default=1 << 24,
                    help="fixed sample budget of the sampler-throughput leg, SURVEY 8(d): ids [0, 2^24) (0: skip)")
    ap.add_argument("--variant-steps", type=int, default=3,
                    help="timed steps of each NEXT-row variant (log-encoded store, source elimination, "
                         "fresh final phase); 0: skip")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)
    if args.impl == "reference":
        return run_reference(args)

    import numpy as np
    import torch
    import torch.distributed as dist

    import inputs
    import paper_conf_sc_doneyhl25_b200 as eim

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
    c = inputs.CONFIGS[args.config]
    off, nbr = inputs.config_graph(args.config, seed=GRAPH_SEED)
    n, m = off.size - 1, nbr.size

    nccl_id = None
    if world > 1:
        obj = [eim.eim_nccl_get_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        nccl_id = obj[0]
    stream = torch.cuda.Stream(dev)
    torch.cuda.set_stream(stream)
    ctx = eim.eim_create(local, rank, world, nccl_id, stream.cuda_stream)
    g = eim.eim_load_graph_csr(ctx, off, nbr)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize(dev)

    def step():
        return eim.eim_imm_run(ctx, g, c["k"], c["eps"], c["ell"], c["model"], RUN_SEED)

    for _ in range(args.warmup):
        seeds, theta, spread, st = step()
    stats = []
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    with ClockSampler(local) as clocks:
        # extra untimed steps so the clock sampler sees the GPU under load
        for _ in range(2):
            step()
        barrier()
        for i in range(args.steps):
            flush.zero_()  # L2 flush (256 MiB > 126 MB L2), outside the timed events
            ev[i][0].record(stream)
            seeds, theta, spread, st = step()
            ev[i][1].record(stream)
            stats.append(st)
        barrier()
    ms = sum(a.elapsed_time(b) for a, b in ev)
    t = torch.tensor([ms], dtype=torch.float64, device=dev)
    edges = torch.tensor([float(sum(s["edges_examined"] for s in stats))], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        dist.all_reduce(edges, op=dist.ReduceOp.SUM)
    ms_per_step = float(t.item()) / args.steps
    theta_all = stats[-1]["theta"]
    value = theta_all / (ms_per_step / 1e3)

    # dominant kernel: the sampler; per-launch duration from CUDA events on its stream
    k_ms = sum(s["ms_sample_kernel"] for s in stats)
    k_launch = sum(s["sample_launches"] for s in stats)
    k_edges_local = sum(s["edges_examined"] for s in stats)
    probe = []
    if c["model"] == "IC":
        peak, peak_src, probe = philox_roof_gwords() if rank == 0 else (1630.0, "", [])
        achieved = (k_edges_local / k_launch) / (k_ms / k_launch / 1e3) / 1e9 if k_ms > 0 else None
    else:
        # LT walk step on the walk store: one 16-B entry (v, d(v), off[v]) + one
        # 8-B membership-table key = 24 algorithmic bytes
        peak = float(_peaks().get("hbm_gbs", 8000.0))
        peak_src = "MEASURED_PEAKS.json hbm_gbs" if "hbm_gbs" in _peaks() else "fallback 8 TB/s"
        achieved = (LT_STEP_BYTES * k_edges_local / k_launch) / (k_ms / k_launch / 1e3) / 1e9 if k_ms > 0 else None
    traffic, traffic_src = ncu_traffic(c["model"])  # DRAM bytes per launch, committed ncu --set full capture
    lt_ra = None
    if c["model"] == "LT" and k_ms > 0 and rank == 0:
        # the walk step is a random dependent access: its roof is the random
        # dependent-load + CAS rate at the round's concurrency (tools/gather_roof)
        ra_peak, ra_probe = gather_roof(stats[-1]["theta"])
        ra_ach = (k_edges_local / k_launch) / (k_ms / k_launch / 1e3)
        lt_ra = {"achieved_steps_per_s": ra_ach, "peak_steps_per_s": ra_peak,
                 "frac": (ra_ach / ra_peak) if ra_peak else None, "probe": ra_probe,
                 "basis": "walk steps/s of lt_aug_kernel vs tools/gather_roof --cas (random dependent 16-B loads "
                          "over a 1.9-GB buffer + one CAS into a 2^25-slot table per step, same number of walkers)"}
    # the greedy pick kernel: latency-bound (two grid barriers and ~4 dependent
    # L2 round trips per pick), reported as device time per pick
    g_ms = sum(s["ms_select_kernel"] for s in stats)
    g_picks = sum(s["select_picks"] for s in stats)
    greedy_line = {"kernel": "greedy_kernel (k greedy picks per NodeSelection, cooperative)", "bound": "latency",
                   "us_per_pick": (g_ms * 1e3 / g_picks) if g_picks else None,
                   "selections_per_imm": stats[-1]["select_launches"], "picks_per_imm": stats[-1]["select_picks"],
                   "kernel_ms_per_imm": g_ms / args.steps,
                   "note": "concurrent selections (the rounds one sampler launch covers) each count their "
                           "device time"}

    # end to end through the public API with host buffers: H2D of the graph
    # from pinned memory + IMM + D2H of the result, every step
    off_p = torch.from_numpy(off).pin_memory()
    nbr_p = torch.from_numpy(nbr).pin_memory()
    e2e_ms = []
    for i in range(args.e2e_steps + 1 if args.e2e_steps > 0 else 0):
        flush.zero_()
        barrier()
        t0 = time.perf_counter()
        g2 = eim.eim_load_graph_csr_ptr(ctx, n, m, off_p.data_ptr(), nbr_p.data_ptr())
        s2, th2, sp2, _ = eim.eim_imm_run(ctx, g2, c["k"], c["eps"], c["ell"], c["model"], RUN_SEED)
        eim.eim_graph_free(g2)
        torch.cuda.synchronize(dev)
        dt = (time.perf_counter() - t0) * 1e3
        if i > 0:
            e2e_ms.append(dt)
        assert np.array_equal(s2, seeds) and th2 == theta_all
    # sampler throughput on a fixed sample budget: theta-
    # independent, so the rate is not masked by the IMM rounds' tails.  This
    # rank samples its share of ids [0, B); device time of the sampler kernels.
    # NEXT-row variants: the same IMM with the log-encoded graph
    # store (NEXT-2), source-vertex elimination (NEXT-1) and the fresh final
    # phase (NEXT-4); CUDA events on the same stream, L2 flushed between steps.
    variants = []
    if args.variant_steps > 0 and world == 1:
        g_packed = eim.eim_load_graph_csr(ctx, off, nbr, gflags=eim.EIM_G_LOG_ENCODE)
        # NEXT-3 layout: the weighted-cascade probabilities given as per-edge
        # thresholds (R25), streamed from HBM -- same results as the plain run
        d = np.diff(off).astype(np.uint64)
        if c["model"] == "IC":
            x_wc = (np.uint64(2**32 - 1) // np.repeat(d, d.astype(np.int64))).astype(np.uint32)
        else:
            x_wc = None  # LT: the WC run needs no weights; the general LT path is covered by the parity tests
        g_w = eim.eim_load_graph_csr(ctx, off, nbr, edge_x=x_wc) if x_wc is not None else None
        runs = [("log_encoded_store", g_packed, 0),
                ("source_elim", g, eim.EIM_F_SOURCE_ELIM),
                ("source_elim+log_encoded_store", g_packed, eim.EIM_F_SOURCE_ELIM),
                ("fresh_final", g, eim.EIM_F_FRESH_FINAL)]
        if g_w is not None:
            runs.append(("per_edge_thresholds", g_w, 0))
        for name, gv, flags in runs:
            for _ in range(2):
                eim.eim_imm_run(ctx, gv, c["k"], c["eps"], c["ell"], c["model"], RUN_SEED, flags=flags)
            vms, vst = 0.0, None
            for _ in range(args.variant_steps):
                flush.zero_()
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(stream)
                vs, vth, vsp, vst = eim.eim_imm_run(ctx, gv, c["k"], c["eps"], c["ell"], c["model"], RUN_SEED,
                                                    flags=flags)
                b.record(stream)
                torch.cuda.synchronize(dev)
                vms += a.elapsed_time(b)
            vms /= args.variant_steps
            variants.append({"variant": name, "ms_per_step": vms, "rrr_sets_per_s": vth / (vms / 1e3),
                             "theta": vth, "ids_sampled": vst["ids_sampled"], "arena_elems": vst["arena_elems"],
                             "arena_bytes": vst["arena_bytes"], "graph_bytes": eim.eim_graph_bytes(gv),
                             "edges_examined": vst["edges_examined"],
                             "sample_kernel_ms": vst["ms_sample_kernel"], "select_ms": vst["ms_select"],
                             "seeds_head": vs[:5].tolist(),
                             "seeds_equal_plain": bool(np.array_equal(vs, seeds)) if flags == 0 else None})
            if name == "per_edge_thresholds" and vst["ms_sample_kernel"] > 0:
                # 4 B of threshold per examined in-edge streamed from HBM (plus the
                # WC path's per-vertex bytes): the HBM-bound layout of SURVEY §8(d)
                gbs = 4.0 * vst["edges_examined"] / (vst["ms_sample_kernel"] / 1e3) / 1e9
                hbm = float(_peaks().get("hbm_gbs", 8000.0))
                variants[-1]["threshold_stream_gbs"] = gbs
                variants[-1]["threshold_stream_frac_hbm"] = gbs / hbm
                variants[-1]["edges_per_s"] = vst["edges_examined"] / (vst["ms_sample_kernel"] / 1e3)
                if args.budget_ids > 0:  # the same layout on the fixed sample budget (no round tails)
                    sb = eim.eim_sample_rrr_stats(ctx, gv, c["model"], RUN_SEED, 0, args.budget_ids)
                    bgbs = 4.0 * sb["edges_examined"] / (sb["ms_sample_kernel"] / 1e3) / 1e9
                    variants[-1]["fixed_budget"] = {
                        "ids": args.budget_ids, "kernel_ms": sb["ms_sample_kernel"],
                        "edges_per_s": sb["edges_examined"] / (sb["ms_sample_kernel"] / 1e3),
                        "threshold_stream_gbs": bgbs, "threshold_stream_frac_hbm": bgbs / hbm}
        eim.eim_graph_free(g_packed)
        if g_w is not None:
            eim.eim_graph_free(g_w)
    budget = None
    if args.budget_ids > 0:
        lo_b, hi_b = eim.eim_shard_range(0, args.budget_ids, rank, world)
        eim.eim_sample_rrr(ctx, g, c["model"], RUN_SEED, lo_b, min(hi_b - lo_b, 4096))  # warm-up
        sb = eim.eim_sample_rrr_stats(ctx, g, c["model"], RUN_SEED, lo_b, hi_b - lo_b)
        bt = torch.tensor([sb["ms_sample_kernel"], float(sb["edges_examined"])], dtype=torch.float64, device=dev)
        if world > 1:
            bmax = bt[:1].clone()
            dist.all_reduce(bmax, op=dist.ReduceOp.MAX)
            dist.all_reduce(bt, op=dist.ReduceOp.SUM)
            bt[0] = bmax[0]
        b_ms, b_edges = float(bt[0].item()), float(bt[1].item())
        budget = {"ids": args.budget_ids, "kernel_ms": b_ms, "sets_per_s": args.budget_ids / (b_ms / 1e3),
                  "edges_per_s": b_edges / (b_ms / 1e3), "edges": b_edges, "launches": sb["sample_launches"]}
    te = torch.tensor([statistics.mean(e2e_ms) if e2e_ms else float("nan")], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(te, op=dist.ReduceOp.MAX)
    e2e_ms_step = float(te.item())

    out = None
    if rank == 0:
        cb = None
        if world == 1 and not args.no_cpu_baseline:
            cb = cpu_baseline(args, off, nbr)
            cb["seeds_match"] = bool(cb.pop("_seeds") == seeds.tolist() and cb.pop("_theta") == theta_all)
        clk = clocks.summary()
        out = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "u32", "data": "synthetic",
            "config": {"workload": workload_desc(args.config), "theta": theta_all,
                       "parallelism": f"sample-range dp{world} (graph replicated)",
                       "l2": f"flushed between steps (256 MiB write); graph {(off.nbytes + nbr.nbytes) / 1e6:.0f} MB > 126 MB L2"},
            "imm_s": ms_per_step / 1e3,
            "traversed_edges_per_s": float(edges.item()) / (ms * 1e-3) if world == 1 else float(edges.item()) / (float(t.item()) * 1e-3),
            "sampler_sets_per_s": theta_all / (sum(s["ms_sample"] for s in stats) / args.steps / 1e3),
            "phase_ms": {"sample": sum(s["ms_sample"] for s in stats) / args.steps,
                         "sample_kernel": k_ms / args.steps,
                         "select_kernel": g_ms / args.steps,
                         "select": sum(s["ms_select"] for s in stats) / args.steps,
                         "comm": sum(s["ms_comm"] for s in stats) / args.steps},
            "roofline": ({"bound": "alu", "kernel": "ic_kernel (IC sampler, incl. split-off tasks)", "achieved": achieved,
                          "peak": peak, "unit": "Gedge/s", "frac": (achieved / peak) if achieved else None,
                          "traffic": traffic, "traffic_source": traffic_src,
                          "peak_basis": "Philox4x32-10 word rate of this GPU (one word per examined in-edge; best of the "
                                        "plain and the sampler's hoisted form, tools/philox_roof), "
                                        + peak_src + "; DESIGN.md §6", "peak_probe": probe} if c["model"] == "IC" else
                         {"bound": "hbm", "kernel": "lt_aug_kernel (LT reverse walks on the walk store)", "achieved": achieved,
                          "peak": peak, "unit": "GB/s", "frac": (achieved / peak) if achieved else None,
                          "traffic": traffic, "traffic_source": traffic_src,
                          "peak_basis": f"{LT_STEP_BYTES:.0f} algorithmic bytes per walk step; " + peak_src + "; DESIGN.md §6",
                          "random_access": lt_ra}),
            "greedy": greedy_line,
            # IC: examined edges/s vs the Philox roof; LT: LT_STEP_BYTES per walk step vs HBM
            "sampler_fixed_budget": (dict(budget, frac=(budget["edges_per_s"] / 1e9 / world / peak)
                                          if c["model"] == "IC" else
                                          (LT_STEP_BYTES * budget["edges_per_s"] / 1e9 / world / peak))
                                     if budget else None),
            "cpu_baseline": cb,
            "e2e": {"value": theta_all / (e2e_ms_step / 1e3), "unit": UNIT,
                    "h2d_bytes_per_step": int(off.nbytes + nbr.nbytes), "d2h_bytes_per_step": int(4 * c["k"] + 16),
                    "ms_per_step": e2e_ms_step},
            "gpu_launches": int(sum(s["kernel_launches"] for s in stats)),
            "memory": {"graph_bytes": eim.eim_graph_bytes(g), "arena_bytes": stats[-1]["arena_bytes"],
                       "graph_bytes_log_encoded": next((v["graph_bytes"] for v in variants
                                                        if v["variant"] == "log_encoded_store"), None)},
            "variants": variants,
            "clocks": clk,
            "result": {"seeds_head": seeds[:10].tolist(), "theta": theta_all, "spread": spread,
                       "rounds": stats[-1]["rounds"], "spilled_samples": stats[-1]["spilled_samples"],
                       "edges_examined": stats[-1]["edges_examined"]},
        }
        print(json.dumps(out), flush=True)
    eim.eim_graph_free(g)
    eim.eim_destroy(ctx)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
