#!/usr/bin/env python
"""bench.py — ATF search-space generation on B200 (BASELINE.json metric:
"valid configs generated/sec (and constraint evals/sec) at 1/2/4/8 B200 vs roofline").

Workload (config.workload): C5 = BASELINE.json configs[4], the 24-parameter,
3-group chained-divisibility space over ranges 1..4096 — the config the metric is
quoted on at 1/2/4/8 GPUs (sharded).  One step = one complete generation of every
group's tree (all §8(a) rows: count, scan, emit on every level, group sizes, S).
At N=1 rank 0 also measures the other configs (C3-IS2/IS4 generation, C4 decode of
10^8 indices, C2) and reports them under "secondary".

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]

--impl reference times the CPU oracle (oracle/atf_oracle, as it stands) on the
host cores on a bounded sample of the same workload.
"""
import argparse
import json
import os
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import atfspec as A  # noqa: E402

METRIC = "valid configs generated/sec (and constraint evals/sec) at 1/2/4/8 B200 vs roofline"


def _peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return json.load(f)
    except OSError:
        return {}


def int_peak_ops(sm_mhz, sms=148):
    """INT32 issue bound: 4 SMSPs x 32 lanes x SMs x clock (one warp instruction per SMSP per
    cycle)."""
    return 4 * 32 * sms * sm_mhz * 1e6


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled DURING the timed region."""

    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.proc = None
        self.lines = []

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except OSError:
            self.proc = None
        time.sleep(0.25)
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def __exit__(self, *a):
        time.sleep(0.15)
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except subprocess.TimeoutExpired:
                self.proc.kill()

    def summary(self):
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 8:
                continue
            try:
                sm.append(float(f[0]))
                mx = float(f[1])
            except ValueError:
                continue
            for nm, v in zip(names, f[4:8]):
                if v.lower() == "active":
                    reasons.add(nm)
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": mx,
                "reasons": sorted(reasons), "samples": len(sm)}


def flush_l2(buf):
    buf.add_(1)  # 512 MiB write > 126 MB L2


# ------------------------------------------------------------------ our arm
# The headline evaluates EVERY (frontier node, candidate) pair: all f_{k-1} r_k candidate
# evaluations of the spec as written ("iterating over the constrained
# ranges").  The segment-bound variant (whole candidate segments of a divisibility filter
# rejected by their |x| bounds, same space) is reported as a secondary line.
def headline_flags():
    from paper_conf_hpdc_raschg18_b200 import _lib as L
    return L.ATF_FLAG_NO_SEG_BOUNDS


def run_generation(spec, steps, warmup, dist_ctx=None, timing=False, serial=False, flags=None):
    """Times `steps` generations of `spec`; returns per-step ms (max over ranks), stats.
    The production configuration runs the groups' levels concurrently (one stream per group)
    without per-level events; `timing` + `serial` is the roofline pass: the same kernels,
    groups one after another, CUDA events around every level and every expand kernel."""
    import torch
    from paper_conf_hpdc_raschg18_b200 import Space, _lib as L
    dev = torch.cuda.current_device()
    stream = torch.cuda.current_stream()
    flush = torch.empty(128 << 20, dtype=torch.int32, device="cuda")
    flags = (headline_flags() if flags is None else flags) | (L.ATF_FLAG_TIMING if timing else 0) | \
        (L.ATF_FLAG_SERIAL_GROUPS if serial else 0)
    sp = Space(spec, device=dev, stream=stream, flags=flags)
    world = dist_ctx["world"] if dist_ctx else 1
    rank = dist_ctx["rank"] if dist_ctx else 0

    def one_step():
        if world == 1:
            sp.generate()
            return None
        from paper_conf_hpdc_raschg18_b200.shard import generate_balanced
        return generate_balanced(sp)  # every level redistributed; one NCCL all-gather per round

    for _ in range(warmup):
        one_step()
        flush_l2(flush)
    torch.cuda.synchronize()
    if dist_ctx:
        dist_ctx["dist"].barrier()
    torch.cuda.synchronize()
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(steps)]
    level_ms, level_exp_ms = [], []
    for i in range(steps):
        evs[i][0].record(stream)
        one_step()
        evs[i][1].record(stream)
        if timing:
            sts = sp.stats()
            level_ms.append([s["ms"] for s in sts])
            level_exp_ms.append([s["expand_ms"] for s in sts])
        flush_l2(flush)
    torch.cuda.synchronize()
    if dist_ctx:
        dist_ctx["dist"].barrier()
    torch.cuda.synchronize()
    ms = [a.elapsed_time(b) for a, b in evs]
    st = sp.stats()
    launches = sum(x["launches"] for x in st)
    res = {"ms": ms, "stats": st, "size": sp.size(), "group_sizes": sp.group_sizes(),
           "plan": sp.plan_json(), "level_ms": level_ms, "level_exp_ms": level_exp_ms, "launches": launches}
    sp.close()
    return res


def _traffic_db():
    """ncu-measured DRAM bytes per launch (dram__bytes_read.sum + dram__bytes_write.sum from one
    `ncu --set full` capture), keyed "spec:g<group>:l<level>"; written by tools/traffic_db.py
    from the committed profiles/ captures."""
    try:
        with open(os.path.join(ROOT, "profiles", "traffic.json")) as f:
            return json.load(f)
    except OSError:
        return {}


def roofline_of(res, sm_mhz, spec_name=None, step_ms=None):
    """Roofline of the dominant kernel: the level-expansion launch with the largest
    device time.  achieved = its algorithmic integer ops (evals_k x c_k, the planner's cost table)
    / its average launch duration (CUDA events around the expand kernel alone, on the launch
    stream, in the serialized timing pass); peak = 4 SMSP x 32 lanes x SMs x clock (bound
    "alu").  "step" = all launches of a generation: ops of every level / the production
    step time (concurrent groups) when given, else the sum of the serialized level times."""
    plan = res["plan"]
    lv = [(gi, k, l) for gi, g in enumerate(plan["groups"]) for k, l in enumerate(g["levels"])]
    costs = [l["cost"] for _, _, l in lv]
    st = res["stats"]
    # evaluated pairs: the spec's f_{k-1} x r_k, less the pairs the warp-tile hot loop rejects
    # wholesale by its per-segment |x| bounds (stats "pairs", ATF_FLAG_TIMING)
    ops = [s["pairs"] * c for s, c in zip(st, costs)]   # timing pass: pairs = evaluated pairs
    exp_ms = np.array(res["level_exp_ms"], dtype=np.float64).mean(axis=0)
    lvl_ms = np.array(res["level_ms"], dtype=np.float64).mean(axis=0)
    d = int(np.argmax(exp_ms))
    g, k, _ = lv[d]
    peak = int_peak_ops(sm_mhz)
    achieved = ops[d] / (exp_ms[d] * 1e-3)
    W = plan["groups"][g].get("words", 4)
    f_prev = st[d]["evals"] // max(1, st[d]["r"])
    alg_bytes = f_prev * W * 4 + st[d]["f"] * W * 4 + (f_prev + 1) * 8
    tdb = _traffic_db()
    tr = tdb.get(f"{spec_name}:g{g}:l{k}") if spec_name else None
    kname = {0: "expand_narrow", 1: "expand_wide", 2: "expand_wtile", 3: "expand_nfast", 4: "atf_nfast_jit",
             5: "tail_count+tail_emit", 6: "atf_tail_count+atf_tail_emit (NVRTC)"}.get(st[d].get("kernel", -1), "expand")
    step_ops = float(sum(ops))
    step_ms = float(step_ms) if step_ms else float(lvl_ms.sum())
    return {"bound": "alu", "achieved": achieved / 1e12, "peak": peak / 1e12, "unit": "Tops/s",
            "frac": achieved / peak, "traffic": tr["dram_bytes"] if tr else None,
            "traffic_source": tr["source"] if tr else None,
            "kernel": kname, "launch": f"group {g} level {k + 1} (r={st[d]['r']}, evals={st[d]['evals']}, "
                                       f"evaluated pairs={st[d]['pairs']})",
            "ops_per_launch": ops[d], "launch_ms": float(exp_ms[d]), "algorithmic_bytes_per_launch": int(alg_bytes),
            "peak_clock_mhz": sm_mhz, "peak_source": "4 SMSP x 32 lanes x 148 SMs x clock (B200_PROFILING.md unit counts)",
            "cost_table": "DIVX/MULX/DIVPROD 2, QDIV 6, CMP 2, AND 1, GENERIC = bytecode ops",
            "step": {"ops": step_ops, "ms": step_ms, "achieved": step_ops / (step_ms * 1e-3) / 1e12,
                     "frac": step_ops / (step_ms * 1e-3) / peak,
                     "pairs_evaluated": int(sum(s["pairs"] for s in st)),
                     "pairs_decided": int(sum(s["evals"] for s in st))}}


def e2e_generation(spec, steps, dist_ctx=None):
    """Same metric through the public API from HOST inputs: every step builds a new space from
    the host spec (ranges + bytecode uploaded), generates it (sharded over the ranks when
    world > 1, counts all-gathered over NCCL) and reads S + the group sizes back.  Timed by the
    host clock around device-synchronised steps; max over ranks."""
    import torch
    from paper_conf_hpdc_raschg18_b200 import Space
    # per parameter the library uploads [values][magics][|values|] padded to 128 entries plus
    # the sorted value table (encode); constraint programs travel as kernel parameters
    h2d = sum(4 * len(c) for p in spec.params for c in p.constraints)
    for p in spec.params:
        r = p.range
        n = len(r["values"]) if r["kind"] == "set" else max(0, (r["end"] - r["begin"]) // r["step"] + 1)
        h2d += 12 * ((n + 127) // 128 * 128) + 8 * n
    times, d2h = [], 0
    warm = 3  # fresh-space steps discarded (allocator cache, NVRTC / module loads), as the device timing's W >= 3
    for i in range(steps + warm):
        torch.cuda.synchronize()
        if dist_ctx:
            dist_ctx["dist"].barrier()
        t0 = time.perf_counter()
        with Space(spec, flags=headline_flags()) as sp:
            if dist_ctx:
                from paper_conf_hpdc_raschg18_b200.shard import generate_balanced
                generate_balanced(sp)
            else:
                sp.generate()
            S = sp.size()
            gs = sp.group_sizes()
            nlev = sum(sp.num_levels(g) for g in range(len(gs)))
        torch.cuda.synchronize()
        dt = time.perf_counter() - t0
        if dist_ctx:
            t = torch.tensor([dt], dtype=torch.float64, device=dist_ctx["dev"])
            dist_ctx["dist"].all_reduce(t, op=dist_ctx["dist"].ReduceOp.MAX)
            dt = float(t.item())
        if i >= warm:
            times.append(dt)
        d2h = 12 * nlev
    print(f"[bench] e2e steps (ms): {[round(t * 1e3, 2) for t in times]}", file=sys.stderr, flush=True)
    return {"s_per_step": float(np.mean(times)), "h2d": h2d, "d2h": d2h, "S": S,
            "median_s": float(np.median(times)), "steps": len(times)}


def secondary_n1(steps, warmup, sm_mhz):
    import torch
    from paper_conf_hpdc_raschg18_b200 import Space
    out = {}
    # C5 with the per-segment |x| bounds (same space; pairs decided without evaluation)
    spec = A.c5_chains(4096, 8)
    res = run_generation(spec, steps, warmup, flags=0)
    ms = float(np.mean(res["ms"]))
    leaves = sum(res["group_sizes"])
    res_t = run_generation(spec, steps, 2, timing=True, serial=True, flags=0)
    rf = roofline_of(res_t, sm_mhz, spec.name + ":segbounds", step_ms=ms)
    out["C5-segment-bounds"] = {
        "ms_per_step": ms, "configs_per_s": leaves / (ms * 1e-3),
        "pairs_decided_per_s": rf["step"]["pairs_decided"] / (ms * 1e-3),
        "pairs_evaluated_per_s": rf["step"]["pairs_evaluated"] / (ms * 1e-3),
        "pairs_evaluated": rf["step"]["pairs_evaluated"], "pairs_decided": rf["step"]["pairs_decided"],
        "roofline_frac_step_on_evaluated_pairs": rf["step"]["frac"], "dominant_launch": rf["launch"],
        "dominant_frac_on_evaluated_pairs": rf["frac"],
        "note": "flags 0: warp-tile hot loop rejects candidate segments by their |x| bounds (DESIGN.md §5)"}
    for name, mk in (("C1", A.c1_toy), ("C3-IS1", lambda: A.c3_xgemm("IS1")), ("C3-IS3", lambda: A.c3_xgemm("IS3"))):
        res = run_generation(mk(), steps, warmup)
        ms = float(np.mean(res["ms"]))
        out[name] = {"ms_per_step": ms, "S": str(res["size"]), "group_leaves": sum(res["group_sizes"]),
                     "configs_per_s": sum(res["group_sizes"]) / (ms * 1e-3),
                     "note": "launch-latency bound (SURVEY.md §8(d)); device time of one generation"}
    for name, mk in (("C3-IS2", lambda: A.c3_xgemm("IS2")), ("C3-IS4", lambda: A.c3_xgemm("IS4")),
                     ("C2", lambda: A.c2_xgemm_direct(256))):
        res = run_generation(mk(), steps, warmup)
        ms = float(np.mean(res["ms"]))
        leaves = sum(res["group_sizes"])
        evals = sum(s["evals"] for s in res["stats"])
        res_t = run_generation(mk(), steps, 2, timing=True, serial=True)
        rf = roofline_of(res_t, sm_mhz, mk().name, step_ms=ms)
        res["level_ms"] = res_t["level_ms"]
        out[name] = {"ms_per_step": ms, "configs_per_s": leaves / (ms * 1e-3), "evals_per_s": evals / (ms * 1e-3),
                     "S": str(res["size"]), "group_leaves": leaves, "evals": evals,
                     "roofline_frac_step": rf["step"]["frac"], "dominant_launch": rf["launch"],
                     "dominant_frac": rf["frac"], "kernel_ms": rf["step"]["ms"],
                     "level_ms": [round(x, 4) for x in np.mean(res["level_ms"], axis=0).tolist()]}
    # P:280's 32x32 experiment: CLTune-style filtering of the full product (SURVEY.md §8(f)
    # NEXT-4; 6.87e10 tuples, the paper's CLTune run was aborted after 3 hours) vs the tree
    spec = A.c2_xgemm_direct(32)
    with Space(spec) as sp:
        sp.filter_product()  # warm-up (upload, module load)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        cnt, tot = sp.filter_product()
        t_filter = time.perf_counter() - t0
        res = run_generation(spec, steps, warmup)
        out["C2-32-full-product-filter"] = {
            "tuples": tot, "valid": cnt, "filter_s": t_filter, "tuples_per_s": tot / t_filter,
            "tree_ms_per_step": float(np.mean(res["ms"])), "tree_S": str(res["size"]),
            "note": "P:280: CLTune-style generation of the 32x32 XgemmDirect space aborted after 3 h (CPU)"}
    # C4: decode 10^8 random indices into C3-IS2
    from atfspec.fuzz import splitmix64_indices
    spec = A.c3_xgemm("IS2")
    with Space(spec) as sp:
        sp.generate()
        S = sp.size()
        n = 100_000_000
        idx = torch.from_numpy(splitmix64_indices(n, S, A.c4_indices_seed()).view(np.int64)).cuda()
        outb = torch.empty((len(spec.params), n), dtype=torch.int32, device="cuda")
        flush = torch.empty(128 << 20, dtype=torch.int32, device="cuda")
        for _ in range(warmup):
            sp.decode(idx, out=outb)
        torch.cuda.synchronize()
        ts = []
        for _ in range(steps):
            flush_l2(flush)
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            sp.decode(idx, out=outb)
            b.record()
            torch.cuda.synchronize()
            ts.append(a.elapsed_time(b))
        ms = float(np.mean(ts))
        io = n * (8 + 4 * len(spec.params))
        out["C4-decode-1e8"] = {"ms": ms, "indices_per_s": n / (ms * 1e-3), "io_GBps": io / (ms * 1e-3) / 1e9,
                                "io_bytes": io}
        del outb, idx
    return out


def predicted_scaling(spec, worlds=(2, 4, 8), reps=3, ag_us=25.0, flag_us=10.0):
    """One-GPU prediction of the balanced multi-GPU generation (atf_space_generate_dist,
    DESIGN.md §6): N virtual ranks (N spaces of this process) run the real per-level protocol
    (same kernels, same partition, parent slices copied between ranks' arenas), one rank at a
    time per level round, so each rank's round runs alone on the GPU.

    "sync": the synchronous protocol (first generations): each rank's round timed on the host
    (launches + device work + sync); T_N = sum over rounds of the slowest rank's round + rounds x
    an all-gather latency (ag_us, an assumption: a < 2 KB NCCL all-gather over NVLink).
    "replay": the steady state (every later generation; no host synchronisation per round, device
    flags between ranks): each rank's round timed on the DEVICE (CUDA events around its kernels,
    CSR fix-ups and peer copies, ATF_FLAG_TIMING); T_N = sum over rounds of the slowest rank's
    device round + exchanged rounds x flag_us (a flag-set + flag-wait over NVLink, assumed) + one
    verdict all-gather (ag_us).  Validated at N = 1: the measured replay time of one rank
    ("replay_measured_1_ms", CUDA events around generate_dist, world 1, steady state).
    efficiency = T_1 / (N T_N) with T_1 from the same procedure.  A prediction, not a scaling
    measurement (no NVLink transfers, no contention between real GPUs)."""
    import torch
    from paper_conf_hpdc_raschg18_b200 import Space, _lib as L
    from paper_conf_hpdc_raschg18_b200.shard import virtual_ranks
    out = {}
    for N in (1,) + tuple(worlds):
        rec = {}
        for mode, extra in (("sync", L.ATF_FLAG_NO_REPLAY), ("replay", L.ATF_FLAG_TIMING)):
            spaces = [Space(spec, flags=headline_flags() | extra) for _ in range(N)]
            try:
                virtual_ranks(spaces)  # warm-up: arenas, JIT, IPC mappings
                best = None
                for _ in range(reps):
                    torch.cuda.synchronize()
                    vag = virtual_ranks(spaces, serialize=True)
                    if mode == "sync":
                        per = [vag.round_s[r] for r in range(N)]
                        rounds = len(per[0])
                        t = sum(max(per[r][i] for r in range(N)) for i in range(rounds)) + (rounds - 1) * ag_us * 1e-6
                    else:
                        per = [[x * 1e-3 for x in sp.dist_round_ms()] for sp in spaces]
                        rounds = len(per[0])
                        ex = vag.calls[0]  # exchanged rounds (one all-gather each)
                        t = sum(max(per[r][i] for r in range(N)) for i in range(rounds)) + \
                            (ex * flag_us + ag_us) * 1e-6
                    if best is None or t < best[0]:
                        best = (t, rounds, [sum(x) for x in per],
                                [round(max(per[r][i] for r in range(N)) * 1e3, 3) for i in range(rounds)])
                rec[mode] = {"T_ms": best[0] * 1e3, "rounds": best[1], "rank_busy_ms": [round(x * 1e3, 3) for x in best[2]],
                             "round_max_ms": best[3]}
            finally:
                for sp in spaces:
                    sp.close()
        out[N] = rec
    # N = 1 steady-state replay, measured (validates the device-time model)
    sp = Space(spec, flags=headline_flags(), stream=torch.cuda.Stream())
    try:
        with torch.cuda.stream(sp._stream_obj):
            for _ in range(3):
                sp.generate_dist(0, 1, lambda b: b)
            ts = []
            for _ in range(reps + 2):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                sp.generate_dist(0, 1, lambda b: b)
                e1.record()
                torch.cuda.synchronize()
                ts.append(e0.elapsed_time(e1))
        measured1 = min(ts)
    finally:
        sp.close()
    res = {"method": predicted_scaling.__doc__.split("\n\n")[0].replace("\n", " "),
           "allgather_us_assumed": ag_us, "flag_us_assumed": flag_us, "replay_measured_1_ms": measured1}
    for mode in ("sync", "replay"):
        t1 = out[1][mode]["T_ms"]
        res[mode] = {str(N): dict(out[N][mode], **({"efficiency": t1 / (N * out[N][mode]["T_ms"])} if N > 1 else {}))
                     for N in out}
    return res


def cpu_baseline(spec, budget_s=15.0):
    from oracle import run as orc
    orc.build()
    cores = os.cpu_count() or 1
    d = orc.time_sample(spec, threads=cores, budget_s=budget_s, timeout=budget_s * 10 + 120)
    return {"value": d["leaves"] / d["seconds"], "unit": "configs/s", "cores": cores, "kind": "oracle",
            "evals_per_s": d["evals"] / d["seconds"],
            "sample": (f"O2 (pruned nested loop, interpreted bytecode) on {spec.name}: groups in order, level-1 "
                       f"values in a strided order (spanning the range) until {budget_s:.0f}s CPU budget; {d['level1_done']}/{d['level1_total']} "
                       f"level-1 values, {d['evals']} evals, {d['leaves']} leaves in {d['seconds']:.2f}s")}


# ------------------------------------------------------------------ main
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-secondary", action="store_true")
    ap.add_argument("--cpu-budget", type=float, default=15.0)
    a = ap.parse_args()
    a.warmup = max(a.warmup, 3)

    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    spec = A.c5_chains(4096, 8)
    config = {"workload": "C5: configs[4] synthetic 24-parameter 3-group chained divisibility, ranges 1..4096",
              "spec": spec.name, "global_batch": 1, "parallelism": f"shard{world}" if world > 1 else "single",
              "l2": "flushed between steps (512 MiB write); outputs ~2 GB > L2"}

    if a.impl == "reference":
        if rank != 0:
            return
        t0 = time.time()
        vals = []
        budget = max(1.0, min(6.0, 60.0 / max(1, a.steps + a.warmup)))
        for i in range(a.warmup + a.steps):
            cb = cpu_baseline(spec, budget_s=budget)
            if i >= a.warmup:
                vals.append(cb)
        v = float(np.mean([c["value"] for c in vals]))
        line = {"impl": "reference", "metric": METRIC, "value": v, "unit": "configs/s", "n_gpus": a.gpus,
                "steps": a.steps, "warmup": a.warmup, "ms_per_step": None, "higher_is_better": True,
                "scaling": "strong", "vs_baseline": None, "dtype": "int64", "data": "synthetic (deterministic spec)",
                "config": config,
                "cpu_baseline": {"value": v, "unit": "configs/s", "cores": vals[0]["cores"], "kind": "oracle",
                                 "sample": vals[0]["sample"]},
                "e2e": {"value": v, "unit": "configs/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
                "wall_s": time.time() - t0}
        print(json.dumps(line), flush=True)
        return

    import torch
    # one process per GPU; ATF_DIST_BACKEND=gloo (ranks may then share a GPU) only exercises the
    # sharded path on a single-GPU box — its timings are not a scaling measurement
    backend = os.environ.get("ATF_DIST_BACKEND", "nccl")
    dev_index = local % max(1, torch.cuda.device_count()) if backend != "nccl" else local
    torch.cuda.set_device(dev_index)
    local = dev_index
    dist_ctx = None
    if world > 1:
        import torch.distributed as dist
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)
        dist_ctx = {"dist": dist, "rank": rank, "world": world,
                    "dev": torch.device("cuda", local) if backend == "nccl" else torch.device("cpu")}

    peaks = _peaks()
    sm_max = float(peaks.get("sm_max_mhz", 1965.0))
    with ClockSampler(local) as clk:
        res = run_generation(spec, a.steps, a.warmup, dist_ctx)
    clocks = clk.summary()
    ms = float(np.mean(res["ms"]))
    if dist_ctx:
        t = torch.tensor([ms], dtype=torch.float64, device=dist_ctx["dev"])
        dist_ctx["dist"].all_reduce(t, op=dist_ctx["dist"].ReduceOp.MAX)
        ms = float(t.item())
    leaves = sum(res["group_sizes"])                      # global (finalize_shard) sizes
    plan = res["plan"]
    value = leaves / (ms * 1e-3)
    # our kernels per step: every non-empty level launches expand_narrow (r <= 64) or
    # expand_wide, then scan_kernel and level_emit_kernel
    n_launch = res["launches"]  # library-counted kernel launches of one generation
    e2e = e2e_generation(spec, max(2, a.steps // 2), dist_ctx)
    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": "configs/s", "n_gpus": world, "steps": a.steps,
                "warmup": a.warmup, "ms_per_step": ms, "higher_is_better": True,
                "scaling": "strong", "vs_baseline": None, "dtype": "int64 (int32 values, 16/32-bit magics)",
                "data": "synthetic (deterministic spec, no dataset)", "config": config,
                "S": str(res["size"]), "group_leaves": res["group_sizes"], "gpu_launches": n_launch * a.steps,
                "clocks": clocks,
                "e2e": {"value": leaves / e2e["s_per_step"], "unit": "configs/s",
                        "h2d_bytes_per_step": e2e["h2d"], "d2h_bytes_per_step": e2e["d2h"],
                        "s_per_step": e2e["s_per_step"], "median_s_per_step": e2e["median_s"],
                        "steps": e2e["steps"], "warmup": 3}}
        if world == 1:
            evals_total = sum(s["evals"] for s in res["stats"])
            # every pair evaluated (headline flags): evaluated = decided = f_{k-1} r_k
            line["pairs_decided_per_s"] = evals_total / (ms * 1e-3)
            line["flags"] = "ATF_FLAG_NO_SEG_BOUNDS (every f_{k-1} r_k pair evaluated)"
            # roofline: a serialized timing pass of the same generation (per-launch events)
            res_t = run_generation(spec, max(3, a.steps // 2), 2, timing=True, serial=True)
            line["roofline"] = roofline_of(res_t, sm_max, spec.name, step_ms=ms)
            # evaluated pairs counted on the device (ATF_FLAG_TIMING statistics of the timing pass)
            line["pairs_evaluated_per_s"] = line["roofline"]["step"]["pairs_evaluated"] / (ms * 1e-3)
            line["roofline"]["timing_pass"] = ("serialized groups, CUDA events per level / expand kernel, "
                                               f"{max(3, a.steps // 2)} steps after the timed region")
            line["roofline_at_load_clock"] = (roofline_of(res_t, clocks["sm_mhz"], spec.name, step_ms=ms)["frac"]
                                              if clocks.get("sm_mhz") else None)

            try:
                line["cpu_baseline"] = cpu_baseline(spec, budget_s=a.cpu_budget)
            except Exception as ex:  # noqa: BLE001
                line["cpu_baseline"] = {"error": str(ex)}
            try:
                line["predicted_scaling"] = predicted_scaling(spec)
            except Exception as ex:  # noqa: BLE001
                line["predicted_scaling"] = {"error": str(ex)}
            if not a.no_secondary:
                line["secondary"] = secondary_n1(max(3, a.steps // 2), 3, sm_max)
        print(json.dumps(line), flush=True)
    if dist_ctx:
        dist_ctx["dist"].barrier()
        dist_ctx["dist"].destroy_process_group()


if __name__ == "__main__":
    main()
