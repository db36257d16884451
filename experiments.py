"""Paper experiments re-run on B200 (bench.py --sweep / --kbe).

config 2 (tile sweep, §5.2 Figs 12-13, Eq 10): the fused kernel's
  measured time T(Δ) for Δ = 2^9..2^22 rows next to the A9 model's estimate
  for the same Δ; reports Eq 10 relative error |T_meas - T_est| / T_meas per
  point and the model's argmin vs the measured argmin. Results must be
  identical at every Δ (checked).
config 5 (fused vs KBE, §2.2 Obs 1 / §5.3.2 Figs 3, 16-18): Q14 with shipdate
  windows giving ~1-100% selectivity, Q5 and Q9-wide at SF 10: kernel/step
  latency of the fused pipeline, of the kernel-at-a-time materialising
  baseline (KBE) and of GPL (w/o CE) (KBE kernels run tile by tile, Fig 16),
  and the intermediate bytes materialised, normalised to input.

Both print one JSON line and write the full table to --out.
"""
from __future__ import annotations

import json
import math
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)


def _setup(q, sf, seed, tables=None):
    import numpy as np  # noqa: F401
    import torch

    import tpchgen
    from paper_conf_sigmod_paulhh16_b200 import gpl, queries
    dev = torch.device("cuda", 0)
    torch.cuda.set_stream(torch.cuda.Stream(device=dev))  # a real stream shared with libgpl
    stream = torch.cuda.current_stream()
    db = tpchgen.generate(sf, seed=seed, tables=tables or sorted(set(queries.TABLES[q]) | {"region", "nation"}))

    class D:
        pass
    ddb = D()
    ddb.tables = {t: {c: torch.from_numpy(a).to(dev) for c, a in cols.items()} for t, cols in db.tables.items()}
    ctx = gpl.Context(0, stream=stream)
    queries.load_database(ctx, ddb)
    flush = torch.empty(2 * torch.cuda.get_device_properties(dev).L2_cache_size, dtype=torch.uint8, device=dev)
    return db, ctx, flush, stream


def tile_sweep(q="Q5", sf=1.0, seed=20160626, reps=5, out=None, calibration=None, setup=None):
    import torch

    from paper_conf_sigmod_paulhh16_b200 import queries
    db, ctx, flush, stream = setup or _setup(q, sf, seed)
    if calibration is not None:
        ctx.set_calibration(calibration)  # Γ points ([] = the uncalibrated model)
    segs = queries.segments(queries.plan_text(q, db))
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)

    def measure(tile):
        ts, r = [], None
        for i in range(reps + 2):
            for s in segs[:-1]:
                ctx.build_hash(s)
            flush.zero_()
            ctx.run_plan(segs[-1], tile)
            r = ctx.fetch_result()
            if i >= 2:
                ts.append(r.stats["kernel_ms"])
        return statistics.median(ts), r

    t_auto, r_auto = measure(0)
    ref = (r_auto.keys, r_auto.aggs)
    rows = []
    for e in range(9, 23):
        tile = 1 << e
        t, r = measure(tile)
        assert (r.keys, r.aggs) == ref, "result changed with tile_rows"
        est = r.stats["predicted_ms"]
        rows.append({"tile_rows": r.stats["tile_rows_used"], "tile_bytes": r.stats["tile_rows_used"] * r.stats["bytes_scanned"] / max(1, r.stats["rows_scanned"]),
                     "measured_ms": t, "predicted_ms": est, "rel_error": abs(t - est) / t,
                     "stage_rows": r.stats["stage_rows"], "ring_depth": r.stats["ring_depth"],
                     "consumer_warps": r.stats["consumer_warps"]})
    best_meas = min(rows, key=lambda x: x["measured_ms"])
    best_pred = min(rows, key=lambda x: (x["predicted_ms"], -x["tile_rows"]))
    summary = {"experiment": "tile_sweep (config 2)", "query": q, "sf": sf,
               "gamma_calibrated": bool(calibration),
               "auto": {"tile_rows": r_auto.stats["tile_rows_used"], "measured_ms": t_auto,
                        "predicted_ms": r_auto.stats["predicted_ms"]},
               "measured_argmin_tile_rows": best_meas["tile_rows"], "measured_min_ms": best_meas["measured_ms"],
               "model_argmin_tile_rows": best_pred["tile_rows"],
               "model_pick_vs_best": t_auto / best_meas["measured_ms"],
               "mean_rel_error": statistics.mean(x["rel_error"] for x in rows),
               "results_identical_across_tiles": True, "points": rows}
    if out:
        with open(out, "w") as f:
            json.dump(summary, f, indent=1)
    return summary


def gamma_calibration(q="Q5", sfs=(1.0, 10.0), seed=20160626, out=None):
    """NEXT-1: the channel calibration Γ(n, s, k, d) (§2.1, Eq 1, Fig 2 / Fig 23 analog:
    ring throughput vs data size for each ring depth n and stage size s), then the config-2 tile sweep of
    `q` at each SF with the uncalibrated and the Γ-calibrated model: Eq 10 relative error and the model
    pick's gap to the measured best, both ways (the paper's Figs 11-13 / 24-26 check of its model)."""
    setup = _setup(q, sfs[0], seed)
    ctx = setup[1]
    pts = ctx.calibrate()
    curves = {}
    for p in pts:
        curves.setdefault(f"n={p['ring_depth']} s={p['stage_rows']} k={p['ctas_per_sm']}", []).append(
            {"rows": p["rows"], "MB": p["bytes"] / 1e6, "ms": p["ms"], "gbs": p["gbs"], "t0_us": 1e3 * p["t0_ms"]})
    peak = max(p["gbs"] for p in pts)
    best_shape = max(curves, key=lambda k: curves[k][-1]["gbs"])
    sweeps = []
    for i, sf in enumerate(sfs):
        st = setup if i == 0 else _setup(q, sf, seed)
        if i > 0:
            st[1].set_calibration(pts)
        for cal in ([], pts):
            s = tile_sweep(q, sf, seed, calibration=cal, setup=st)
            sweeps.append({k: s[k] for k in ("query", "sf", "gamma_calibrated", "mean_rel_error", "model_pick_vs_best",
                                              "measured_argmin_tile_rows", "model_argmin_tile_rows", "auto")})
            sweeps[-1]["points"] = [{k: x[k] for k in ("tile_rows", "measured_ms", "predicted_ms", "rel_error")}
                                    for x in s["points"]]
    summary = {"experiment": "gamma calibration (NEXT-1; Fig 2/23 + Eq 10 analog)",
               "gamma_peak_gbs": peak, "best_shape_at_largest_d": best_shape,
               "curves": curves, "sweeps": sweeps}
    if out:
        with open(out, "w") as f:
            json.dump(summary, f, indent=1)
    return summary


def warp_sweep(q="Q8", sf=10.0, seed=20160626, reps=5, out=None):
    """Figs 14-15 analog: the work-group setting S_i ↦ consumer warps per CTA W (2..16), other knobs
    from the model; measured kernel time vs the model's estimate (Eq 10 error) and the model's delay term
    (t_tail: the Eq 8 imbalance between producer and consumers plus the last wave), results identical."""
    from paper_conf_sigmod_paulhh16_b200 import queries
    db, ctx, flush, stream = _setup(q, sf, seed)
    segs = queries.segments(queries.plan_text(q, db))
    rows, ref = [], None
    for w in (2, 4, 6, 8, 12, 16):
        ctx.set_option("consumer_warps", w)
        ts, r = [], None
        try:
            for i in range(reps + 2):
                for s in segs[:-1]:
                    ctx.build_hash(s)
                flush.zero_()
                ctx.run_plan(segs[-1])
                r = ctx.fetch_result()
                if i >= 2:
                    ts.append(r.stats["kernel_ms"])
        except Exception as e:  # a shape that does not fit
            rows.append({"consumer_warps": w, "error": str(e)})
            continue
        if ref is None:
            ref = (r.keys, r.aggs)
        assert (r.keys, r.aggs) == ref, "result changed with consumer warps"
        m = ctx.choose_tile_rows(segs[-1], 0)
        t = statistics.median(ts)
        rows.append({"consumer_warps": w, "measured_ms": t, "predicted_ms": r.stats["predicted_ms"],
                     "rel_error": abs(t - r.stats["predicted_ms"]) / t, "model_delay_tail_ms": m["t_tail_ms"],
                     "stage_rows": r.stats["stage_rows"], "ring_depth": r.stats["ring_depth"],
                     "tile_rows": r.stats["tile_rows_used"]})
    ctx.set_option("consumer_warps", -1)
    ok = [x for x in rows if "measured_ms" in x]
    best_meas = min(ok, key=lambda x: x["measured_ms"])
    best_pred = min(ok, key=lambda x: x["predicted_ms"])
    summary = {"experiment": "consumer-warp sweep (Figs 14-15 analog)", "query": q, "sf": sf,
               "measured_argmin_warps": best_meas["consumer_warps"], "model_argmin_warps": best_pred["consumer_warps"],
               "model_pick_vs_best": best_pred["measured_ms"] / best_meas["measured_ms"],
               "mean_rel_error": statistics.mean(x["rel_error"] for x in ok), "results_identical": True,
               "points": rows}
    if out:
        with open(out, "w") as f:
            json.dump(summary, f, indent=1)
    return summary


def kbe_compare(sf=10.0, seed=20160626, reps=3, out=None):
    import numpy as np
    import torch

    import tpchgen
    from paper_conf_sigmod_paulhh16_b200 import queries
    tables = ["part", "partsupp", "supplier", "customer", "orders", "lineitem", "nation", "region"]
    db, ctx, flush, stream = _setup("Q9", sf, seed, tables)
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    sd = np.sort(db.tables["lineitem"]["l_shipdate"][:: max(1, db.nrows("lineitem") // 200000)])
    cases = []
    for pct in (1, 5, 10, 25, 50, 75, 100):  # Q14 selectivity sweep (Fig 3/18)
        lo = 19920101
        hi = 19990101 if pct == 100 else int(sd[min(len(sd) - 1, int(len(sd) * pct / 100))])
        cases.append((f"Q14 sel~{pct}%", "Q14", (lo, hi)))
    cases.append(("Q5", "Q5", None))
    n_part = tpchgen.sizes(sf)["part"]
    cases.append(("Q9-wide", "Q9", (math.ceil(0.054 * n_part),)))  # reading R5: ~%green% share
    rows = []
    for name, q, params in cases:
        segs = queries.segments(queries.plan_text(q, db, params))

        def timed(kbe, kbe_tile=0):
            ctx.set_option("kbe_tile_rows", kbe_tile)
            ts, r = [], None
            warm = 1 if kbe else 6  # fused: λ profile + the profiled runs re-plan (and JIT-compile) first
            for i in range(reps + warm):
                for s in segs[:-1]:
                    ctx.build_hash(s)
                flush.zero_()
                ev0.record(stream)
                if kbe:
                    ctx.run_plan_kbe(segs[-1])
                else:
                    ctx.run_plan(segs[-1])
                ev1.record(stream)
                r = ctx.fetch_result()
                if i >= warm:
                    ts.append(ev0.elapsed_time(ev1))
            ctx.set_option("kbe_tile_rows", 0)
            return statistics.median(ts), r
        tf, rf = timed(False)
        tk, rk = timed(True)
        # GPL (w/o CE): the KBE kernels tile by tile, with the
        # paper's default 1 MB tile in rows of this query's scan width
        bpr = max(1, int(rf.stats["bytes_scanned"] / max(1, rf.stats["rows_scanned"])))
        tw, rw = timed(True, (1 << 20) // bpr)
        # ... and with the paper's largest swept tile, 16 MB: fewer, larger tiles
        tw16, rw16 = timed(True, (16 << 20) // bpr)
        # the same 1 MB / 16 MB tile loops launched kernel by kernel instead of replayed as one graph
        ctx.set_option("kbe_graph", 0)
        tl, _ = timed(True, (1 << 20) // bpr)
        tl16, _ = timed(True, (16 << 20) // bpr)
        ctx.set_option("kbe_graph", 1)
        assert (rf.keys, rf.aggs) == (rk.keys, rk.aggs) == (rw.keys, rw.aggs) == (rw16.keys, rw16.aggs), name
        inp = rf.stats.get("bytes_full_scan") or rf.stats["bytes_scanned"]  # the input: every column read, once
        ops = rf.stats["op_pass"]
        sel = (ops[0] / rf.stats["rows_scanned"]) if q == "Q14" and ops else None
        rows.append({"case": name, "selectivity": sel, "input_bytes": inp,
                     "fused_ms": tf, "kbe_ms": tk, "speedup": tk / tf,
                     "wo_ce_ms": tw, "wo_ce_tile_rows": rw.stats["tile_rows_used"],
                     "wo_ce_over_kbe": tw / tk, "wo_ce_intermediate_bytes": rw.stats["intermediate_bytes"],
                     "wo_ce_16mb_ms": tw16, "wo_ce_16mb_tile_rows": rw16.stats["tile_rows_used"],
                     "wo_ce_16mb_over_kbe": tw16 / tk,
                     "wo_ce_launched_ms": tl, "wo_ce_16mb_launched_ms": tl16,
                     "fused_moved_bytes": rf.stats["bytes_scanned"], "fused_lazy_columns": rf.stats.get("lazy_columns"),
                     "fused_intermediate_bytes": rf.stats["intermediate_bytes"],
                     "kbe_intermediate_bytes": rk.stats["intermediate_bytes"],
                     "kbe_intermediate_over_input": rk.stats["intermediate_bytes"] / inp,
                     "fused_kernel_ms": rf.stats["kernel_ms"]})
    summary = {"experiment": "fused vs KBE (config 5)", "sf": sf, "points": rows,
               "paper_context": "AMD A10: KBE intermediates 1.38x input at 100% Q14 selectivity vs 0.22x for GPL "
                                "(P:402); GPL up to 48% faster than KBE (P:384)"}
    if out:
        with open(out, "w") as f:
            json.dump(summary, f, indent=1)
    return summary


def knob_sweep(q="Q5", sf=1.0, seed=20160626, reps=3, out=None, setup=None):
    """Config 2 over the channel knobs (PAPER.md Figs 12-13; Eq 10): stage rows s in
    {512, 1024, 2048} (the packet analog), ring depth n in {2, 3, 4} (the number of channels) and
    Δ = 2^9 .. 2^22 rows (at least one stage), every other knob from the A9 model. Measured kernel time
    vs the model's estimate for the same configuration (Eq 10 relative error), the model's argmin vs the
    measured argmin, and bit-identical results at every point."""
    from paper_conf_sigmod_paulhh16_b200 import queries
    db, ctx, flush, stream = setup or _setup(q, sf, seed)
    segs = queries.segments(queries.plan_text(q, db))
    for _ in range(4):  # λ profile + the model's profiling input (the paper profiles the first tile)
        ctx.run_query(queries.plan_text(q, db))
        ctx.fetch_result()
    rows, ref = [], None
    try:
        for S in (512, 1024, 2048):
            for n in (2, 3, 4):
                ctx.set_option("stage_rows", S)
                ctx.set_option("ring_depth", n)
                for e in range(9, 23):
                    tile = 1 << e
                    if tile < S:
                        continue
                    ts, r = [], None
                    for i in range(reps + 1):
                        for sg in segs[:-1]:
                            ctx.build_hash(sg)
                        flush.zero_()
                        ctx.run_plan(segs[-1], tile)
                        r = ctx.fetch_result()
                        if i >= 1:
                            ts.append(r.stats["kernel_ms"])
                    if ref is None:
                        ref = (r.keys, r.aggs)
                    assert (r.keys, r.aggs) == ref, "result changed with the knobs"
                    t = statistics.median(ts)
                    est = r.stats["predicted_ms"]
                    rows.append({"stage_rows": S, "ring_depth": n, "tile_rows": r.stats["tile_rows_used"],
                                 "consumer_warps": r.stats["consumer_warps"], "measured_ms": t, "predicted_ms": est,
                                 "rel_error": abs(t - est) / t})
    finally:
        ctx.set_option("stage_rows", -1)
        ctx.set_option("ring_depth", -1)
    best_meas = min(rows, key=lambda x: x["measured_ms"])
    best_pred = min(rows, key=lambda x: (x["predicted_ms"], -x["tile_rows"]))
    summary = {"experiment": "knob sweep (config 2: s x n x Δ)", "query": q, "sf": sf, "points_measured": len(rows),
               "mean_rel_error": statistics.mean(x["rel_error"] for x in rows),
               "median_rel_error": statistics.median(x["rel_error"] for x in rows),
               "measured_best": best_meas, "model_pick": best_pred,
               "model_pick_vs_best": best_pred["measured_ms"] / best_meas["measured_ms"],
               "results_identical": True, "points": rows}
    if out:
        with open(out, "w") as f:
            json.dump(summary, f, indent=1)
    return summary


def model_vs_autotune(qs=("Q5", "Q7", "Q8", "Q9", "Q14", "Q3"), sf=100.0, seed=20160626, reps=5, out=None):
    """A9 without autotune (config 4): the shape the re-derived model picks on its own (after the
    λ profile and the profiled run) vs the shape gpl_autotune measures best; kernel times
    (median of reps, L2 flushed), the model's Eq 10 error for its own pick, identical results."""
    from paper_conf_sigmod_paulhh16_b200 import queries
    tables = sorted({t for q in qs for t in queries.TABLES[q]} | {"region", "nation"})
    db, ctx, flush, stream = _setup(qs[0], sf, seed, tables)
    rows = []
    for q in qs:
        text = queries.plan_text(q, db)

        def timed():
            ts, r = [], None
            for i in range(reps + 1):
                flush.zero_()
                ctx.run_query(text)
                r = ctx.fetch_result()
                if i >= 1:
                    ts.append(r.stats["kernel_ms"])
            return statistics.median(ts), r
        for _ in range(6):  # λ, then the profiled runs; the model re-plans with its fitted costs
            ctx.run_query(text)
            ctx.fetch_result()
        tm, rm = timed()
        m = ctx.autotune(text)
        ta, ra = timed()
        assert (rm.keys, rm.aggs) == (ra.keys, ra.aggs), q
        shape = lambda r: {k: r.stats[k] for k in ("stage_rows", "ring_depth", "consumer_warps", "grid",  # noqa: E731
                                                    "tile_rows_used", "probe_split", "packets")}
        rows.append({"query": q, "model_ms": tm, "model_predicted_ms": rm.stats["predicted_ms"],
                     "model_rel_error": abs(tm - rm.stats["predicted_ms"]) / tm, "autotune_ms": ta,
                     "model_over_autotune": tm / ta, "candidates_measured": m["candidates"],
                     "model_shape": shape(rm), "autotune_shape": shape(ra)})
        ctx.set_option("stage_rows", -1)  # un-pin for the next query
    summary = {"experiment": "A9 model pick vs autotune (config 4)", "sf": sf, "points": rows,
               "max_model_over_autotune": max(x["model_over_autotune"] for x in rows),
               "mean_model_rel_error": statistics.mean(x["model_rel_error"] for x in rows)}
    if out:
        with open(out, "w") as f:
            json.dump(summary, f, indent=1)
    return summary


if __name__ == "__main__":
    which = sys.argv[1] if len(sys.argv) > 1 else "sweep"
    if which == "sweep":
        s = tile_sweep(out=os.path.join(ROOT, "gpurun_out", "sweep_config2.json"))
    elif which == "gamma":
        s = gamma_calibration(out=os.path.join(ROOT, "gpurun_out", "gamma_calibration.json"))
        s.pop("curves", None)
        for x in s["sweeps"]:
            x.pop("points", None)
    elif which == "warps":
        s = warp_sweep(out=os.path.join(ROOT, "gpurun_out", "warp_sweep.json"))
    elif which == "knobs":
        s = knob_sweep(out=os.path.join(ROOT, "gpurun_out", "knob_sweep_config2.json"))
    elif which == "model":
        s = model_vs_autotune(out=os.path.join(ROOT, "gpurun_out", "model_vs_autotune_sf100.json"))
    else:
        s = kbe_compare(out=os.path.join(ROOT, "gpurun_out", "kbe_config5.json"))
    s.pop("points", None)
    print(json.dumps(s))
