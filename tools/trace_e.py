#!/usr/bin/env python
"""Config E (BASELINE.json configs[4]): three-model hot-swap trace, replayed on one B200.

Engines: Llama-3.1-8B (TP=1, logical GPU 0), DS-R1-Distill-Qwen-14B (TP=1, logical GPU 1) and
Qwen2.5-32B (TP=2, logical GPUs 0+1) — one GPU pair of SURVEY.md §8(d) E. Each engine's shards
live in VMM arenas (real HBM release on swap-out) on the one physical device; the scheduler
enforces a per-logical-GPU budget so the 32B engine conflicts with both others while 8B and 14B
co-reside. Arrivals: workloads.trace_e (diurnal sinusoid x on/off bursts, shares 50/30/20 %,
lognormal service mean 2 s). Swaps are real (checkpoint + release, re-acquire + restore + HBM
verify, all through libswap); service is simulated on a virtual clock that the measured swap
times advance. Prints one JSON summary.

    python tools/trace_e.py --duration 600 --seed 0
"""
import argparse
import json
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import workloads as W  # noqa: E402
from paper_conf_sc_stoyanovsracb25_b200.hotswap import Engine, HotSwapController, Shard  # noqa: E402
from paper_conf_sc_stoyanovsracb25_b200.swap import Arena, Swapper  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--duration", type=float, default=600.0, help="trace seconds (one 'day' = 600 s)")
ap.add_argument("--seed", type=int, default=0)
ap.add_argument("--rate", type=float, default=0.25, help="base arrivals per second")
ap.add_argument("--kv-tokens", type=int, default=1 << 16)
ap.add_argument("--budget-gb", type=float, default=60.0, help="per logical GPU")
ap.add_argument("--mechanism", default="auto")
ap.add_argument("--duplex", action="store_true", help="overlap swap-out and swap-in (swap_exchange)")
ap.add_argument("--out", default=None)
args = ap.parse_args()

torch.cuda.set_device(0)
stream = torch.cuda.Stream()
LAYOUT = [("8b", [0]), ("14b", [1]), ("32b", [0, 1])]
engines = []
t0 = time.perf_counter()
with torch.cuda.stream(stream):
    for bid, (model, gpus) in enumerate(LAYOUT):
        e = Engine(bid, model)
        for rank, g in enumerate(gpus):
            specs = W.engine_e(model, rank, args.kv_tokens)
            offs, total = W.place(specs)
            arena = Arena(total)
            base, view = arena.alloc(total)
            W.fill_device_arena(view, specs, offs, seed=100 * bid + rank)
            regions = [(base + o, r.nbytes, r.kind, i) for i, (r, o) in enumerate(zip(specs, offs))]
            sw = Swapper(regions, mechanism=args.mechanism, device=0, rank=rank, world=len(gpus))
            sw.bind_arena(arena)  # restore re-acquires HBM group by group, overlapped with the copies
            # snapshot right after initialisation, then park the engine
            sw.swap_out(arena, stream)
            e.shards.append(Shard(g, arena, sw, sum(r.nbytes for r in specs)))
        engines.append(e)
t_setup = time.perf_counter() - t0
ctl = HotSwapController(engines, [int(args.budget_gb * 1e9)] * 2, stream, duplex=args.duplex,
                        stream_in=torch.cuda.Stream() if args.duplex else None)

trace = W.trace_e(args.seed, args.duration, rate_per_s=args.rate)
names = {e.name: e.bid for e in engines}
busy_until = {e.bid: 0.0 for e in engines}
last_access = {e.bid: 0.0 for e in engines}
inflight = {e.bid: [] for e in engines}  # (arrival, end)
vt = 0.0
lat, swapin, hits, req_lat, swaptotal = [], [], 0, [], []
wall0 = time.perf_counter()
with torch.cuda.stream(stream):
    for (t, model, svc) in trace:
        bid = names[model]
        vt = max(vt, t)
        for b in inflight:  # queue length seen by the policy: requests not finished at vt
            inflight[b] = [(a, z) for (a, z) in inflight[b] if z > vt]
            ctl.touch(b, len(inflight[b]), last_access[b])
        victims_busy = 0.0
        if not ctl.resident(bid):
            plan = ctl.sched.plan(bid) or []
            victims_busy = max([busy_until[v] for v in plan], default=0.0)  # in-flight work drains first
        hit, victims, t_out, t_in = ctl.ensure_resident(bid, priority=t)
        if hit:
            hits += 1
            ready = t
        else:
            vt = max(vt, victims_busy) + t_out + t_in
            ready = vt
            swapin.append((model, t_in, engines[bid].payload))
            swaptotal.append(t_out + t_in)
        start = max(ready, busy_until[bid])
        end = start + svc
        busy_until[bid] = end
        inflight[bid].append((t, end))
        last_access[bid] = t
        req_lat.append(end - t)
wall = time.perf_counter() - wall0


def pct(xs, p):
    xs = sorted(xs)
    return xs[min(len(xs) - 1, int(round(p / 100 * (len(xs) - 1))))] if xs else None


per_model = {}
for m in names:
    ts = [x[1] for x in swapin if x[0] == m]
    if ts:
        payload = engines[names[m]].payload
        per_model[m] = {"swap_ins": len(ts), "payload_GB": round(payload / 1e9, 2),
                        "latency_s_p50": round(pct(ts, 50), 4), "latency_s_p99": round(pct(ts, 99), 4),
                        "GBps_mean": round(statistics.mean(payload / x for x in ts) / 1e9, 2)}
outs = [x for x in ctl.log if x[0] == "out"]
virtual_h = max(vt, trace[-1][0] if trace else 0) / 3600
rec = {
    "workload": "E: three-model hot-swap trace (8B / 14B / 32B TP=2) on one GPU pair, replayed on one B200",
    "requests": len(trace), "hit_rate": round(hits / max(1, len(trace)), 4),
    "swap_ins": len(swapin), "swap_outs": len(outs),
    "swap_in_latency_s": {"p50": pct([x[1] for x in swapin], 50), "p99": pct([x[1] for x in swapin], 99)},
    "swap_in_GBps_mean": round(statistics.mean(x[2] / x[1] for x in swapin) / 1e9, 2) if swapin else None,
    "swap_out_GBps_mean": round(statistics.mean(x[3] / x[2] for x in outs) / 1e9, 2) if outs else None,
    "swaps_per_hour": round((len(swapin) + len(outs)) / virtual_h, 1) if virtual_h else None,
    "request_latency_s": {"p50": round(pct(req_lat, 50), 3), "p99": round(pct(req_lat, 99), 3)},
    "swap_time_s": {"p50": pct(swaptotal, 50), "p99": pct(swaptotal, 99), "mean": round(statistics.mean(swaptotal), 4)
                    if swaptotal else None,
                    "what": "request-visible swap time: victims out + requested engine in (+ HBM verify)"},
    "per_model": per_model,
    "config": {"duration_s": args.duration, "seed": args.seed, "rate_per_s": args.rate,
               "kv_tokens": args.kv_tokens, "budget_GB_per_logical_gpu": args.budget_gb,
               "mechanism": args.mechanism, "duplex": args.duplex},
    "wall_s": round(wall, 1), "setup_s": round(t_setup, 1), "virtual_s": round(vt, 1),
}
s = json.dumps(rec)
print(s, flush=True)
if args.out:
    with open(args.out, "w") as f:
        f.write(s + "\n")
ctl.close()
