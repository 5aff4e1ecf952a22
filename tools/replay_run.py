"""configs[4]: trace replay on Llama-3-8B shapes driving the QoServe scheduler.

  python tools/replay_run.py --mode engine --dataset azure_conv --qps 10,20,30 --duration 60
  python tools/replay_run.py --mode model  --dataset azure_code --qps 5,10,20,30,40 --duration 1800
  python tools/replay_run.py --mode model  --dataset azure_conv --qps 80,160,240 --replicas 8

engine: every step is a real device-timed qos_hybrid_step (virtual clock += measured ms); the
        scheduler's latency model is fitted to a quick qos_profile_step sweep of this engine.
model:  steps are priced by the latency model committed in profiles/latency_table_r2d.json
        (fitted to the B200 profile) — fast what-if replays over long horizons.
Prints one JSON line per QPS and a summary with goodput = max QPS with <= 1% violations
(PAPER.md:1152-1155).
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import synth  # noqa: E402
from paper_conf_asplos_goelmkar26_b200.latency_model import LatencyModel, StepShape  # noqa: E402
from paper_conf_asplos_goelmkar26_b200.replay import EngineExecutor, ModelExecutor, replay, replay_replicas  # noqa: E402
from paper_conf_asplos_goelmkar26_b200.scheduler import QoServeScheduler, SchedulerConfig  # noqa: E402

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--mode", default="engine", choices=["engine", "model"])
    ap.add_argument("--dataset", default="azure_conv")
    ap.add_argument("--qps", default="10,20,30")
    ap.add_argument("--duration", type=float, default=60.0)
    ap.add_argument("--alpha", type=float, default=8.0)
    ap.add_argument("--max-chunk", type=int, default=4096)
    ap.add_argument("--out", default=None)
    ap.add_argument("--replicas", type=int, default=1,
                    help="round-robin TP1 replicas (1 per GPU); engine mode replays them one after another")
    ap.add_argument("--policy", default="slack", choices=["slack", "medha"],
                    help="chunk sizing: QoServe's slack-based dynamic chunking or Medha-style fixed-target")
    ap.add_argument("--medha-target-ms", type=float, default=50.0)
    ap.add_argument("--only-dc", action="store_true",
                    help="the paper's Medha-comparison ablation: FCFS order, no relegation, no selective "
                         "preemption (PAPER.md:1645-1649)")
    ap.add_argument("--max-seq", type=int, default=8192, help="engine max_seq_len (long_10k needs 10500)")
    ap.add_argument("--max-decodes", type=int, default=256,
                    help="decode-set bound (long_10k: 90, so the running requests' KV fits the pool)")
    a = ap.parse_args()
    results = []
    eng = None
    if a.mode == "engine":
        import torch
        from paper_conf_asplos_goelmkar26_b200 import qoserve as q
        from paper_conf_asplos_goelmkar26_b200.presets import preset
        torch.cuda.set_device(0)
        cfg = q.model_cfg(**preset("llama3-8b"), num_blocks=int(140e9 / (32 * 2 * 8 * 128 * 2 * 16)),
                          max_seq_len=a.max_seq, max_requests=4096, max_batch_tokens=a.max_chunk + 512,
                          max_batch_rows=257)
        eng = q.Engine(cfg)
        eng.qos_engine_load_synthetic(0)
        shapes, ms = [], []
        eng.qos_profile_step(2048, [2048] * 64, reps=5, warmup=5)
        # the grid varies every feature the model separates: chunk length, the chunk's cached
        # prefix (kv_start), decode count and decode context (KV bytes), so neither the prefix
        # coefficient nor the per-KV-byte coefficient is left unidentified
        for c in (0, 256, 512, 1024, 2048, 3072, 4096):
            for nd in (0, 16, 64, 128, 256):
                long = ((10000, 0), (4096, 6144)) if a.max_seq > 10500 else ()
                for ctx, ks in ((512, 0), (2048, 2048), (6144, 0), (1536, 4096)) + long:
                    if ((c == 0 and nd == 0) or c > a.max_chunk or (c == 0 and ks) or nd * (ctx + 1) > 1_000_000
                            or ks + c > a.max_seq or ctx + 1 > a.max_seq):
                        continue
                    t, _ = eng.qos_profile_step(c, [ctx] * nd, reps=3, warmup=2, kv_start=ks)
                    shapes.append(StepShape([(ks, c)] if c else [], [ctx] * nd))
                    ms.append(t)
        model = LatencyModel().fit(shapes, ms)
    else:
        prof = json.load(open(os.path.join(ROOT, "profiles", "latency_table_r2d.json")))
        model = LatencyModel.from_json(json.dumps(prof["model_json"]))

    def pred(chunks, ctx):
        return model.predict(StepShape(list(chunks), list(ctx)))

    for qps in [float(x) for x in a.qps.split(",")]:
        tr = synth.trace(qps, a.duration, a.dataset)

        def mk_sched():
            return QoServeScheduler(SchedulerConfig(alpha_ms_per_token=a.alpha, max_chunk=a.max_chunk,
                                                    max_decodes=a.max_decodes, max_rows=257,
                                                    max_tokens=a.max_chunk + 512, chunk_policy=a.policy,
                                                    medha_target_ms=a.medha_target_ms, fcfs=a.only_dc,
                                                    relegation=not a.only_dc, preemption=not a.only_dc), pred)
        if a.mode == "engine" and a.replicas > 1:
            # round-robin replicas replayed one after another on the one GPU (replicas share
            # nothing; each runs its share of the trace on its own virtual clock)
            out = replay_replicas(tr, a.replicas, mk_sched,
                                  lambda: EngineExecutor(eng, 128256,
                                                         lambda r, s, n: synth.request_tokens(r, n, 128256, start=s)))
        elif a.mode == "engine":
            ex = EngineExecutor(eng, 128256, lambda r, s, n: synth.request_tokens(r, n, 128256, start=s))
            out = replay(tr, mk_sched(), ex)
        elif a.replicas > 1:
            out = replay_replicas(tr, a.replicas, mk_sched, lambda: ModelExecutor(pred))
        else:
            out = replay(tr, mk_sched(), ModelExecutor(pred))
        out.update({"qps": qps, "dataset": a.dataset, "mode": a.mode, "duration_s": a.duration, "alpha": a.alpha,
                    "replicas": a.replicas, "policy": a.policy, "only_dc": a.only_dc})
        series = out.pop("chunk_series", None)
        print(json.dumps(out), flush=True)
        out["chunk_series"] = series
        results.append(out)
    ok = [r["qps"] for r in results if r["violations_pct"] <= 1.0]
    summary = {"goodput_qps": max(ok) if ok else 0.0, "dataset": a.dataset, "mode": a.mode,
               "replicas": a.replicas, "qps_tested": [r["qps"] for r in results], "policy": a.policy,
               "only_dc": a.only_dc}
    print(json.dumps(summary), flush=True)
    if a.out:
        json.dump({"summary": summary, "runs": results}, open(a.out, "w"), indent=1)
    if eng is not None:
        eng.close()


if __name__ == "__main__":
    main()
