"""End-to-end: the QoServe scheduler drives the CUDA engine and the fp64 oracle in lockstep over
a synthetic trace (tiny config).  Every step's logits must agree within 1e-2 and the greedy
tokens wherever the oracle's top-2 gap exceeds the tolerance; the oracle's tokens are fed back
to both so the trajectories stay identical.  Also a short replay on Llama-3-8B shapes driven
by real device-timed steps."""
import numpy as np
import pytest

import synth
from helpers import TOL_LOGITS, make_engine, row_rel_err
from paper_conf_asplos_goelmkar26_b200.replay import replay
from paper_conf_asplos_goelmkar26_b200.scheduler import QoServeScheduler, SchedulerConfig

pytestmark = pytest.mark.gpu


def lin_model(chunks, ctx):
    T = sum(n for _, n in chunks) + len(ctx)
    return 2.0 + 0.01 * T


class Lockstep:
    def __init__(self, q, eng, orc, vocab):
        self.q, self.eng, self.orc, self.vocab = q, eng, orc, vocab
        self.next_tok, self.steps, self.max_err, self.known = {}, 0, 0.0, set()

    def admit(self, chunks, decodes):
        for r, n in chunks:
            self.eng.qos_kv_alloc(r.req_id, r.prefill_done + n)
            self.orc.kv_alloc(r.req_id, r.prefill_done + n)
            self.known.add(r.req_id)
        for r in decodes:
            self.eng.qos_kv_alloc(r.req_id, r.ctx_len + 1)
            self.orc.kv_alloc(r.req_id, r.ctx_len + 1)
        return chunks

    def execute(self, chunks, decodes):
        pre = [(r.req_id, r.prefill_done,
                synth.request_tokens(r.req_id, n, self.vocab, start=r.prefill_done)) for r, n in chunks]
        dec = [(r.req_id, r.ctx_len, self.next_tok[r.req_id]) for r in decodes]
        lg, tk = self.eng.step_host(self.q.make_batch(pre, dec), self.vocab)
        ref = self.orc.hybrid_step([(a, b, [int(x) for x in c]) for a, b, c in pre], dec)
        self.max_err = max(self.max_err, row_rel_err(lg, ref))
        srt = np.sort(ref, 1)
        gap = (srt[:, -1] - srt[:, -2]) / np.abs(ref).max(1)
        rt = np.argmax(ref, 1)
        assert all(tk[i] == rt[i] or gap[i] <= 2 * TOL_LOGITS for i in range(len(rt)))
        for (r, _), t in zip(chunks, rt[:len(pre)]):
            self.next_tok[r.req_id] = int(t)
        for r, t in zip(decodes, rt[len(pre):]):
            self.next_tok[r.req_id] = int(t)
        self.steps += 1
        return lin_model([(0, sum(n for _, n in chunks))], [r.ctx_len for r in decodes])

    def release(self, r):
        if r.req_id in self.known:
            self.eng.qos_kv_free(r.req_id)
            self.orc.kv_free(r.req_id)


def test_scheduler_drives_engine_and_oracle_in_lockstep():
    from oracle.engine import OracleEngine
    from oracle.model import PRESETS
    q, cfg, eng = make_engine("tiny", num_blocks=512, max_batch_tokens=512, max_batch_rows=32)
    eng.qos_engine_load_synthetic(0)
    orc = OracleEngine(PRESETS["tiny"], seed=0, num_blocks=512)
    rng = np.random.default_rng(0)
    tr = [{"req_id": i, "t_arrival": 0.01 * i, "prompt_len": int(rng.integers(20, 300)),
           "decode_len": int(rng.integers(1, 12)), "tier": ("Q1", "Q2", "Q3")[i % 3],
           "app_id": "t", "important": True} for i in range(12)]
    sched = QoServeScheduler(SchedulerConfig(max_chunk=256, min_chunk=16, chunk_step=16), lin_model)
    ex = Lockstep(q, eng, orc, cfg.vocab)
    out = replay(tr, sched, ex)
    assert out["finished"] == len(tr)
    assert ex.max_err <= TOL_LOGITS, ex.max_err
    assert ex.steps > 10
    assert eng.qos_kv_free_blocks() == 512 and orc.alloc.n_free == 512   # all KV released
    eng.close()


@pytest.mark.slow
def test_replay_llama8b_engine_executor():
    """configs[4] smoke: a 20 s Azure-Conv-shaped trace on Llama-3-8B shapes, every step a real
    device-timed qos_hybrid_step; the latency model is the engine's profile."""
    from paper_conf_asplos_goelmkar26_b200.latency_model import LatencyModel, StepShape
    from paper_conf_asplos_goelmkar26_b200.replay import EngineExecutor
    q, cfg, eng = make_engine("llama3-8b", num_blocks=40000, max_seq_len=8192, max_requests=512,
                              max_batch_tokens=4096 + 256, max_batch_rows=257)
    eng.qos_engine_load_synthetic(0)
    pts = [(c, nd) for c in (0, 256, 1024, 2048, 4096) for nd in (0, 32, 128) if c or nd]
    shapes, ms = [], []
    for c, nd in pts:
        t, _ = eng.qos_profile_step(c, [1024] * nd, reps=3)
        shapes.append(StepShape([(0, c)] if c else [], [1024] * nd))
        ms.append(t)
    model = LatencyModel().fit(shapes, ms)
    pred = lambda chunks, ctx: model.predict(StepShape(list(chunks), list(ctx)))   # noqa: E731
    tr = synth.trace(4.0, 20.0, "azure_conv")
    sched = QoServeScheduler(SchedulerConfig(max_chunk=4096), pred)
    ex = EngineExecutor(eng, cfg.vocab, lambda r, s, n: synth.request_tokens(r, n, cfg.vocab, start=s))
    out = replay(tr, sched, ex)
    assert out["finished"] == len(tr)
    assert out["tokens_per_s"] > 1000
    eng.close()
