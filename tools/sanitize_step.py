"""Workload for compute-sanitizer (SURVEY.md §4 test pyramid: memcheck / racecheck / synccheck
on the tiny config): every kernel family of the step, each launched at least once, small shapes.

  compute-sanitizer --tool memcheck   python tools/sanitize_step.py
  compute-sanitizer --tool racecheck  python tools/sanitize_step.py
  compute-sanitizer --tool synccheck  python tools/sanitize_step.py --sync
  bash tools/sanitize.sh            (all four tools, summaries in gpurun_out/sanitize_*.log)
  compute-sanitizer --tool racecheck  python tools/sanitize_step.py --wide   (Llama-3-8B width)

--sync skips the prefill chunks (decode-only steps on synthetic KV): synccheck flags the
prefill attention's o_full barrier, whose phases are completed once per P.V but observed by the
softmax warps only before a (rare) O rescale — by design, with the phase-parity argument in
attention_tc.cu; synccheck aborts the kernel at the first unobserved phase.

Covers: the tiny scenario (chunked prefills, a 128-token chunk + 4 decodes: weight-streaming
GEMMs, persistent prefill attention, split-K decode attention, norms, LM head, argmax), a
1700-token step (folded RMSNorm on the tile GEMMs), the TP2 peer group on one GPU (fused
reduce + residual + RMSNorm, logits gather), and op-level GEMMs on the CTA-pair kernel, the
ordered split-K, the stream-K and split-K tile kernel and the weight-streaming kernel.
No oracle comparison here (the tests do that); the sanitizer's report is the result.
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_asplos_goelmkar26_b200 import qoserve as q  # noqa: E402
from paper_conf_asplos_goelmkar26_b200.presets import preset  # noqa: E402


def tiny_engine(**over):
    caps = dict(num_blocks=512, max_seq_len=4096, max_requests=64, max_batch_tokens=2048, max_batch_rows=32)
    caps.update(over)
    return q.model_cfg(**preset("tiny"), **caps)


def scenario(engs, vocab):
    ctxs, warm, main, second = synth.tiny_scenario(vocab)
    run = (lambda f: [f(e) for e in engs]) if len(engs) == 1 else (lambda f: q.run_ranks(lambda k, e: f(e), engs))
    for r, n in ctxs.items():
        run(lambda e: e.qos_kv_alloc(r, n + 2))
    run(lambda e: e.qos_kv_alloc(0, 256))
    for b in warm + [main, second]:
        kb = q.batch_from_synth(b)
        run(lambda e: e.step_host(kb, vocab))


def decode_only(engs, vocab):
    run = (lambda f: [f(e) for e in engs]) if len(engs) == 1 else (lambda f: q.run_ranks(lambda k, e: f(e), engs))
    ctx = {201: 37, 202: 200, 203: 511, 204: 1000}
    for r, n in ctx.items():
        run(lambda e: e.qos_kv_alloc(r, n + 4))
        run(lambda e: e.qos_kv_fill_synthetic(r, n, 2))
    for k in range(3):
        kb = q.make_batch([], [(r, n + k, (r + k) % vocab) for r, n in ctx.items()])
        run(lambda e: e.step_host(kb, vocab))


def wide():
    """Llama-3-8B width, 2 layers: a 2048-token chunk + 16 decodes @1k (CTA-pair GEMMs with the
    folded norm, persistent prefill attention over 512 items with 5-D K/V boxes, split decode
    attention), then a second step with the CTA-pair prefill and persistent decode kernels."""
    cfg = q.model_cfg(**preset("llama3-8b", n_layers=2), num_blocks=(2048 + 16 * 1100) // 16 + 64,
                      max_seq_len=4096, max_requests=32, max_batch_tokens=2048 + 16, max_batch_rows=17)
    eng = q.Engine(cfg)
    eng.qos_engine_load_synthetic(0)
    b = synth.hybrid_batch(cfg.vocab, 2048, 16, 1024)
    eng.qos_kv_alloc(0, 2048)
    for d in b.decode:
        eng.qos_kv_alloc(d.req, 1025)
        eng.qos_kv_fill_synthetic(d.req, 1024, 2)
    eng.step_host(q.batch_from_synth(b), cfg.vocab)
    # the round-2 options: CTA-pair prefill attention (cta_group::2) and persistent decode
    # attention, on a second chunk and the decodes' next positions
    eng.qos_engine_set_option("fa_pair", 1)
    eng.qos_engine_set_option("decode_persist", 1)
    eng.qos_kv_alloc(1, 2048)
    for d in b.decode:
        eng.qos_kv_alloc(d.req, 1026)
    b2 = q.make_batch([(1, 0, np.asarray(b.prefill[0].tokens, dtype=np.int32))],
                      [(d.req, 1025, d.token) for d in b.decode])
    eng.step_host(b2, cfg.vocab)
    eng.close()
    print("sanitize workload done")


def main():
    if "--wide" in sys.argv:
        torch.cuda.set_device(0)
        wide()
        return
    sync = "--sync" in sys.argv
    torch.cuda.set_device(0)
    cfg = tiny_engine()
    eng = q.Engine(cfg)
    eng.qos_engine_load_synthetic(0)
    if sync:
        decode_only([eng], cfg.vocab)
        eng.close()
        g = q.Group(2)
        engs = [q.Engine(cfg, 0, r, 2, group=g) for r in range(2)]
        q.run_ranks(lambda r, e: e.qos_engine_load_synthetic(0), engs)
        decode_only(engs, cfg.vocab)
        for e in engs:
            e.close()
        g.close()
        op_gemms()
        return
    scenario([eng], cfg.vocab)
    # folded RMSNorm: a 1700-token chunk + 2 decodes (tile GEMMs, fold producer / consumer)
    rng = np.random.default_rng(11)
    eng.qos_kv_alloc(100, 1700)
    for r, n in ((101, 40), (102, 300)):
        eng.qos_kv_alloc(r, n + 1)
        eng.qos_kv_fill_synthetic(r, n, 2)
    b = q.make_batch([(100, 0, rng.integers(0, cfg.vocab, 1700).astype(np.int32))],
                     [(101, 40, 3), (102, 300, 5)])
    eng.step_host(b, cfg.vocab)
    eng.close()
    # TP2 peer group on one GPU
    g = q.Group(2)
    engs = [q.Engine(cfg, 0, r, 2, group=g) for r in range(2)]
    q.run_ranks(lambda r, e: e.qos_engine_load_synthetic(0), engs)
    scenario(engs, cfg.vocab)
    for e in engs:
        e.close()
    g.close()
    op_gemms()


def op_gemms():
    """op-level GEMMs on every kernel path"""
    gen = torch.Generator(device="cuda").manual_seed(0)

    def mk(M, N, K):
        A = (torch.rand(M, K, device="cuda", generator=gen) - 0.5).to(torch.bfloat16)
        B = ((torch.rand(N, K, device="cuda", generator=gen) - 0.5) / K ** 0.5).to(torch.bfloat16)
        return A, B

    for M, N, K, epi, ks in [(2176, 1024, 512, "add_f32", -3),      # CTA-pair kernel
                             (2176, 1024, 512, "silu_gate", -3),
                             (512, 1024, 8192, "add_f32", 2),       # ordered split-K
                             (300, 768, 640, "store_bf16", 3),      # split-K with parked partials
                             (777, 1280, 2048, "store_f32", -2),    # stream-K tile kernel
                             (16, 4096, 1024, "add_f32", -1),       # weight-streaming kernel
                             (100, 640, 1536, "silu_gate", -1)]:
        A, B = mk(M, N, K)
        ncol = N // 2 if epi == "silu_gate" else N
        C = torch.zeros(M, ncol, device="cuda", dtype=torch.float32 if "f32" in epi else torch.bfloat16)
        q.qos_op_gemm_ex(A.data_ptr(), B.data_ptr(), C.data_ptr(), M, N, K, epi, None, ks)
    torch.cuda.synchronize()
    print("sanitize workload done")


if __name__ == "__main__":
    main()
