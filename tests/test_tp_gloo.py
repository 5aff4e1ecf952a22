"""Tensor-parallel path on CPU (world_size 2, gloo): the library's shard plan
(`qos_shard_plan`, the same `make_shard` the engine loads weights with) drives a sharded fp64
forward whose partial O / down projections are summed with a real all-reduce and whose vocab
shards are all-gathered — exactly the collectives the engine issues over NCCL (SURVEY.md §8(e),
PAPER.md:899-902 vLLM TP).  The result must equal the unsharded oracle forward."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, preset, out_q):
    import sys
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import synth
        from oracle.engine import OracleEngine
        from oracle.model import PRESETS, apply_rope, causal_attention, logits_of, rms_norm, silu
        from paper_conf_asplos_goelmkar26_b200 import qoserve as q
        from paper_conf_asplos_goelmkar26_b200.presets import preset as ppreset
        c = PRESETS[preset]
        cfg = q.model_cfg(**ppreset(preset), num_blocks=64)
        sp = q.qos_shard_plan(cfg, rank, world)
        orc = OracleEngine(c, seed=0, num_blocks=64)
        W = orc.W
        hd, g = c.head_dim, c.n_heads // c.n_kv_heads
        qs = slice(sp.head0 * hd, (sp.head0 + sp.n_heads) * hd)
        ks = slice(sp.kv_head0 * hd, (sp.kv_head0 + sp.n_kv_heads) * hd)
        fs = slice(sp.ffn0, sp.ffn0 + sp.ffn)
        vs = slice(sp.vocab0, sp.vocab0 + sp.vocab)
        n = 45
        toks = synth.request_tokens(3, n, c.vocab)
        pos = np.arange(n)
        x = W.embed(toks)

        def allreduce(a):
            t = torch.from_numpy(np.ascontiguousarray(a))
            dist.all_reduce(t)
            return t.numpy()

        for l in range(c.n_layers):
            w = W.layer(l)
            h = rms_norm(x, w["ln1"], c.rms_eps)
            qq = h @ w["wq"][qs].T
            kk = h @ w["wk"][ks].T
            vv = h @ w["wv"][ks].T
            if c.qkv_bias:
                qq, kk, vv = qq + w["bq"][qs], kk + w["bk"][ks], vv + w["bv"][ks]
            qq = apply_rope(qq.reshape(n, sp.n_heads, hd), pos, c.rope_theta)
            kk = apply_rope(kk.reshape(n, sp.n_kv_heads, hd), pos, c.rope_theta)
            vv = vv.reshape(n, sp.n_kv_heads, hd)
            o = causal_attention(qq, kk, vv, 0, g).reshape(n, sp.n_heads * hd)
            x = x + allreduce(o @ w["wo"][:, qs].T)              # a9 + a10
            h2 = rms_norm(x, w["ln2"], c.rms_eps)
            m = (silu(h2 @ w["wg"][fs].T) * (h2 @ w["wu"][fs].T)) @ w["wd"][:, fs].T
            x = x + allreduce(m)                                  # a12 + a10
        loc = rms_norm(x[-1:], W.final_norm(), c.rms_eps) @ W.head()[vs].T
        parts = [torch.zeros_like(torch.from_numpy(loc)) for _ in range(world)]
        dist.all_gather(parts, torch.from_numpy(np.ascontiguousarray(loc)))   # a13 vocab all-gather
        logits = torch.cat(parts, dim=1).numpy()
        if rank == 0:
            orc.kv_alloc(3, n)
            ref = logits_of(c, W, orc.forward_run(3, list(toks), 0)[-1:])
            out_q.put((float(np.abs(logits - ref).max() / np.abs(ref).max()),
                       [(p.head0, p.n_heads, p.kv_head0, p.n_kv_heads, p.ffn0, p.ffn, p.vocab0, p.vocab)
                        for p in [q.qos_shard_plan(cfg, r, world) for r in range(world)]]))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("preset", ["tiny", "tiny-qwen"])
def test_tp2_sharded_forward_matches_unsharded_oracle(preset):
    ctx = mp.get_context("spawn")
    out_q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, preset, out_q)) for r in range(2)]
    for p in procs:
        p.start()
    err, plans = out_q.get(timeout=300)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    assert err < 1e-10, err
    # the plan tiles heads / kv heads / FFN / vocab exactly (disjoint, complete)
    from oracle.model import PRESETS
    c = PRESETS[preset]
    for field, total in ((0, c.n_heads), (2, c.n_kv_heads), (4, c.ffn_dim), (6, c.vocab)):
        spans = sorted((pl[field], pl[field] + pl[field + 1]) for pl in plans)
        assert spans[0][0] == 0 and spans[-1][1] == total
        assert all(a[1] == b[0] for a, b in zip(spans, spans[1:]))


def test_shard_plan_8way_llama70b():
    from paper_conf_asplos_goelmkar26_b200 import qoserve as q
    from paper_conf_asplos_goelmkar26_b200.presets import preset
    cfg = q.model_cfg(**preset("llama3-70b"), num_blocks=16)
    plans = [q.qos_shard_plan(cfg, r, 8) for r in range(8)]
    assert [p.kv_head0 for p in plans] == list(range(8))
    assert all(p.n_heads == 8 and p.n_kv_heads == 1 and p.ffn == 3584 and p.vocab == 16032 for p in plans)
    with pytest.raises(q.QosError):
        q.qos_shard_plan(cfg, 8, 8)
