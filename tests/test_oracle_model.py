"""Model-level pins of the oracle (CPU only).

* the whole tiny forward against Hugging Face ``transformers`` Llama / Qwen2 in fp64 loaded
  with the same generated weights (an independent implementation of the convention of
  reading s1-s3: norm placement, rotate-half RoPE, GQA head map, SwiGLU, untied head, bias);
* the invariants the paper fixes: chunked prefill over any split == one full prefill
  (PAPER.md:337-343, 946-948), a decode == the last row of a full causal prefill, and row
  independence of the fused batch.
"""
import numpy as np
import pytest
import torch

import synth
from oracle.engine import OracleBadKVStart, OracleEngine, OracleNotAllocated, greedy
from oracle.model import PRESETS, logits_of


def _hf_model(cfg, W):
    from transformers import LlamaConfig, LlamaForCausalLM, Qwen2Config, Qwen2ForCausalLM
    kw = dict(vocab_size=cfg.vocab, hidden_size=cfg.d_model, intermediate_size=cfg.ffn_dim,
              num_hidden_layers=cfg.n_layers, num_attention_heads=cfg.n_heads,
              num_key_value_heads=cfg.n_kv_heads, rms_norm_eps=cfg.rms_eps,
              rope_theta=cfg.rope_theta, tie_word_embeddings=False,
              max_position_embeddings=4096)
    if cfg.qkv_bias:
        hf = Qwen2ForCausalLM(Qwen2Config(**kw))
    else:
        hf = LlamaForCausalLM(LlamaConfig(head_dim=cfg.head_dim, **kw))
    sd = {"model.embed_tokens.weight": np.stack([W.embed([t])[0] for t in range(cfg.vocab)]),
          "model.norm.weight": W.final_norm(), "lm_head.weight": W.head()}
    from oracle.model import tensor_names
    for l in range(cfg.n_layers):
        w = W.layer(l)
        nm = tensor_names(cfg, l)
        for key in ("ln1", "wq", "wk", "wv", "wo", "ln2", "wg", "wu", "wd") + (
                ("bq", "bk", "bv") if cfg.qkv_bias else ()):
            sd[nm[key]] = w[key]
    hf = hf.to(torch.float64)
    missing, unexpected = hf.load_state_dict({k: torch.from_numpy(np.asarray(v)) for k, v in sd.items()},
                                             strict=False)
    assert not unexpected, unexpected
    assert all("rotary" in m for m in missing), missing
    # HF's SDPA path keeps the fp64 dtype; its eager path, its RMSNorm and its rotary angles
    # drop to fp32 (~1e-7 error).  Re-evaluate norm and angles in fp64 so the comparison can be
    # tight; both formulas are pinned independently in test_oracle_pins (F.rms_norm, complex
    # rotation), so this pin checks how HF *composes* them (placement, GQA map, rotate-half).
    hf.config._attn_implementation = "sdpa"
    for mod in hf.modules():
        if type(mod).__name__.endswith("RMSNorm"):
            def nfwd(x, _m=mod):
                return torch.nn.functional.rms_norm(x, (x.shape[-1],), _m.weight, eps=cfg.rms_eps)
            mod.forward = nfwd
    rot = hf.model.rotary_emb
    hd = cfg.head_dim

    def fwd64(x, position_ids):
        inv = 1.0 / (cfg.rope_theta ** (torch.arange(0, hd, 2, dtype=torch.float64) / hd))
        fr = position_ids[..., None].to(torch.float64) * inv
        emb = torch.cat([fr, fr], dim=-1)
        return emb.cos().to(x.dtype), emb.sin().to(x.dtype)
    rot.forward = fwd64
    return hf.eval()


@pytest.mark.parametrize("preset", ["tiny", "tiny-mha", "tiny-qwen"])
def test_tiny_forward_matches_transformers(preset):
    cfg = PRESETS[preset]
    eng = OracleEngine(cfg, seed=0, num_blocks=64)
    toks = synth.request_tokens(5, 70, cfg.vocab)
    eng.kv_alloc(5, 70)
    x = eng.forward_run(5, list(toks), 0)
    ours = logits_of(cfg, eng.W, x)
    hf = _hf_model(cfg, eng.W)
    with torch.no_grad():
        ref = hf(torch.from_numpy(toks.astype(np.int64))[None]).logits[0].numpy()
    err = np.abs(ours - ref).max() / np.abs(ref).max()
    assert err < 1e-10, err


def _fresh(cfg, nb=256):
    return OracleEngine(cfg, seed=0, num_blocks=nb)


def test_chunk_split_invariance():
    cfg = PRESETS["tiny"]
    toks = synth.request_tokens(3, 150, cfg.vocab)
    a = _fresh(cfg)
    a.kv_alloc(3, 150)
    la = a.hybrid_step([(3, 0, list(toks))], [])
    b = _fresh(cfg)
    b.kv_alloc(3, 150)
    b.hybrid_step([(3, 0, list(toks[:64]))], [])
    b.hybrid_step([(3, 64, list(toks[64:114]))], [])
    lb = b.hybrid_step([(3, 114, list(toks[114:]))], [])
    assert np.abs(la - lb).max() / np.abs(la).max() < 1e-12
    for l in range(cfg.n_layers):
        for i in range(2):
            assert np.allclose(a.kv[3][l][i], b.kv[3][l][i], rtol=1e-12, atol=1e-13)


def test_decode_equals_last_row_of_full_prefill():
    cfg = PRESETS["tiny"]
    toks = synth.request_tokens(9, 101, cfg.vocab)
    a = _fresh(cfg)
    a.kv_alloc(9, 101)
    la = a.hybrid_step([(9, 0, list(toks))], [])
    b = _fresh(cfg)
    b.kv_alloc(9, 101)
    b.hybrid_step([(9, 0, list(toks[:100]))], [])
    lb = b.hybrid_step([], [(9, 100, int(toks[100]))])
    assert np.abs(la - lb).max() / np.abs(la).max() < 1e-12


def test_batch_composition_invariance():
    cfg = PRESETS["tiny"]
    ctxs, warm, main, _ = synth.tiny_scenario(cfg.vocab)
    e = _fresh(cfg)
    for r, n in ctxs.items():
        e.kv_alloc(r, n + 2)
    e.kv_alloc(0, 256)
    for b in warm:
        e.hybrid_step(*b.as_oracle())
    mixed = e.hybrid_step(*main.as_oracle())
    # each request alone on a fresh engine
    for i, (req, n) in enumerate(sorted(ctxs.items())):
        s = _fresh(cfg)
        s.kv_alloc(req, n + 2)
        toks = synth.request_tokens(req, n + 1, cfg.vocab)
        s.hybrid_step([(req, 0, list(toks[:n]))], [])
        alone = s.hybrid_step([], [(req, n, int(toks[n]))])
        assert np.abs(mixed[1 + i] - alone[0]).max() / np.abs(alone).max() < 1e-12


@pytest.mark.parametrize("preset", ["tiny", "tiny-qwen"])
def test_layer_major_step_equals_request_major_step(preset):
    """hybrid_step_layer_major (layer loop outside, used for the full-depth bench-size check)
    gives bit-identical logits and KV to hybrid_step (request loop outside) over the whole tiny
    scenario: the same operations in the same order per request."""
    cfg = PRESETS[preset]
    ctxs, warm, main, second = synth.tiny_scenario(cfg.vocab)
    a, b = _fresh(cfg), _fresh(cfg)
    for e in (a, b):
        for r, n in ctxs.items():
            e.kv_alloc(r, n + 2)
        e.kv_alloc(0, 256)
    for st in warm + [main, second]:
        la = a.hybrid_step(*st.as_oracle())
        lb = b.hybrid_step_layer_major(*st.as_oracle())
        assert np.array_equal(la, lb)
    for r in list(ctxs) + [0]:
        for l in range(cfg.n_layers):
            assert np.array_equal(a.kv[r][l][0], b.kv[r][l][0]) and np.array_equal(a.kv[r][l][1], b.kv[r][l][1])
    with pytest.raises(ValueError):
        b.hybrid_step_layer_major([(0, 0, [1])], [(0, 0, 1)])
    with pytest.raises(OracleBadKVStart):
        b.hybrid_step_layer_major([(0, 3, [1])], [])


def test_step_semantics_errors():
    cfg = PRESETS["tiny"]
    e = _fresh(cfg, nb=4)
    e.kv_alloc(1, 16)
    with pytest.raises(OracleNotAllocated):
        e.hybrid_step([(1, 0, [1] * 17)], [])
    e.hybrid_step([(1, 0, [1] * 10)], [])
    with pytest.raises(OracleBadKVStart):
        e.hybrid_step([(1, 0, [1] * 3)], [])
    with pytest.raises(ValueError):
        e.hybrid_step([(1, 10, [1])], [(1, 10, 2)])


def test_greedy_lowest_index_on_ties():
    assert list(greedy(np.array([[1.0, 3.0, 3.0, 2.0], [0.0, 0.0, 0.0, 0.0]]))) == [1, 0]
