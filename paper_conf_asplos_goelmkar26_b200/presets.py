"""Model shapes served by the engine (SURVEY.md §8 preset table).

The paper names the models only (Table 1); dims are the public configs [ext].
`tiny` is configs[0] (L=2, d=256, 4 heads, block 16) with our readings for Hkv/F/V/theta (s15).
"""
from __future__ import annotations

PRESETS = {
    "tiny": dict(n_layers=2, d_model=256, n_heads=4, n_kv_heads=2, head_dim=64, ffn_dim=768, vocab=1024,
                 rope_theta=10000.0, rms_eps=1e-5, qkv_bias=False),
    "tiny-mha": dict(n_layers=2, d_model=256, n_heads=4, n_kv_heads=4, head_dim=64, ffn_dim=768, vocab=1024,
                     rope_theta=10000.0, rms_eps=1e-5, qkv_bias=False),
    "tiny-qwen": dict(n_layers=2, d_model=256, n_heads=4, n_kv_heads=2, head_dim=64, ffn_dim=768, vocab=1024,
                      rope_theta=1e6, rms_eps=1e-6, qkv_bias=True),
    "llama3-8b": dict(n_layers=32, d_model=4096, n_heads=32, n_kv_heads=8, head_dim=128, ffn_dim=14336,
                      vocab=128256, rope_theta=500000.0, rms_eps=1e-5, qkv_bias=False),
    "qwen2.5-14b": dict(n_layers=48, d_model=5120, n_heads=40, n_kv_heads=8, head_dim=128, ffn_dim=13824,
                        vocab=152064, rope_theta=1e6, rms_eps=1e-6, qkv_bias=True),
    "llama3-70b": dict(n_layers=80, d_model=8192, n_heads=64, n_kv_heads=8, head_dim=128, ffn_dim=28672,
                       vocab=128256, rope_theta=500000.0, rms_eps=1e-5, qkv_bias=False),
}


def preset(name: str, **over) -> dict:
    d = dict(PRESETS[name])
    d.update(over)
    return d
