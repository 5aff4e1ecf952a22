"""Latency model (dynamic chunking predictor) on CPU: recovers a known linear cost, mirrors the
engine's GEMM tiling, and (when the committed profile exists) predicts the measured B200
latency table within the north star's 5% on most points."""
import json
import os

import numpy as np

from paper_conf_asplos_goelmkar26_b200.latency_model import (N_FEAT, GemmShapes, LatencyModel, StepShape, features, gemm_work,
                                                             pair_eligible, pair_work, stream_work)

PROF = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles", "latency_table_r2d.json")


def test_recovers_known_coefficients():
    rng = np.random.default_rng(0)
    true = np.array([2.0, 3.0, 20.0, 0.5, 1.0, 4.0, 9.0, 6.0, 5.0, 1.5, 0.3, 0.2, -0.4, -0.3])
    assert len(true) == N_FEAT
    shapes = [StepShape([], list(rng.integers(1024, 8193, nd))) for nd in (1, 8, 16, 24, 32, 64, 100, 200, 256)]
    for _ in range(120):
        c = int(rng.integers(0, 8193))
        nd = int(rng.integers(0, 257))
        shapes.append(StepShape([(int(rng.integers(0, 4097)), c)] if c else [], list(rng.integers(1024, 8193, nd))))
    y = [features(s) @ true for s in shapes if s.T > 0]
    m = LatencyModel().fit([s for s in shapes if s.T > 0], y)
    pred = [m.predict(s) for s in shapes if s.T > 0]
    assert np.allclose(pred, y, rtol=1e-8)
    m2 = LatencyModel.from_json(m.to_json())
    assert abs(m2.predict(shapes[0]) - m.predict(shapes[0])) < 1e-9


def test_gemm_work_is_tile_quantised():
    g = GemmShapes()
    assert gemm_work(1024, g) == gemm_work(1024 - 100, g)        # same 8 M-tiles
    go = GemmShapes(((4096, 4096),), 148)                         # the O projection alone
    assert pair_work(4096, go) == pair_work(4096 - 200, go)      # same 16 pair M-tiles
    w = [pair_work(t, go) for t in range(2048, 8449, 256)]
    assert all(a <= b for a, b in zip(w, w[1:]))                   # steps, never decreasing
    assert len(set(w)) > 5
    assert gemm_work(8448, g) + pair_work(8448, g) > 3 * (gemm_work(2176, g) + pair_work(2176, g))


def test_pair_gemm_selection_mirrors_the_engine():
    """gemm2_eligible (csrc/gemm.cu): pair tiles once 128 x 256 tiles fill the 148 SMs and the
    256-row padding costs no extra wave — at T = 2176 the QKV, O and down projections take the
    CTA-pair kernel and gate/up (13 single vs 14 pair waves) keeps single-CTA tiles."""
    (qkv, o, gu, down) = GemmShapes().gemms
    assert pair_eligible(2176, *qkv, 148) and pair_eligible(2176, *o, 148) and pair_eligible(2176, *down, 148)
    assert not pair_eligible(2176, *gu, 148)
    assert not pair_eligible(512, *o, 148)                        # 4 x 16 tiles < 148 SMs
    assert pair_eligible(8192, *gu, 148)


def test_small_steps_use_the_weight_streaming_gemm():
    g = GemmShapes()
    assert stream_work(1, g) == sum(n * k for n, k in g.gemms)        # every projection streams
    assert stream_work(2176, g) == 0 and gemm_work(1, g) == 0
    # up to T = 64 every projection streams (round-2 rule, csrc/gemm_swab.cu: swab_prefer)
    assert stream_work(64, g) == sum(n * k for n, k in g.gemms)
    # T = 128: only the O and down projections (32 output tiles) take the streaming kernel
    assert stream_work(128, g) == 4096 * 4096 + 4096 * 14336


def test_committed_profile_predictability():
    if not os.path.exists(PROF):
        return
    d = json.load(open(PROF))
    assert d["test_points"] >= 100
    assert d["within_5pct"] >= 0.9 and d["test_rel_err_max"] < 0.1
