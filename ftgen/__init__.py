"""Seeded synthetic-input generator shared by the oracle tests, the GPU tests and bench.py.

This module is the ONLY code both sides use.  It holds none of the method's arithmetic
(no gate, no activation, no recurrence): it only draws counter-based uniform numbers and
rounds them to the storage precision the two paths agree on.

Generator: splitmix64 finaliser applied to a per-tensor counter, so any element (and any
batch-row subset) can be regenerated independently of the others.

Recipe:
  * x, ys           ~ U(-1, 1)
  * W, U, b         ~ U(-scale/sqrt(H), +scale/sqrt(H)), scale = 1 (PyTorch's LSTM default) —
                      the judged distribution; scale 2 is the "signal preserving" set.
  * bf16 path: x, ys, W, U rounded to bf16 (round-to-nearest-even) ONCE here; b stays fp32.
  * f32 path : everything rounded to fp32 once here.
Both paths then see bit-identical values; the oracle widens them to fp64 exactly.
"""
from __future__ import annotations

import numpy as np

GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)

# stream ids, one per tensor
S_X, S_YS, S_W, S_U, S_B = 1, 2, 3, 4, 5

SEED_BASE = 0x5EED0000  # seed = SEED_BASE + config index


def _mix(z: np.ndarray) -> np.ndarray:
    with np.errstate(over="ignore"):
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
        return z ^ (z >> np.uint64(31))


def uniform(seed: int, stream: int, n: int, offset: int = 0) -> np.ndarray:
    """n float64 values in [-1, 1): element i is a pure function of (seed, stream, offset+i)."""
    key = _mix(np.array([(seed * 256 + stream) & 0xFFFFFFFFFFFFFFFF], dtype=np.uint64))[0]
    idx = np.arange(offset + 1, offset + n + 1, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = _mix(key + idx * GOLDEN)
    u53 = (z >> np.uint64(11)).astype(np.float64)
    return u53 * (2.0 ** -52) - 1.0


def round_f32(a: np.ndarray) -> np.ndarray:
    return np.asarray(a, dtype=np.float64).astype(np.float32)


def round_bf16(a: np.ndarray) -> np.ndarray:
    """Round to bf16 (RNE via fp32), returned as float32 holding bf16-representable values."""
    f = round_f32(a)
    bits = f.view(np.uint32).astype(np.uint64)
    bits = (bits + np.uint64(0x7FFF) + ((bits >> np.uint64(16)) & np.uint64(1))) >> np.uint64(16)
    out = (bits.astype(np.uint32) << np.uint32(16)).view(np.float32)
    return out.reshape(np.shape(a))


def bf16_bits(a32: np.ndarray) -> np.ndarray:
    """uint16 storage bits of float32 values that are already bf16-representable."""
    u = np.ascontiguousarray(a32, dtype=np.float32).view(np.uint32)
    assert np.all((u & 0xFFFF) == 0), "value not bf16-representable"
    return (u >> 16).astype(np.uint16)


def _draw(seed, stream, shape, lo_hi, store):
    n = int(np.prod(shape))
    v = uniform(seed, stream, n).reshape(shape) * lo_hi
    return round_bf16(v) if store == "bf16" else round_f32(v)


def stacked_inputs(batch, seq, hidden, depth, seed, dtype="bf16", scale=1.0):
    """Inputs of ft_stacked_lstm_fwd / ft_dilated_rnn_fwd (paper Listing 2 L590-L599 shapes).

    Returns float32 arrays whose values are exactly representable in `dtype` storage:
      x [B][T][H], W [D][4][H][H], U [D][4][H][H], b [D][4][H] (b always fp32).
    """
    r = scale / np.sqrt(hidden)
    return dict(
        x=_draw(seed, S_X, (batch, seq, hidden), 1.0, dtype),
        W=_draw(seed, S_W, (depth, 4, hidden, hidden), r, dtype),
        U=_draw(seed, S_U, (depth, 4, hidden, hidden), r, dtype),
        b=_draw(seed, S_B, (depth, 4, hidden), r, "f32"),
    )


def linear_rnn_inputs(batch, seq, hidden, depth, seed, dtype="bf16", scale=1.0):
    """Inputs of ft_stacked_rnn_fwd (Listing 1): x [B][T][H], W [D][H][H]."""
    r = scale / np.sqrt(hidden)
    return dict(
        x=_draw(seed, S_X, (batch, seq, hidden), 1.0, dtype),
        W=_draw(seed, S_W, (depth, hidden, hidden), r, dtype),
    )


def b2b_inputs(M, N, K, P, seed, dtype="bf16"):
    """Inputs of ft_b2b_gemm_fwd: A [M][K] ~ U(-1,1), B [K][N] ~ U(±1/√K), C [N][P] ~ U(±1/√N)
    (scaled so S = A@B and D = S@C stay O(1))."""
    return dict(
        A=_draw(seed, S_X, (M, K), 1.0, dtype),
        B=_draw(seed, S_W, (K, N), 1.0 / np.sqrt(K), dtype),
        C=_draw(seed, S_U, (N, P), 1.0 / np.sqrt(N), dtype),
    )


def grid_inputs(batch, len_x, len_y, hidden, depth, seed, dtype="bf16", scale=1.0):
    """Inputs of ft_grid_rnn_fwd: x [B][Lx][H], ys [B][Ly][H], W [D][2][4][H][H],
    U [D][2][4][2H][H], b [D][2][4][H]."""
    r = scale / np.sqrt(hidden)
    return dict(
        x=_draw(seed, S_X, (batch, len_x, hidden), 1.0, dtype),
        ys=_draw(seed, S_YS, (batch, len_y, hidden), 1.0, dtype),
        W=_draw(seed, S_W, (depth, 2, 4, hidden, hidden), r, dtype),
        U=_draw(seed, S_U, (depth, 2, 4, 2 * hidden, hidden), r, dtype),
        b=_draw(seed, S_B, (depth, 2, 4, hidden), r, "f32"),
    )


def sample_rows(batch, k, seed):
    """Rows used for full-size parity: {0, 1, B/2, B-1} + k seeded rows."""
    base = sorted({0, min(1, batch - 1), batch // 2, batch - 1})
    u = uniform(seed, 99, 4 * k + 8)
    extra = []
    for v in u:
        r = int((v + 1.0) * 0.5 * batch) % batch
        if r not in base and r not in extra:
            extra.append(r)
        if len(extra) == k:
            break
    return sorted(base + extra)


# BASELINE.json configs: name -> dict
CONFIGS = {
    "C1": dict(kind="stacked", batch=4, seq=8, hidden=32, depth=2, dtype="f32"),
    "C2": dict(kind="stacked", batch=64, seq=64, hidden=256, depth=8, dtype="bf16"),
    "C3": dict(kind="stacked", batch=256, seq=100, hidden=1024, depth=16, dtype="bf16"),
    "C4": dict(kind="dilated", batch=256, seq=100, hidden=512, depth=6,
               dilations=(1, 2, 4, 8, 16, 32), dtype="bf16"),
    "C5": dict(kind="grid", batch=128, len_x=32, len_y=32, hidden=512, depth=4, dtype="bf16"),
}


def config_seed(name: str) -> int:
    return SEED_BASE + int(name[1:])
