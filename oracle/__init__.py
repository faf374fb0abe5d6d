"""CPU oracle (TEST INFRASTRUCTURE ONLY).

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs may
import this package.  It wraps the plain-C loop nest in ft_oracle.c (the paper's definitions,
see that file's header for the PAPER.md citations) through ctypes.  It shares no code with the
CUDA path (paper_conf_sosp_liuqc0hs0y24_b200/) and never imports it.

Pins: tests/test_oracle_pins.py (P1–P14 of SURVEY.md §8(c) c.6).  The grid cell (R12–R14)
is "parity unpinned" by the paper beyond its Ly=1 / Lx=1 reductions (P8): the paper never
defines it.  The oracle's reading is pinned by P8/P8b, the no-recurrence closed form P8c and
the exact dependence cone P8d.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "liboracle.so")
_SOURCES = [os.path.join(_HERE, "ft_oracle.c"), os.path.join(_HERE, "ft_oracle_impl.h")]


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc (-O2 -fopenmp; no -ffast-math: IEEE semantics kept)."""
    newest = max(os.path.getmtime(s) for s in _SOURCES)
    if not force and os.path.exists(LIB_PATH) and os.path.getmtime(LIB_PATH) >= newest:
        return LIB_PATH
    cmd = ["gcc", "-O2", "-march=x86-64-v2", "-fopenmp", "-fPIC", "-shared", "-std=c11",
           "-fvisibility=hidden", "-ffp-contract=off", "-o", LIB_PATH + ".tmp", _SOURCES[0], "-lm"]
    subprocess.check_call(cmd, cwd=_HERE)
    os.replace(LIB_PATH + ".tmp", LIB_PATH)
    return LIB_PATH


def _host_key() -> str:
    """Identifies the host CPU, so a -march=native build is never loaded on another CPU model."""
    import hashlib
    model = ""
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith(("model name", "flags")):
                    model += line
                    if line.startswith("flags"):
                        break
    except OSError:
        pass
    return hashlib.sha1(model.encode()).hexdigest()[:12]


def timing_lib_path() -> str:
    return os.path.join(_HERE, f"liboracle_timing_{_host_key()}.so")


def build_timing(force: bool = False) -> str:
    """The CPU-baseline build of the SAME source: -O3 -march=native for the
    host it runs on, still -ffp-contract=off and no -ffast-math, so every output is bitwise the
    parity build's (pinned in tests/test_oracle_pins.py).  Compiled on first use on each host
    (the GPU box's CPU may differ from the build machine's)."""
    path = timing_lib_path()
    newest = max(os.path.getmtime(s) for s in _SOURCES)
    if not force and os.path.exists(path) and os.path.getmtime(path) >= newest:
        return path
    cmd = ["gcc", "-O3", "-march=native", "-fopenmp", "-fPIC", "-shared", "-std=c11",
           "-fvisibility=hidden", "-ffp-contract=off", "-o", path + ".tmp", _SOURCES[0], "-lm"]
    subprocess.check_call(cmd, cwd=_HERE)
    os.replace(path + ".tmp", path)
    return path


_libs = {}


def lib(which: str = "parity"):
    """The oracle library: "parity" (-O2, portable; the tests' reference) or "timing" (the
    CPU-baseline build of the same source, bitwise identical results)."""
    if which not in _libs:
        path = build() if which == "parity" else build_timing()
        L = ctypes.CDLL(path)
        for sfx in ("f64", "f32", "bf16emu"):
            for name in ("stacked_lstm", "dilated_rnn", "grid_rnn", "lstm_cell", "stacked_rnn",
                         "b2b_gemm"):
                fn = getattr(L, f"ft_oracle_{name}_{sfx}")
                fn.restype = ctypes.c_int if name != "lstm_cell" else None
        _libs[which] = L
    return _libs[which]


def num_threads(which: str = "parity") -> int:
    return int(lib(which).ft_oracle_num_threads())


def _p(a):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def _prec(precision):
    if precision == "f64":
        return np.float64
    if precision in ("f32", "bf16emu"):  # bf16emu: diagnostic, float with h rounded to bf16 per cell
        return np.float32
    raise ValueError(precision)


def _c(a, dt):
    return np.ascontiguousarray(a, dtype=dt)


def stacked_lstm(x, W, U, b, precision="f64", want_all=False, build_kind="parity"):
    """Stacked LSTM oracle (Listing 2).  x [B][T][H], W/U [D][4][H][H], b [D][4][H]."""
    dt = _prec(precision)
    B, T, H = x.shape
    D = W.shape[0]
    x, W, U, b = (_c(a, dt) for a in (x, W, U, b))
    y = np.empty((B, T, H), dt)
    h_n = np.empty((B, D, H), dt)
    c_n = np.empty((B, D, H), dt)
    h_all = np.empty((B, D, T, H), dt) if want_all else None
    c_all = np.empty((B, D, T, H), dt) if want_all else None
    rc = getattr(lib(build_kind), f"ft_oracle_stacked_lstm_{precision}")(
        B, T, H, D, _p(x), _p(W), _p(U), _p(b), _p(y), _p(h_n), _p(c_n), _p(h_all), _p(c_all))
    if rc:
        raise RuntimeError(f"oracle stacked_lstm failed: {rc}")
    out = dict(y=y, h_n=h_n, c_n=c_n)
    if want_all:
        out.update(h_all=h_all, c_all=c_all)
    return out


def dilated_rnn(x, W, U, b, dilations, precision="f64", want_all=False):
    dt = _prec(precision)
    B, T, H = x.shape
    D = W.shape[0]
    dil = np.ascontiguousarray(dilations, dtype=np.int32)
    assert dil.shape == (D,)
    x, W, U, b = (_c(a, dt) for a in (x, W, U, b))
    y = np.empty((B, T, H), dt)
    h_n = np.empty((B, D, H), dt)
    c_n = np.empty((B, D, H), dt)
    h_all = np.empty((B, D, T, H), dt) if want_all else None
    c_all = np.empty((B, D, T, H), dt) if want_all else None
    rc = getattr(lib(), f"ft_oracle_dilated_rnn_{precision}")(
        B, T, H, D, _p(dil), _p(x), _p(W), _p(U), _p(b), _p(y), _p(h_n), _p(c_n),
        _p(h_all), _p(c_all))
    if rc:
        raise RuntimeError(f"oracle dilated_rnn failed: {rc}")
    out = dict(y=y, h_n=h_n, c_n=c_n)
    if want_all:
        out.update(h_all=h_all, c_all=c_all)
    return out


def grid_rnn(x, ys, W, U, b, precision="f64", want_all=False):
    """Grid RNN oracle (readings R12–R14).  x [B][Lx][H], ys [B][Ly][H], W [D][2][4][H][H],
    U [D][2][4][2H][H], b [D][2][4][H]."""
    dt = _prec(precision)
    B, Lx, H = x.shape
    Ly = ys.shape[1]
    D = W.shape[0]
    x, ys, W, U, b = (_c(a, dt) for a in (x, ys, W, U, b))
    out = np.empty((B, Lx, Ly, 2, H), dt)
    h_n = np.empty((B, D, 2, H), dt)
    c_n = np.empty((B, D, 2, H), dt)
    h_all = np.empty((B, D, Lx, Ly, 2, H), dt) if want_all else None
    c_all = np.empty((B, D, Lx, Ly, 2, H), dt) if want_all else None
    rc = getattr(lib(), f"ft_oracle_grid_rnn_{precision}")(
        B, Lx, Ly, H, D, _p(x), _p(ys), _p(W), _p(U), _p(b), _p(out), _p(h_n), _p(c_n),
        _p(h_all), _p(c_all))
    if rc:
        raise RuntimeError(f"oracle grid_rnn failed: {rc}")
    res = dict(out=out, h_n=h_n, c_n=c_n)
    if want_all:
        res.update(h_all=h_all, c_all=c_all)
    return res


def lstm_cell(a, W4, hp, U4, b4, cp, precision="f64"):
    """One cell (Listing 2).  a [Ka], W4 [4][Ka][H], hp [Kh] or None, U4 [4][Kh][H],
    b4 [4][H], cp [H] or None.  Returns (h, c)."""
    dt = _prec(precision)
    H = b4.shape[1]
    a = _c(a, dt)
    W4 = _c(W4, dt)
    U4 = _c(U4, dt)
    b4 = _c(b4, dt)
    hp = None if hp is None else _c(hp, dt)
    cp = None if cp is None else _c(cp, dt)
    h = np.empty(H, dt)
    c = np.empty(H, dt)
    z = np.empty(4 * H, dt)
    Kh = U4.shape[1]
    getattr(lib(), f"ft_oracle_lstm_cell_{precision}")(
        H, _p(a), a.shape[0], _p(W4), _p(hp), Kh, _p(U4), _p(b4), _p(cp), _p(h), _p(c), _p(z))
    return h, c


def stacked_rnn(x, W, precision="f64"):
    """Stacked linear RNN oracle (Listing 1): y[d][t] = a @ W[d] + y[d][t-1].
    x [B][T][H], W [D][H][H] → ysss [B][D][T][H]."""
    dt = _prec(precision)
    B, T, H = x.shape
    D = W.shape[0]
    x, W = _c(x, dt), _c(W, dt)
    ys = np.empty((B, D, T, H), dt)
    rc = getattr(lib(), f"ft_oracle_stacked_rnn_{precision}")(B, T, H, D, _p(x), _p(W), _p(ys))
    if rc:
        raise RuntimeError(f"oracle stacked_rnn failed: {rc}")
    return ys


def b2b_gemm(A, B, C, precision="f64"):
    """Back-to-back GEMMs (Table 6; reading R22): D = (A @ B) @ C.
    A [M][K], B [K][N], C [N][P] → D [M][P]."""
    dt = _prec(precision)
    M, K = A.shape
    N = B.shape[1]
    P = C.shape[1]
    A, B, C = _c(A, dt), _c(B, dt), _c(C, dt)
    D = np.empty((M, P), dt)
    rc = getattr(lib(), f"ft_oracle_b2b_gemm_{precision}")(M, N, K, P, _p(A), _p(B), _p(C), _p(D))
    if rc:
        raise RuntimeError(f"oracle b2b_gemm failed: {rc}")
    return D
