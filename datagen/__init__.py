"""Seeded synthetic inputs for the CART hot path (host side).

This module is the ONLY code the oracle and the CUDA path have in common: it makes
inputs and holds none of the method's arithmetic (no sums, splits, gains, metrics).

Row schema follows the paper's dataset row d = (y, p, c_1..c_m, t) (Eq. 1):
p = executed PTX instructions, c_i = GPU architectural descriptors (CUDA cores,
memory, L2, clocks, memory bandwidth), t = trainable parameters
(P:140).  The paper's data is private, so values are synthetic; the recipe is stated in
DESIGN.md ("Input recipe") and mirrored bit-for-bit by the device generator
(`dt_gen_table` in the product library), which is why only +, -, *, /, floor, ldexp and
a hand-written exp (Horner polynomial, no FMA) are used below: every step is an IEEE
correctly-rounded operation that the GPU reproduces exactly.

Counter-based RNG: h(seed, stream, i, k) = mix64(mix64(seed ^ (stream << 56)) + i*G + k*H)
(SplitMix64 finaliser), uniform = (h >> 11) * 2^-53.
"""
from __future__ import annotations

import math

import numpy as np

M64 = (1 << 64) - 1
G = 0x9E3779B97F4A7C15
H = 0xD1B54A32D192ED03
TWO_M53 = 2.0 ** -53
LOG2E = 1.4426950408889634        # float(1/ln 2)
LN2 = 0.6931471805599453          # float(ln 2)
EXP_COEF = tuple(1.0 / math.factorial(j) for j in range(15))  # Horner, degree 14

# Table I input sizes, for the p model; the efficientnetb5 "156" is read as
# 456 (garbled).
SIDES = (224.0, 240.0, 260.0, 299.0, 300.0, 331.0, 380.0, 456.0, 528.0, 600.0)
MEM_GB = (4.0, 8.0, 11.0, 16.0, 24.0, 32.0, 48.0, 80.0, 96.0, 141.0, 192.0)

# Stream ids (high byte of the seed key) -- one per independent draw family.
S_ROWCNN, S_ROWGPU, S_ROWNOISE, S_CNN, S_GPU, S_SPLIT = 1, 2, 3, 4, 5, 6


def _u64(x):
    return np.asarray(x, dtype=np.uint64)


def mix64(z):
    z = _u64(z)
    with np.errstate(over="ignore"):
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        return z ^ (z >> np.uint64(31))


def hash64(seed: int, stream: int, i, k: int):
    key = mix64(np.uint64((seed ^ (stream << 56)) & M64))
    with np.errstate(over="ignore"):
        c = key + _u64(i) * np.uint64(G) + np.uint64((k * H) & M64)
    return mix64(c)


def uniform(seed: int, stream: int, i, k: int):
    """Uniform fp64 in [0, 1) from the counter (seed, stream, i, k)."""
    return (hash64(seed, stream, i, k) >> np.uint64(11)).astype(np.float64) * TWO_M53


def exp_det(x):
    """exp(x) from +, *, floor, ldexp only (bit-reproducible on the GPU, |x| < 700)."""
    x = np.asarray(x, dtype=np.float64)
    t = x * LOG2E
    k = np.floor(t)
    s = (t - k) * LN2
    p = np.full_like(s, EXP_COEF[14])
    for j in range(13, -1, -1):
        p = p * s + EXP_COEF[j]
    return np.ldexp(p, k.astype(np.int32))


def log_uniform(u, lo: float, hi: float):
    """lo * exp(u * ln(hi/lo)); ln(hi/lo) as a Python float constant."""
    return lo * exp_det(u * math.log(hi / lo))


def irwin_hall(seed, stream, i, k0, clip=4.0):
    """Approximately N(0,1): sum of 12 uniforms - 6, clipped to [-clip, clip]."""
    z = np.zeros(np.shape(i), dtype=np.float64)
    for j in range(12):
        z = z + uniform(seed, stream, i, k0 + j)
    z = z - 6.0
    return np.minimum(np.maximum(z, -clip), clip)


# --------------------------------------------------------------- CNN x GPU table ----

def _cnn_cols(seed, cid, n_extra=False):
    """CNN-side columns of pool entry cid: t, p, h0..h7 (+ S32 extras)."""
    t = log_uniform(uniform(seed, S_CNN, cid, 0), 3.5e6, 9.4e8)      # Table I range
    side = np.asarray(SIDES)[(hash64(seed, S_CNN, cid, 1) % np.uint64(len(SIDES))).astype(np.int64)]
    z = irwin_hall(seed, S_CNN, cid, 2)
    ratio = side / 224.0
    p = t * (ratio * ratio) * exp_det(3.0 + 0.5 * z)                  # lognormal(3, 0.5)
    nh = 16 if n_extra else 8
    w = [uniform(seed, S_CNN, cid, 20 + 2 * j) + uniform(seed, S_CNN, cid, 21 + 2 * j)
         for j in range(nh)]
    wsum = np.zeros_like(p)
    for j in range(nh):
        wsum = wsum + w[j]
    h = [p * (w[j] / wsum) for j in range(nh)]
    out = dict(t=t, p=p, h=h, side=side)
    if n_extra:
        out["layers"] = np.floor(8.0 + uniform(seed, S_CNN, cid, 60) * 1034.0)   # 8..1041
        out["neurons"] = log_uniform(uniform(seed, S_CNN, cid, 61), 6.5e5, 1.05e9)
    return out


def _gpu_cols(seed, gid, extra=False):
    sms = 5.0 + np.floor(uniform(seed, S_GPU, gid, 0) * 156.0)          # [5, 160]
    clk = 1000.0 + np.floor(uniform(seed, S_GPU, gid, 1) * 1001.0)      # MHz
    bw = log_uniform(uniform(seed, S_GPU, gid, 2), 80.0, 8000.0)        # GB/s
    l2 = log_uniform(uniform(seed, S_GPU, gid, 3), 1.0, 128.0)          # MB
    mem = np.asarray(MEM_GB)[(hash64(seed, S_GPU, gid, 4) % np.uint64(len(MEM_GB))).astype(np.int64)]
    cps = np.where((hash64(seed, S_GPU, gid, 5) & np.uint64(1)) == 0, 64.0, 128.0)
    out = dict(sms=sms, clk=clk, bw=bw, l2=l2, mem=mem, cps=cps)
    if extra:
        out["boost"] = clk + np.floor(uniform(seed, S_GPU, gid, 6) * 500.0)
        out["regs"] = np.where((hash64(seed, S_GPU, gid, 7) & np.uint64(1)) == 0, 65536.0, 131072.0)
        out["smem"] = 64.0 + np.floor(uniform(seed, S_GPU, gid, 8) * 165.0)
        out["tdp"] = 50.0 + np.floor(uniform(seed, S_GPU, gid, 9) * 951.0)
        out["tflops"] = sms * out["cps"] * 2.0 * out["boost"] * 1e-6
    return out


def _assemble(cnn, gpu, extra):
    cols = [cnn["t"], cnn["p"], *cnn["h"][:8], gpu["sms"], gpu["clk"], gpu["bw"], gpu["l2"],
            gpu["mem"], gpu["cps"]]
    if extra:
        cols += [cnn["layers"], cnn["neurons"], cnn["side"], *cnn["h"][8:16], gpu["boost"],
                 gpu["regs"], gpu["smem"], gpu["tdp"], gpu["tflops"]]
    return np.stack([np.asarray(c, dtype=np.float64).astype(np.float32) for c in cols], axis=1)


def latency_target(X, noise_z, real: bool, unit_us: float = 1.0):
    """Synthetic performance target from the (f32) features: roofline-style latency
    max(compute, memory) * (1 + 0.05 z) in units of ``unit_us`` microseconds; integer
    (ceil) unless ``real``.  Column layout as in ``cnn_gpu_table``."""
    Xd = X.astype(np.float64)
    t, p = Xd[:, 0], Xd[:, 1]
    sms, clk, bw = Xd[:, 10], Xd[:, 11], Xd[:, 12]
    compute = p / (((sms * clk) * 1e6) * 4.0)          # ipc_max = 4
    memory = (4.0 * t) / (bw * 1e9)
    lat = np.maximum(compute, memory) * (1.0 + 0.05 * noise_z)
    v = (lat * 1e6) / unit_us
    return v if real else np.ceil(v)


def cnn_gpu_table(seed: int, n: int, d: int = 16, real: bool = False, row0: int = 0,
                  cnn_pool_bits: int = 16, gpu_pool_bits: int = 8, unit_us: float = 1.0):
    """Rows = (CNN, GPU) pairs drawn from pools of 2^cnn_pool_bits CNNs x 2^gpu_pool_bits
    GPUs (realistic ties).  d = 16 (schema S16) or 32 (S32).  Returns X (n x d f32,
    row-major) and y (n f64)."""
    if d not in (16, 32):
        raise ValueError("d must be 16 or 32")
    rows = np.arange(row0, row0 + n, dtype=np.uint64)
    cid = hash64(seed, S_ROWCNN, rows, 0) % np.uint64(1 << cnn_pool_bits)
    gid = hash64(seed, S_ROWGPU, rows, 0) % np.uint64(1 << gpu_pool_bits)
    extra = d == 32
    X = _assemble(_cnn_cols(seed, cid, extra), _gpu_cols(seed, gid, extra), extra)
    z = irwin_hall(seed, S_ROWNOISE, rows, 0)
    y = latency_target(X, z, real, unit_us)
    return X, y


def dse_candidates(seed: int, row0: int, n: int, cnn_bits: int = 20, gpu_bits: int = 10):
    """DSE sweep (BASELINE configs[3]): the full cross product of 2^cnn_bits CNNs x
    2^gpu_bits GPU configs; candidate r = (cnn = r >> gpu_bits, gpu = r & mask).
    Returns X (n x 16 f32) for candidates [row0, row0+n)."""
    rows = np.arange(row0, row0 + n, dtype=np.uint64)
    cid = rows >> np.uint64(gpu_bits)
    gid = rows & np.uint64((1 << gpu_bits) - 1)
    return _assemble(_cnn_cols(seed, cid), _gpu_cols(seed, gid), False)


def dse_tables(seed: int, cnn_row0: int, n_cnn: int, n_gpu: int):
    """The factors of the DSE cross product (factored predict, include/dt.h
    dt_predict_dse): CNN pool rows cnn_row0 .. cnn_row0 + n_cnn - 1 (the 10 CNN-side S16
    columns) and GPU pool rows 0 .. n_gpu - 1 (the 6 GPU-side columns), plus feature_src
    (S16 column f -> CNN column f for f < 10, GPU column f - 10 as -1 - (f - 10)).
    Candidate (i, j) composes to dse_candidates(seed, ((cnn_row0 + i) << b) + j, 1, b)
    for n_gpu == 2^b."""
    cid = np.arange(cnn_row0, cnn_row0 + n_cnn, dtype=np.uint64)
    gid = np.arange(n_gpu, dtype=np.uint64)
    cnn = _assemble(_cnn_cols(seed, cid), _gpu_cols(seed, np.zeros(n_cnn, dtype=np.uint64)), False)[:, :10]
    gpu = _assemble(_cnn_cols(seed, np.zeros(n_gpu, dtype=np.uint64)), _gpu_cols(seed, gid), False)[:, 10:]
    src = list(range(10)) + [-1 - g for g in range(6)]
    return np.ascontiguousarray(cnn), np.ascontiguousarray(gpu), src


def holdout_mask(seed: int, n: int):
    """Reading R11: row r is held out for evaluation iff h(seed, r) mod 10 < 3 (~30%)."""
    rows = np.arange(n, dtype=np.uint64)
    return (hash64(seed, S_SPLIT, rows, 0) % np.uint64(10)) < np.uint64(3)


# --------------------------------------------------------------- paper-sized table ----

# Table I, first 20 models: (name, input side, trainable parameters).
TABLE_I_20 = (
    ("BiT-m-r50x1", 224, 25549552), ("BiT-m-r50x3", 224, 217319080),
    ("BiT-m-r101x3", 224, 387934888), ("BiT-m-r101x1", 224, 44541480),
    ("BiT-m-r154x4", 224, 936533224), ("resnet101", 224, 44601832),
    ("resnet152", 224, 60268520), ("resnet50v2", 224, 25568360),
    ("resnet101v2", 224, 44577896), ("resnet152v2", 224, 60236904),
    ("nasnetmobile", 224, 5289978), ("nasnetlarge", 331, 88753150),
    ("densenet121", 224, 7978856), ("densenet169", 224, 14149480),
    ("densenet201", 224, 20013928), ("mobilenet", 224, 4231976),
    ("inceptionv3", 299, 23817352), ("vgg16", 224, 138357544),
    ("vgg19", 224, 143667240), ("efficientnetb0", 224, 5288548),
)
# The two training GPUs: public specs (not in the paper): (mem BW GB/s, SMs, MHz).
TRAIN_GPUS = (("V100S", 1134.0, 80.0, 1245.0), ("GTX1080Ti", 484.0, 28.0, 1480.0))


def paper_table(seed: int = 0, real: bool = False):
    """BASELINE configs[0]: 40 rows = 20 Table I CNNs x {V100S, GTX 1080Ti}, d = 4 columns
    [p, memBW, SMs, t] (Eq. 1 order p, c_1..c_m, t).  y = latency in integer us (or real
    IPC-like latency when ``real``)."""
    X = np.zeros((40, 4), dtype=np.float32)
    y = np.zeros(40, dtype=np.float64)
    for ci, (_, side, t) in enumerate(TABLE_I_20):
        z = irwin_hall(seed, S_CNN, np.array([ci], dtype=np.uint64), 2)[0]
        ratio = side / 224.0
        p = float(t) * (ratio * ratio) * float(exp_det(3.0 + 0.5 * z))
        for gi, (_, bw, sms, clk) in enumerate(TRAIN_GPUS):
            r = 2 * ci + gi
            X[r] = (p, bw, sms, float(t))
            pf, tf = float(X[r, 0]), float(X[r, 3])
            zz = float(irwin_hall(seed, S_ROWNOISE, np.array([r], dtype=np.uint64), 0)[0])
            lat = max(pf / (sms * clk * 1e6 * 4.0), 4.0 * tf / (bw * 1e9)) * (1.0 + 0.05 * zz)
            y[r] = lat * 1e6 if real else math.ceil(lat * 1e6)
    return X, y


# --------------------------------------------------------------- generic test tables ----

def random_table(seed: int, n: int, d: int, kind: str = "continuous", int_y: bool = True,
                 y_range: int = 20):
    """Generic seeded test tables.

    kind: "continuous" (distinct f32 values), "ties" (small-integer features, many ties),
    "mixed" (half tied columns), "collinear" (duplicated / affinely dependent columns, as
    GPU descriptor columns are when only a few GPUs are in the pool).
    """
    rng = np.random.default_rng(seed)
    if kind == "continuous":
        X = rng.standard_normal((n, d)).astype(np.float32)
    elif kind == "ties":
        X = rng.integers(0, 4, size=(n, d)).astype(np.float32)
    elif kind == "mixed":
        X = rng.standard_normal((n, d)).astype(np.float32)
        X[:, ::2] = rng.integers(0, 5, size=(n, (d + 1) // 2)).astype(np.float32)
    elif kind == "collinear":
        base = rng.integers(0, 6, size=(n, max(1, d // 2))).astype(np.float32)
        X = np.concatenate([base, base * 2.0 + 1.0], axis=1)[:, :d]
        if X.shape[1] < d:
            X = np.concatenate([X, base[:, :1]], axis=1)
        X = np.ascontiguousarray(X[:, :d], dtype=np.float32)
    else:
        raise ValueError(kind)
    if int_y:
        y = rng.integers(0, y_range, size=n).astype(np.float64)
    else:
        y = rng.standard_normal(n) * 3.0 + 10.0
    return np.ascontiguousarray(X), y
