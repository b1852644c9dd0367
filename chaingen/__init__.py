"""Seeded synthetic layer-chain generator (shared by tests, bench and oracle runs).

This module holds NONE of the MadPipe method's arithmetic (no prefix sums, no
memory model, no DP): it only draws layer profiles -- per-layer forward and
backward durations u_F, u_B (seconds), weight sizes W (bytes) and activation
sizes a (bytes, a[0] = network input) -- shaped like the networks of the
paper's evaluation (ResNet-50, Inception at 1000x1000 images, batch 8)
and like the BASELINE.json configs.  The recipe is stated in DESIGN.md
section 4.  Every draw is seeded (numpy PCG64).

A chain is a dict  {"uF": float64[L], "uB": float64[L], "W": int64[L],
"a": int64[L+1], "name": str}.
"""
from __future__ import annotations

import hashlib
import math

import numpy as np

BATCH = 8            # mini-batch size of the paper's experiments
IMG = 1000           # image side
FP32 = 4
CONV_FLOPS = 10e12   # effective conv throughput used to turn MACs into time
ELEM_BW = 900e9      # bytes/s for element-wise / pooling layers


def _finish(name, uF, uB, W, a):
    ch = {"name": name,
          "uF": np.asarray(uF, np.float64), "uB": np.asarray(uB, np.float64),
          "W": np.asarray(W, np.int64), "a": np.asarray(a, np.int64)}
    L = len(ch["uF"])
    assert len(ch["uB"]) == L and len(ch["W"]) == L and len(ch["a"]) == L + 1
    assert np.all(ch["uF"] > 0) and np.all(ch["uB"] > 0)
    return ch


def digest(ch) -> str:
    """Stable content hash of a chain (used to detect generator drift)."""
    h = hashlib.sha256()
    for key in ("uF", "uB", "W", "a"):
        h.update(np.ascontiguousarray(ch[key]).tobytes())
    return h.hexdigest()[:16]


# --------------------------------------------------------------------------
# CNN helper: a list of layer descriptors -> profile
# --------------------------------------------------------------------------
class _CNN:
    def __init__(self, rng, c_in=3, hw=IMG, noise_f=0.15, noise_b=0.10):
        self.rng = rng
        self.c, self.h = c_in, hw
        self.uF, self.uB, self.W = [], [], []
        self.a = [BATCH * c_in * hw * hw * FP32]   # a_0 = input images
        self.noise_f, self.noise_b = noise_f, noise_b

    def _push(self, macs, w_elems, c_out, h_out, elem=False):
        if elem:
            t = 2.0 * self.a[-1] / ELEM_BW
        else:
            t = 2.0 * BATCH * macs / CONV_FLOPS
        t = max(t, 1e-5) * self.rng.lognormal(0.0, self.noise_f)
        self.uF.append(t)
        self.uB.append(2.0 * t * self.rng.lognormal(0.0, self.noise_b))
        self.W.append(int(w_elems) * FP32)
        self.c, self.h = c_out, h_out
        self.a.append(BATCH * c_out * h_out * h_out * FP32)

    def conv(self, c_out, k, stride=1, kw=None, extra_w=0, extra_macs=0):
        kw = k if kw is None else kw
        h_out = max(1, -(-self.h // stride))
        macs = h_out * h_out * c_out * self.c * k * kw + extra_macs
        self._push(macs, c_out * self.c * k * kw + c_out + extra_w, c_out, h_out)

    def pool(self, stride=2, c_out=None):
        h_out = max(1, -(-self.h // stride))
        self._push(0, 0, self.c if c_out is None else c_out, h_out, elem=True)

    def elem(self, c_out=None):
        self._push(0, 0, self.c if c_out is None else c_out, self.h, elem=True)

    def fc(self, n_out):
        macs = self.c * self.h * self.h * n_out
        self._push(macs, self.c * self.h * self.h * n_out + n_out, n_out, 1)

    def chain(self, name):
        return _finish(name, self.uF, self.uB, self.W, self.a)


def resnet50(seed: int = 2):
    """ResNet-50-shaped chain at 1000x1000, batch 8, fp32: 56 layers."""
    n = _CNN(np.random.default_rng(seed))
    n.conv(64, 7, 2)           # stem: 8*64*500*500*4 B = 512 MB output
    n.pool(2)
    for stage, (mid, out, blocks, stride) in enumerate(
            [(64, 256, 3, 1), (128, 512, 4, 2), (256, 1024, 6, 2), (512, 2048, 3, 2)]):
        c_in, h_in = n.c, n.h
        # projection shortcut as its own linearised layer (greedy grouping);
        # its output activation carries the block input and the shortcut result
        n.conv(out, 1, stride)
        n.a[-1] = BATCH * (c_in * h_in * h_in + out * n.h * n.h) * FP32
        n.c, n.h = c_in, h_in
        for b in range(blocks):
            s = stride if b == 0 else 1
            n.conv(mid, 1, 1)
            n.conv(mid, 3, s)
            n.conv(out, 1, 1)
    n.pool(n.h)                # global average pool
    n.fc(1000)
    return n.chain("resnet50")


def vgg19(seed: int = 4):
    """VGG-19-shaped chain (conv and ReLU as separate layers): 43 layers."""
    n = _CNN(np.random.default_rng(seed))
    for c, reps in [(64, 2), (128, 2), (256, 4), (512, 4), (512, 4)]:
        for _ in range(reps):
            n.conv(c, 3, 1)
            n.elem()
        n.pool(2)
    n.pool(max(1, n.h // 7))   # adaptive pool to 7x7
    n.fc(4096); n.elem()
    n.fc(4096); n.elem()
    n.fc(1000)
    return n.chain("vgg19")


def inception_v3(seed: int = 3):
    """Inception-v3-shaped chain; each module's branches linearised: 109 layers."""
    n = _CNN(np.random.default_rng(seed))
    n.conv(32, 3, 2); n.conv(32, 3, 1); n.conv(64, 3, 1); n.pool(2)
    n.conv(80, 1, 1); n.conv(192, 3, 1); n.pool(2)

    def module(branches, c_out, stride=1):
        # branches: list of lists of (c, k, kw); activations inside the module
        # carry the module input plus the branch outputs produced so far.
        c_in, h_in = n.c, n.h
        acc = 0
        for br in branches:
            n.c, n.h = c_in, h_in
            for j, (c, k, kw) in enumerate(br):
                last = j == len(br) - 1
                s = stride if (last and stride > 1) else 1
                if c == 0:
                    n.pool(s)
                else:
                    n.conv(c, k, s, kw)
                if last:
                    acc += n.c
            # the linearised chain keeps input + partial concat alive
            n.a[-1] = BATCH * (c_in + acc) * n.h * n.h * FP32
        n.c = c_out
        n.a[-1] = BATCH * c_out * n.h * n.h * FP32

    for pool_c in (32, 64, 64):                              # 3 x InceptionA
        module([[(64, 1, 1)], [(48, 1, 1), (64, 5, 5)], [(64, 1, 1), (96, 3, 3), (96, 3, 3)],
                [(0, 3, 3), (pool_c, 1, 1)]], 224 + pool_c)
    module([[(384, 3, 3)], [(64, 1, 1), (96, 3, 3), (96, 3, 3)], [(0, 3, 3)]], 768, stride=2)
    for c7 in (128, 160, 160, 192):                          # 4 x InceptionC
        module([[(192, 1, 1)], [(c7, 1, 1), (c7, 1, 7), (192, 7, 1)],
                [(c7, 1, 1), (c7, 7, 1), (c7, 1, 7), (c7, 7, 1), (192, 1, 7)],
                [(0, 3, 3), (192, 1, 1)]], 768)
    module([[(192, 1, 1), (320, 3, 3)], [(192, 1, 1), (192, 1, 7), (192, 7, 1), (192, 3, 3)],
            [(0, 3, 3)]], 1280, stride=2)
    for _ in range(2):                                       # 2 x InceptionE
        module([[(320, 1, 1)], [(384, 1, 1), (384, 1, 3), (384, 3, 1)],
                [(448, 1, 1), (384, 3, 3), (384, 1, 3), (384, 3, 1)],
                [(0, 3, 3), (192, 1, 1)]], 2048)
    n.pool(n.h)
    n.fc(1000)
    return n.chain("inception_v3")


def gpt(seed: int = 5, L: int = 256, H: int = 4096, seq: int = 2048, mbs: int = 8,
        vocab: int = 50304, flops: float = 400e12):
    """GPT-style chain: embedding + (L-2) transformer blocks + LM head, bf16."""
    rng = np.random.default_rng(seed)
    tokens = mbs * seq
    act = tokens * H * 2                                    # 134 MB per block output
    t_blk = 2.0 * tokens * (12 * H * H + 2 * seq * H) / flops   # ~17.8 ms
    uF, W = [], []
    a = [tokens * 8]                                        # int64 token ids
    uF.append(tokens * H * 2 / 3e12); W.append(vocab * H * 2); a.append(act)     # embedding
    for _ in range(L - 2):
        uF.append(t_blk); W.append(12 * H * H * 2); a.append(act)
    uF.append(2.0 * tokens * H * vocab / flops); W.append(vocab * H * 2); a.append(tokens * vocab * 2)
    uF = np.asarray(uF) * rng.lognormal(0.0, 0.05, size=L)
    uB = 2.0 * uF
    return _finish("gpt%d" % L, uF, uB, W, a)


def random_chain(seed: int, L: int | None = None):
    """One chain of the C5 batch: CNN-like (activations halve every L/5 layers)
    or flat, with probability 1/2 each."""
    rng = np.random.default_rng(seed)
    if L is None:
        L = int(rng.integers(32, 513))
    cnn = rng.random() < 0.5
    uF = rng.lognormal(math.log(10e-3), 0.5, size=L)
    uB = 2.0 * uF * rng.lognormal(0.0, 0.1, size=L)
    if cnn:
        a0 = float(rng.uniform(100e6, 500e6))
        stage = np.minimum(np.arange(L + 1) * 5 // L, 4)
        a = a0 * 0.5 ** stage * rng.lognormal(0.0, 0.1, size=L + 1)
        W = 2e6 * 2.0 ** stage[1:] * rng.lognormal(0.0, 1.0, size=L)
    else:
        a = float(rng.uniform(50e6, 200e6)) * rng.lognormal(0.0, 0.1, size=L + 1)
        W = rng.lognormal(math.log(50e6), 0.3, size=L)
    return _finish("rand%d_%s" % (seed, "cnn" if cnn else "flat"), uF, uB,
                   np.round(W).astype(np.int64), np.round(a).astype(np.int64))


def random_batch_params(seed: int):
    """Per-chain P and beta of the C5 batch: P = round(exp U[ln 4, ln 128]),
    beta ~ logU[5, 100] GB/s, memory factor U[0.5, 1]."""
    rng = np.random.default_rng(10_000 + seed)
    P = int(round(math.exp(rng.uniform(math.log(4), math.log(128)))))
    beta = math.exp(rng.uniform(math.log(5e9), math.log(100e9)))
    mfac = float(rng.uniform(0.5, 1.0))
    return P, beta, mfac


def toy(seed: int = 1, L: int = 8):
    """C1 toy chain: uF ~ U[0.5, 2] ms; uB = 2 uF U[0.8, 1.2]; W ~ U{1..20} MB;
    a ~ U{5..60} MB including a_0."""
    rng = np.random.default_rng(seed)
    uF = rng.uniform(0.5e-3, 2e-3, size=L)
    uB = 2.0 * uF * rng.uniform(0.8, 1.2, size=L)
    W = rng.integers(1, 21, size=L) * 1_000_000
    a = rng.integers(5, 61, size=L + 1) * 1_000_000
    return _finish("toy%d" % L, uF, uB, W, a)


def tiny(rng: np.random.Generator, L: int, integer_times: bool = False, mem_scale: float = 1.0,
         zero_mem: bool = False, a_hi: int = 40):
    """Small random chain for fuzz tests (brute force sizes).  ``a_hi`` bounds the
    activation sizes (exclusive); a large value with a small beta gives
    communication-bound chains (C(i) = 2 a_i / beta above the period)."""
    if integer_times:
        uF = rng.integers(1, 6, size=L).astype(np.float64)
        uB = rng.integers(1, 11, size=L).astype(np.float64)
    else:
        uF = rng.uniform(0.2, 2.0, size=L)
        uB = uF * rng.uniform(1.0, 3.0, size=L)
    if zero_mem:
        W = np.zeros(L, np.int64); a = np.zeros(L + 1, np.int64)
    else:
        W = (rng.integers(1, 20, size=L) * mem_scale).astype(np.int64)
        a = (rng.integers(1, a_hi, size=L + 1) * mem_scale).astype(np.int64)
    return _finish("tiny%d" % L, uF, uB, W, a)


def uniform(L: int, u: float = 1.0):
    """Uniform memory-free chain: uF = u/4, uB = 3u/4, so uF + uB = u exactly
    for small integer u; W = a = 0."""
    uF = np.full(L, u / 4.0)
    uB = np.full(L, 3.0 * u / 4.0)
    return _finish("uniform%d" % L, uF, uB, np.zeros(L, np.int64), np.zeros(L + 1, np.int64))


FAMILIES = {"toy": toy, "resnet50": resnet50, "vgg19": vgg19, "inception_v3": inception_v3,
            "gpt": gpt, "random": random_chain}


def make(spec: dict):
    """Build a chain from a config's ``chain`` spec: {"family": ..., "seed": ..., **kw}."""
    spec = dict(spec)
    fam = spec.pop("family")
    return FAMILIES[fam](**spec)
