"""Pins for the oracle's noise and Gumbel-softmax (§4.4; reading Q1, Q7).

The oracle is pinned against things other than itself: published Philox known-answer
vectors, the CUDA toolkit's own Philox (compiled for the host), the Gumbel distribution's
moments, a library softmax (torch) in the noise-free case, and softmax invariances.
"""
import os
import subprocess
import tempfile

import numpy as np
import pytest
import torch

import oracle
from tests import _ref

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _kat_rows():
    rows = []
    for line in open(os.path.join(GOLDEN, "philox_kat.txt")):
        if line.startswith("#") or not line.strip():
            continue
        v = [int(x, 16) for x in line.split()]
        rows.append((v[0:4], v[4:6], v[6:10]))
    return rows


@pytest.mark.parametrize("ctr,key,out", _kat_rows())
def test_philox_known_answers(ctr, key, out):
    assert list(oracle.philox4x32_10(ctr, key)) == out


def test_philox_matches_cuda_toolkit_header():
    """Random counters/keys vs curand_Philox4x32_10 from the CUDA toolkit header, built for the host."""
    src = r'''
#define QUALIFIERS static inline __host__ __device__
#include <cstdio>
#include <cuda_runtime.h>
#include <curand_philox4x32_x.h>
int main(){ unsigned a,b,c,d,e,f;
 while(scanf("%x %x %x %x %x %x",&a,&b,&c,&d,&e,&f)==6){
  uint4 r=curand_Philox4x32_10(make_uint4(a,b,c,d),make_uint2(e,f));
  printf("%08x %08x %08x %08x\n",r.x,r.y,r.z,r.w);} }
'''
    with tempfile.TemporaryDirectory() as td:
        cu, exe = os.path.join(td, "k.cu"), os.path.join(td, "k")
        open(cu, "w").write(src)
        try:
            subprocess.check_call(["nvcc", "-Wno-deprecated-gpu-targets", "-o", exe, cu],
                                  stdout=subprocess.DEVNULL, stderr=subprocess.DEVNULL)
        except (OSError, subprocess.CalledProcessError):
            pytest.skip("nvcc host build unavailable")
        rng = np.random.default_rng(7)
        vals = rng.integers(0, 2**32, size=(64, 6), dtype=np.uint64)
        inp = "\n".join(" ".join("%x" % v for v in row) for row in vals) + "\n"
        out = subprocess.run([exe], input=inp, capture_output=True, text=True, check=True).stdout.split("\n")
        for row, line in zip(vals, out):
            ref = [int(x, 16) for x in line.split()]
            assert list(oracle.philox4x32_10(row[:4], row[4:6])) == ref


def test_uniform_is_open_interval_and_fp32_exact():
    u = np.array([oracle.uniform(0xD6A5EED, i, k, s) for i in range(512) for k in (0, 7) for s in (0, 1)])
    assert (u > 0).all() and (u < 1).all()
    assert (u.astype(np.float32).astype(np.float64) == u).all()   # exactly representable in fp32
    assert abs(u.mean() - 0.5) < 0.03


def test_uniform_uses_word_idx_and_3_of_one_philox_call():
    seed = 0x1234_5678_9ABC
    for base in (0, 4, 4 * 1000003):
        r = oracle.philox4x32_10([base >> 2, 0, 5, 0], [seed & 0xFFFFFFFF, seed >> 32])
        for w in range(4):
            assert oracle.uniform(seed, base + w, 5, 0) == ((int(r[w]) >> 9) + 0.5) / 2**23


def test_gumbel_moments():
    """Gumbel(0,1): mean = Euler-Mascheroni gamma, variance = pi^2/6."""
    g = np.array([oracle.gumbel(99, i, 3, 0) for i in range(60000)])
    assert abs(g.mean() - 0.5772156649) < 0.02
    assert abs(g.var() - np.pi ** 2 / 6) < 0.05


def test_group_sums_are_one(tiny):
    o = oracle.Oracle(tiny)
    o.forward(0.7, oracle.weights())
    q, p = o.probs()
    for s in range(tiny.n_subnets):
        a, b = tiny.sub_path_off[s], tiny.sub_path_off[s + 1]
        assert abs(p[a:b].sum() - 1) < 1e-12
    for n in range(tiny.n_nets):
        a, b = tiny.net_tree_off[n], tiny.net_tree_off[n + 1]
        assert abs(q[a:b].sum() - 1) < 1e-12


def test_noise_free_t1_is_textbook_softmax(tiny):
    """With g = 0 and t = 1 the relaxation is softmax over each sub-net / net (reading Q1)."""
    o = oracle.Oracle(tiny)
    o.forward(1.0, oracle.weights(), noise=False)
    q, p = o.probs()
    w = torch.tensor(tiny.w_path0, dtype=torch.float64)
    for s in range(tiny.n_subnets):
        a, b = tiny.sub_path_off[s], tiny.sub_path_off[s + 1]
        np.testing.assert_allclose(p[a:b], torch.softmax(w[a:b], 0).numpy(), rtol=1e-14, atol=0)
    wt = torch.tensor(tiny.w_tree0, dtype=torch.float64)
    for n in range(tiny.n_nets):
        a, b = tiny.net_tree_off[n], tiny.net_tree_off[n + 1]
        np.testing.assert_allclose(q[a:b], torch.softmax(wt[a:b], 0).numpy(), rtol=1e-14, atol=0)


def test_noisy_softmax_uses_the_candidate_noise(tiny):
    """p_i = softmax((w + g)/t) with g_i = -ln(-ln u_i) of candidate i, iteration k, stream 0."""
    o = oracle.Oracle(tiny)
    o.iteration = 11
    t = 0.37
    o.forward(t, oracle.weights())
    q, p = o.probs()
    g = _ref.path_noise(tiny, 11)
    gt = np.array([oracle.gumbel(tiny.seed, j, 11, 1) for j in range(tiny.n_trees)])
    z = torch.tensor((tiny.w_path0.astype(np.float64) + g) / t)
    zt = torch.tensor((tiny.w_tree0.astype(np.float64) + gt) / t)
    for s in range(tiny.n_subnets):
        a, b = tiny.sub_path_off[s], tiny.sub_path_off[s + 1]
        np.testing.assert_allclose(p[a:b], torch.softmax(z[a:b], 0).numpy(), rtol=1e-12)
    for n in range(tiny.n_nets):
        a, b = tiny.net_tree_off[n], tiny.net_tree_off[n + 1]
        np.testing.assert_allclose(q[a:b], torch.softmax(zt[a:b], 0).numpy(), rtol=1e-12)


def test_shift_invariance(tiny):
    o1, o2 = oracle.Oracle(tiny), oracle.Oracle(tiny)
    wt, wp = o1.logits()
    rng = np.random.default_rng(3)
    shift_p = np.repeat(rng.normal(size=tiny.n_subnets) * 5, np.diff(tiny.sub_path_off))
    shift_t = np.repeat(rng.normal(size=tiny.n_nets) * 5, np.diff(tiny.net_tree_off))
    o2.set_logits(wt + shift_t, wp + shift_p)
    o1.forward(0.5, oracle.weights()); o2.forward(0.5, oracle.weights())
    for a, b in zip(o1.probs(), o2.probs()):
        np.testing.assert_allclose(a, b, rtol=1e-9, atol=1e-15)


def test_low_temperature_is_argmax(tiny):
    """t -> 0 drives the relaxed selection to the argmax of w + g (the annealing intent)."""
    o = oracle.Oracle(tiny)
    o.forward(1e-4, oracle.weights())
    q, p = o.probs()
    g = _ref.path_noise(tiny, 0)
    z = tiny.w_path0.astype(np.float64) + g
    for s in range(tiny.n_subnets):
        a, b = tiny.sub_path_off[s], tiny.sub_path_off[s + 1]
        assert p[a + int(np.argmax(z[a:b]))] > 0.999
