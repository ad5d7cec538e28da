"""GPU execution of the paper's operator splitting (TG_PER_OP, reading R19):
graphs whose operators do not fit the budget run piece by piece with the generic kernels, and
  * the result matches the CPU oracle / the numpy evaluation of the unsplit graph (1e-5
    normwise, reading R16);
  * it is bit-identical to the same graph run unsplit (uncapped budget) -- the halo bands, the
    2-D piece copies and the piece views change no value;
  * the executed schedule is the planned one (launch count = piece operators);
  * matmul split by rows of A and C matches orc_matmul."""
import numpy as np
import pytest

import synth
from gpu_util import need_gpu, normwise, torch
from split_graphs import cnn_spec, edge_spec, lib_graph, mixed_spec, run_unsplit

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def tg():
    need_gpu()
    from paper_conf_ipps_sundaramrc09_b200 import tg as t
    torch.cuda.set_device(0)
    return t


def execute(tg, spec, budget, mode=None):
    out = np.full(spec.shapes[spec.output], np.nan, np.float32)
    g = lib_graph(spec, out, budget=budget, torch_runtime=True)
    p = g.plan(tg.TG_PER_OP if mode is None else mode)
    p.execute()
    return out, p


@pytest.mark.parametrize("frac", [0.5, 0.2, 0.08])
def test_edge_split_gpu(tg, orc, frac):
    K1, K2 = synth.random_edge_filters_np(7)
    spec = edge_spec(301, 64, K1, K2, n=2, rng=3)
    budget = int(spec.total_bytes() * frac) // 256 * 256
    out, p = execute(tg, spec, budget)
    j = p.json()
    assert max(j["k"].values()) > 1
    assert p.launches() == len(j["ops"])
    want = np.stack([orc.edge(spec.data[0][i, 0], K1, K2) for i in range(2)])
    assert normwise(out[:, 0], want) <= 1e-5
    full, _ = execute(tg, spec, 0)
    assert np.array_equal(out, full)


@pytest.mark.parametrize("frac", [0.3, 0.2])
def test_cnn_split_gpu(tg, orc, frac):
    H, W, n5 = 77, 41, 4
    prm = synth.cnn_params_np(11, n5, H, W)
    spec = cnn_spec(1, H, W, n5, prm)
    out, p = execute(tg, spec, int(spec.total_bytes() * frac) // 256 * 256)
    assert max(p.json()["k"].values()) > 1
    assert normwise(out, orc.cnn(spec.data[0], n5, prm)) <= 1e-5
    full, _ = execute(tg, spec, 0)
    assert np.array_equal(out, full)


@pytest.mark.parametrize("frac", [0.4, 0.1])
def test_mixed_split_gpu(tg, frac):
    spec = mixed_spec(83, 30, 7)
    out, p = execute(tg, spec, int(spec.total_bytes() * frac) // 256 * 256)
    assert max(p.json()["k"].values()) > 1
    assert normwise(out, run_unsplit(spec)) <= 1e-5
    full, _ = execute(tg, spec, 0)
    assert np.array_equal(out, full)


def test_large_edge_split_gpu(tg, orc):
    """One 3000 x 2000 image through a 16 MiB budget: every operator split into 9 pieces."""
    K1, K2 = synth.random_edge_filters_np(9)
    img = synth.images_np(synth.seed_for_config(1), 1, 3000, 2000)
    spec = edge_spec(3000, 2000, K1, K2, img=img)
    out, p = execute(tg, spec, 16 << 20)
    assert max(p.json()["k"].values()) >= 8
    assert normwise(out[0], orc.edge(img[0, 0], K1, K2)[None]) <= 1e-5


@pytest.mark.parametrize("m,k,n,budget", [(1000, 512, 300, 1 << 20), (777, 129, 65, 200_000), (64, 64, 64, 0)])
def test_matmul_split_gpu(tg, orc, m, k, n, budget):
    rng = np.random.default_rng(m)
    A = rng.standard_normal((1, 1, m, k)).astype(np.float32)
    B = rng.standard_normal((1, 1, k, n)).astype(np.float32)
    C = np.full((1, 1, m, n), np.nan, np.float32)
    g = tg.Graph()
    a = g.input(A)
    b = g.param(B)
    y = g.matmul(a, b)
    g.output(y, C)
    g.set(budget=budget, torch_runtime=True)
    p = g.plan(tg.TG_PER_OP)
    p.execute()
    if budget:
        assert max(p.json()["k"].values()) > 1
        assert [pc[1:] for pc in p.json()["pieces"] if pc[0] == b] == [[0, k]]   # B whole
    ref = orc.matmul(A[0, 0], B[0, 0])
    assert normwise(C[0], ref[None]) <= 1e-5


def test_matmul_baseline_and_chain(tg, orc):
    """matmul of a split intermediate read whole: tanh(X) (split into pieces) feeds the B
    operand of a matmul whose every piece reads all of tanh(X)'s pieces."""
    rng = np.random.default_rng(5)
    A = rng.standard_normal((1, 1, 300, 96)).astype(np.float32)
    X = rng.standard_normal((1, 1, 96, 800)).astype(np.float32)
    C = np.zeros((1, 1, 300, 800), np.float32)
    g = tg.Graph()
    a = g.input(A)
    x = g.input(X)
    t = g.tanh(x)
    y = g.matmul(a, t)
    g.output(y, C)
    g.set(budget=600_000, torch_runtime=True)
    p = g.plan(tg.TG_PER_OP)
    assert p.json()["k"] == {"0": 2, "1": 5}
    p.execute()
    T = orc.tanh(X[0, 0])
    assert normwise(C[0], orc.matmul(A[0, 0], T)[None]) <= 1e-5
    C2 = np.zeros_like(C)
    g2 = tg.Graph()
    g2.output(g2.matmul(g2.input(A), g2.tanh(g2.input(X))), C2)
    g2.set(torch_runtime=True)
    g2.plan(tg.TG_BASELINE).execute()
    assert np.array_equal(C, C2)


def test_tanh_fp32_accuracy(tg):
    """The fp32 paths' tanh (kernels/tanh_fp32.cuh, via the operator library): within a few
    fp32 ulps of tanh RELATIVE to the result over [-9, 9], incl. values near 0 where the
    one-branch 1 - 2/(1 + e^2x) cancels."""
    x = np.concatenate([np.linspace(-9, 9, 400_001), np.geomspace(1e-30, 0.7, 100_000),
                        -np.geomspace(1e-30, 0.7, 100_000), [0.0, 0.6, -0.6, 0.59999996]]).astype(np.float32)
    x = np.resize(x, 600 * 1001).reshape(1, 1, 600, 1001)
    out = np.zeros_like(x)
    g = tg.Graph()
    xi = g.input(x)
    g.output(g.tanh(xi), out)
    g.set(torch_runtime=True)
    g.plan(tg.TG_PER_OP).execute()
    ref = np.tanh(x.astype(np.float64))
    rel = np.abs(out - ref) / np.maximum(np.abs(ref), 1e-38)
    assert rel.max() <= 3e-7, (rel.max(), x.ravel()[rel.argmax()])
