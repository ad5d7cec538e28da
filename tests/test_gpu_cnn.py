"""GPU parity of the fused CNN units (U1, U2, U3; Fig. 7) against the CPU
oracle: normwise 1e-5 per output plane on the fp32 path (R16), split == unsplit
bit-exactly (rows with streamed bias rows, batches), device-resident == host-streamed, the
delta-kernel geometry (every output is tanh^5 of one input pixel), and sampled rows of the
paper-literal large CNN at 6400x4800 under the 1.5 GB budget."""
import math

import numpy as np
import pytest

import synth
from gpu_util import guard_runtime, need_gpu, normwise, pinned, torch

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def tg():
    need_gpu()
    from paper_conf_ipps_sundaramrc09_b200 import tg as t
    torch.cuda.set_device(0)
    return t


def run_cnn(tg, img, n5, prm, bias="plane", budget=0, device=False, max_chunk_px=None, depth=None,
            precision=None):
    n, _, H, W = img.shape
    h5, w5 = synth.cnn_dims(H, W)[4]
    mode = tg.TG_BIAS_PLANE if bias == "plane" else tg.TG_BIAS_SCALAR
    if device:
        x = torch.from_numpy(img).cuda()
        out = torch.zeros((n, 9, h5, w5), dtype=torch.float32, device="cuda")
        g, _ = tg.cnn_graph(x, n5, prm, out=out, bias_mode=mode, device=True)
    else:
        out = np.zeros((n, 9, h5, w5), np.float32)
        g, _ = tg.cnn_graph(img, n5, prm, out=out, bias_mode=mode)
    g.set(budget=budget, torch_runtime=True, max_chunk_px=max_chunk_px, depth=depth, precision=precision)
    p = g.plan()
    p.execute()
    return (out.cpu().numpy() if device else out), p


@pytest.mark.parametrize("n,H,W,n5,bias", [(2, 92, 100, 20, "plane"), (1, 120, 160, 120, "plane"),
                                          (3, 67, 61, 20, "scalar"), (1, 97, 131, 120, "scalar"),
                                          (1, 483 // 3, 643 // 3, 60, "plane"), (2, 32, 32, 7, "plane"),
                                          # wide rows (T4 pitch > 256): the U3 16 x 64 tile geometry
                                          (1, 70, 1210, 20, "plane"), (1, 45, 1333, 120, "scalar")])
def test_cnn_parity(tg, orc, n, H, W, n5, bias):
    seed = synth.seed_for_config(3)
    img = synth.images_np(seed, n, H, W)
    prm = synth.cnn_params_np(seed, n5, H, W, bias)
    out, _ = run_cnn(tg, img, n5, prm, bias)
    ref = orc.cnn(img, n5, prm, bias_plane=(bias == "plane"))
    assert normwise(out, ref) <= 1e-5


def test_cnn_vga_batch_both_nets(tg, orc):
    """configs[2] shape (480x640 planes), a small batch of it, both nets."""
    seed = synth.seed_for_config(3)
    img = synth.images_np(seed, 2, 480, 640)
    for n5 in (20, 120):
        prm = synth.cnn_params_np(seed, n5, 480, 640)
        out, p = run_cnn(tg, img, n5, prm)
        assert p.stats()["n_ops_fig7"] == (1600 if n5 == 20 else 7500)
        assert normwise(out, orc.cnn(img, n5, prm)) <= 1e-5


@pytest.mark.parametrize("budget,mcp", [(0, 20000), (2_000_000, None), (1_200_000, None)])
def test_cnn_split_equals_unsplit(tg, orc, budget, mcp):
    seed = 77
    n, H, W, n5 = 2, 200, 180, 40
    img = synth.images_np(seed, n, H, W)
    prm = synth.cnn_params_np(seed, n5, H, W)
    full, p0 = run_cnn(tg, img, n5, prm)
    split, p1 = run_cnn(tg, img, n5, prm, budget=budget, max_chunk_px=mcp)
    j = p1.json()
    assert j["n_chunks"] > p0.json()["n_chunks"]
    if budget:
        assert j["arena_bytes"] <= budget
    assert np.array_equal(split, full), j["bias"]
    assert normwise(full, orc.cnn(img, n5, prm)) <= 1e-5


def test_cnn_streamed_bias_rows(tg, orc):
    """A budget too small for the resident bias set forces bias rows to stream per chunk."""
    seed = 78
    img = synth.images_np(seed, 1, 300, 260)
    prm = synth.cnn_params_np(seed, 120, 300, 260)
    out, p = run_cnn(tg, img, 120, prm, budget=3_000_000)
    assert p.json()["bias"] == "streamed"
    full, _ = run_cnn(tg, img, 120, prm)
    assert np.array_equal(out, full)
    assert normwise(out, orc.cnn(img, 120, prm)) <= 1e-5


def test_cnn_device_io_equals_streamed(tg):
    seed = 79
    img = synth.images_np(seed, 3, 100, 120)
    prm = synth.cnn_params_np(seed, 20, 100, 120)
    a, _ = run_cnn(tg, img, 20, prm, device=True)
    b, _ = run_cnn(tg, img, 20, prm, budget=1_500_000)
    assert np.array_equal(a, b)


def _tanh32(v):
    return np.float32(math.tanh(float(v)))


def test_cnn_delta_geometry(tg):
    rng = np.random.default_rng(17)
    H, W, n5 = 83, 91, 20
    (h1, w1), _, (h3, w3), _, (h5, w5) = synth.cnn_dims(H, W)
    x = rng.random((1, 1, H, W)).astype(np.float32)
    a1, p2 = rng.integers(0, 5, (8, 2)), rng.integers(0, 2, (8, 2))
    a3, p4 = rng.integers(0, 5, (20, 2)), rng.integers(0, 2, (20, 2))
    a5 = rng.integers(0, 5, (n5, 2))
    K1 = np.zeros((8, 1, 5, 5), np.float32)
    P2 = np.zeros((8, 2, 2), np.float32)
    K3 = np.zeros((20, 8, 5, 5), np.float32)
    P4 = np.zeros((20, 2, 2), np.float32)
    K5 = np.zeros((n5, 20, 5, 5), np.float32)
    K6 = np.zeros((9, n5, 1, 1), np.float32)
    for j in range(8):
        K1[j, 0, a1[j, 0], a1[j, 1]] = 1
        P2[j, p2[j, 0], p2[j, 1]] = 1
    for j in range(20):
        K3[j, j % 8, a3[j, 0], a3[j, 1]] = 1
        P4[j, p4[j, 0], p4[j, 1]] = 1
    for j in range(n5):
        K5[j, j % 20, a5[j, 0], a5[j, 1]] = 1
    for j in range(9):
        K6[j, j % n5, 0, 0] = 1
    z = [np.zeros((1, c, h, w), np.float32) for c, (h, w) in [(8, (h1, w1)), (20, (h3, w3)), (n5, (h5, w5)), (9, (h5, w5))]]
    prm = [K1, z[0], P2, K3, z[1], P4, K5, z[2], K6, z[3]]
    out, _ = run_cnn(tg, x, n5, prm)
    exp = np.empty((9, h5, w5), np.float32)
    for j in range(9):
        i = j % n5
        m = i % 20
        l = m % 8
        for r in range(h5):
            for c in range(w5):
                R = 2 * (2 * (r + a5[i, 0]) + p4[m, 0] + a3[m, 0]) + p2[l, 0] + a1[l, 0]
                C = 2 * (2 * (c + a5[i, 1]) + p4[m, 1] + a3[m, 1]) + p2[l, 1] + a1[l, 1]
                v = x[0, 0, R, C]
                for _ in range(5):
                    v = _tanh32(v)
                exp[j, r, c] = v
    # exact gathers; only the five tanh evaluations round differently (|err| < 1e-6)
    assert np.abs(out[0] - exp).max() < 1e-6


@pytest.mark.parametrize("prec", ["fp32", "fp32_tc", "bf16_tc"])
def test_large_cnn_paper_size_sampled_rows(tg, orc, prec):
    """Paper-literal configs[3]: large CNN on one 6400x4800 image (17.66e9-float Fig. 7
    footprint) under the 1.5 GB budget: bias rows stream; sampled output rows
    at chunk boundaries match the oracle evaluated on each row's receptive band."""
    H, W, n5 = 4800, 6400, 120
    seed = synth.seed_for_config(4)
    img = synth.images_np(seed, 1, H, W)
    prm = synth.cnn_params_np(seed, n5, H, W)
    h5, w5 = synth.cnn_dims(H, W)[4]
    out, p = run_cnn(tg, img, n5, prm, budget=1536 << 20,
                     precision={"fp32": tg.TG_FP32, "fp32_tc": tg.TG_FP32_TC, "bf16_tc": tg.TG_BF16_TC}[prec])
    j = p.json()
    assert j["bias"] == "streamed" and j["arena_bytes"] <= 1536 << 20
    rows = {0, h5 - 1}
    for ch in j["chunks"][:3]:
        rows |= {ch["out"][0], ch["out"][1] - 1}
    for r in sorted(rows):
        band = np.ascontiguousarray(img[:, :, 4 * r:4 * r + 32])
        bp = list(prm)
        bp[1] = prm[1][:, :, 4 * r:4 * r + 28]
        bp[4] = prm[4][:, :, 2 * r:2 * r + 10]
        bp[7] = prm[7][:, :, r:r + 1]
        bp[9] = prm[9][:, :, r:r + 1]
        ref = orc.cnn(band, n5, bp)[0, :, 0]
        got = out[0, :, r]
        err = np.abs(got.astype(np.float64) - ref).max() / np.abs(ref).max()
        assert err <= (2e-2 if prec == "bf16_tc" else 1e-5), (r, err)


@pytest.mark.parametrize("prec", ["fp32", "bf16_tc", "fp32_tc"])
@pytest.mark.parametrize("n5", [1, 16, 128])
def test_cnn_n5_boundaries(tg, orc, n5, prec):
    """The smallest C5 width, exactly one 16-map chunk (no padding, one TMEM chunk, the degenerate
    one-buffer bias ring) and the largest (128 = the whole accumulator, no padding): every precision
    path against the oracle, two images spanning several U3 bands."""
    seed = synth.seed_for_config(3) + n5
    n, H, W = 2, 100, 130
    img = synth.images_np(seed, n, H, W)
    prm = synth.cnn_params_np(seed, n5, H, W, "plane")
    code = {"fp32": tg.TG_FP32, "bf16_tc": tg.TG_BF16_TC, "fp32_tc": tg.TG_FP32_TC}[prec]
    out, p = run_cnn(tg, img, n5, prm, "plane", precision=code)
    assert p.json()["precision"] == prec
    err = normwise(out, orc.cnn(img, n5, prm, bias_plane=True))
    assert err <= (2e-2 if prec == "bf16_tc" else 1e-5), err


# ------------------------------------------------------------------ tcgen05 bf16 path
@pytest.mark.parametrize("n,H,W,n5,bias", [(2, 92, 100, 20, "plane"), (1, 120, 160, 120, "plane"),
                                          (2, 480, 640, 120, "plane"), (1, 480, 640, 20, "scalar"),
                                          (1, 97, 1003, 120, "plane"), (1, 61, 67, 7, "plane"),
                                          (1, 140, 1400, 33, "scalar"), (2, 100, 300, 80, "plane"),
                                          (1, 60, 1500, 60, "plane"), (1, 200, 260, 120, "scalar")])
def test_cnn_bf16_tc_parity(tg, orc, n, H, W, n5, bias):
    """C3, C5 on tcgen05 (bf16 operands, fp32 accumulation): normwise <= 2e-2 (north_star);
    covers the flattened (narrow) and column-window (wide) band modes of U3."""
    seed = synth.seed_for_config(3) + 17
    img = synth.images_np(seed, n, H, W)
    prm = synth.cnn_params_np(seed, n5, H, W, bias)
    out, p = run_cnn(tg, img, n5, prm, bias, precision=tg.TG_BF16_TC)
    assert p.json()["precision"] == "bf16_tc"
    ref = orc.cnn(img, n5, prm, bias_plane=(bias == "plane"))
    err = normwise(out, ref)
    assert err <= 2e-2, err
    # and it really is the reduced-precision path (not the fp32 kernels)
    out32, _ = run_cnn(tg, img, n5, prm, bias)
    assert not np.array_equal(out, out32)


def test_cnn_bf16_tc_split_equals_unsplit(tg):
    seed = 91
    n, H, W, n5 = 2, 200, 180, 120
    img = synth.images_np(seed, n, H, W)
    prm = synth.cnn_params_np(seed, n5, H, W)
    full, p0 = run_cnn(tg, img, n5, prm, precision=tg.TG_BF16_TC)
    split, p1 = run_cnn(tg, img, n5, prm, budget=2_000_000, precision=tg.TG_BF16_TC)
    assert p1.json()["n_chunks"] > p0.json()["n_chunks"]
    assert np.array_equal(split, full)


# ------------------------------------------------------------------ 3xFP16 path (TG_FP32_TC)
@pytest.mark.parametrize("n,H,W,n5,bias", [(2, 92, 100, 20, "plane"), (1, 120, 160, 120, "plane"),
                                          (3, 67, 61, 20, "scalar"), (1, 97, 1003, 120, "plane"),
                                          (2, 36, 40, 7, "plane"), (2, 100, 300, 80, "plane"),
                                          (1, 60, 1500, 60, "scalar"), (1, 140, 1400, 33, "plane"),
                                          # the fp32 and bf16 lists' smallest cases: 1x1 output
                                          # planes (normwise = the relative error of ONE value)
                                          (2, 32, 32, 7, "plane"), (2, 32, 32, 20, "plane"),
                                          (1, 61, 67, 7, "plane"), (1, 483 // 3, 643 // 3, 60, "plane")])
def test_cnn_fp32_tc_parity(tg, orc, n, H, W, n5, bias):
    """C3 and C5 on tcgen05 with every operand split into two fp16 numbers (3 MMAs per product):
    the fp32 bound, normwise 1e-5 (north_star; R16) -- the same bound and the same
    cases as the FFMA path, incl. single-pixel planes, on narrow and wide rows, every NP."""
    seed = synth.seed_for_config(3) + 29
    img = synth.images_np(seed, n, H, W)
    prm = synth.cnn_params_np(seed, n5, H, W, bias)
    out, p = run_cnn(tg, img, n5, prm, bias, precision=tg.TG_FP32_TC)
    assert p.json()["precision"] == "fp32_tc"
    ref = orc.cnn(img, n5, prm, bias_plane=(bias == "plane"))
    err = normwise(out, ref)
    assert err <= 1e-5, err
    out32, _ = run_cnn(tg, img, n5, prm, bias)  # really a different path from the FFMA kernels
    assert not np.array_equal(out, out32)
    assert normwise(out32, ref) <= 1e-5


def test_cnn_fp32_tc_split_equals_unsplit(tg):
    seed = 93
    n, H, W, n5 = 2, 200, 180, 120
    img = synth.images_np(seed, n, H, W)
    prm = synth.cnn_params_np(seed, n5, H, W)
    full, p0 = run_cnn(tg, img, n5, prm, precision=tg.TG_FP32_TC)
    split, p1 = run_cnn(tg, img, n5, prm, budget=2_500_000, precision=tg.TG_FP32_TC)  # T2/T4 split + B operands
    assert p1.json()["n_chunks"] > p0.json()["n_chunks"]
    assert np.array_equal(split, full)


@pytest.mark.parametrize("n5,prec", [(20, "fp32"), (120, "fp32"), (120, "bf16_tc"), (120, "fp32_tc")])
def test_cnn_config3_full_batch_sampled(tg, orc, n5, prec):
    """BASELINE configs[2] at full size in the bench's launch configuration (64 x 480x640 images,
    device-resident, uncapped): images 0, 31 and 63 match the oracle."""
    n, H, W = 64, 480, 640
    seed = synth.seed_for_config(3)
    x = synth.images_torch(seed, n, H, W, "cuda")
    prm = synth.cnn_params_np(seed, n5, H, W)
    h5, w5 = synth.cnn_dims(H, W)[4]
    y = torch.zeros((n, 9, h5, w5), dtype=torch.float32, device="cuda")
    g, _ = tg.cnn_graph(x, n5, prm, out=y, device=True)
    g.set(torch_runtime=True, precision={"bf16_tc": tg.TG_BF16_TC, "fp32_tc": tg.TG_FP32_TC}.get(prec, tg.TG_FP32))
    p = g.plan()
    p.execute()
    out = y.cpu().numpy()
    img = x.cpu().numpy()
    tol = 2e-2 if prec == "bf16_tc" else 1e-5
    for b in (0, 31, 63):
        ref = orc.cnn(img[b:b + 1], n5, prm)
        assert normwise(out[b:b + 1], ref) <= tol, b


@pytest.mark.parametrize("prec", ["fp32", "bf16_tc", "fp32_tc"])
def test_cnn_invalidate_params(tg, orc, prec):
    """Parameters stay resident in the arena after the first execution; after the caller
    changes them in place, tg_plan_invalidate_params makes the next execution re-upload them
    (and re-derive the tensor-core operands and the channel-quad bias planes). Without it the old
    values are used."""
    seed = 77
    n, H, W, n5 = 2, 100, 120, 20
    img = synth.images_np(seed, n, H, W)
    prm = synth.cnn_params_np(seed, n5, H, W)
    out = np.zeros((n, 9) + synth.cnn_dims(H, W)[4], np.float32)
    g, _ = tg.cnn_graph(img, n5, prm, out=out)
    g.set(torch_runtime=True, precision={"fp32": tg.TG_FP32, "bf16_tc": tg.TG_BF16_TC, "fp32_tc": tg.TG_FP32_TC}[prec])
    p = g.plan()
    p.execute()
    first = out.copy()
    tol = 2e-2 if prec == "bf16_tc" else 1e-5
    assert normwise(first, orc.cnn(img, n5, prm)) <= tol
    for i in (1, 4, 6, 7, 9):          # arena-resident: B1, B3, K5, B5, B6 (K1, K3, P2, P4
        # travel by value with every launch and take effect at once)
        prm[i] *= np.float32(-0.5)
    p.execute()                        # still the resident (old) parameters
    if prec == "fp32":
        assert np.array_equal(out, first)
    p.invalidate_params()
    p.execute()
    assert normwise(out, orc.cnn(img, n5, prm)) <= tol
    assert not np.allclose(out, first)


@pytest.mark.parametrize("bias", ["resident", "streamed"])
def test_cnn_pipelined_async_executions(tg, bias):
    """Back-to-back tg_execute_async calls of one host-I/O plan overlap (the slot ring persists
    across executions); every execution still produces the blocking result bit for bit."""
    seed = 78
    n, H, W, n5 = 3, 160, 150, 20
    img_t = pinned((n, 1, H, W))
    img_t.copy_(torch.from_numpy(synth.images_np(seed, n, H, W)))
    prm = synth.cnn_params_np(seed, n5, H, W)
    out_t = pinned((n, 9) + synth.cnn_dims(H, W)[4])
    g, _ = tg.cnn_graph(img_t, n5, prm, out=out_t)
    # a budget small enough for row chunks (streamed bias rows) or only batch chunks
    g.set(torch_runtime=True, budget=1_000_000 if bias == "streamed" else 0, max_chunk_px=H * W, depth=2)
    p = g.plan()
    assert p.json()["bias"] == bias and p.json()["n_chunks"] >= 3
    p.execute()
    ref = out_t.clone()
    for _ in range(4):
        out_t.zero_()
        torch.cuda.synchronize()
        for _ in range(3):
            p.execute(blocking=False)
        torch.cuda.synchronize()
        assert torch.equal(out_t, ref)


@pytest.mark.parametrize("k3_mul,k5_mul", [(1e-4, 1e-3), (3.0, 1e-5), (1e-5, 1.0), (1.0, 30.0)])
def test_cnn_fp32_tc_weight_magnitudes(tg, orc, k3_mul, k5_mul):
    """3xFP16 scales each layer's weights by a power of two chosen from its largest magnitude
    (cnn_h3_weight_scale), so weights far outside the synthetic +-1/sqrt(fan_in) range -- small
    enough to lose their low parts at a fixed scale, or large -- keep the fp32 bound: 1e-5
    normwise on both fp32 paths (the same bound, the same inputs)."""
    seed = synth.seed_for_config(3) + 41
    n, H, W, n5 = 2, 92, 100, 60
    img = synth.images_np(seed, n, H, W)
    prm = synth.cnn_params_np(seed, n5, H, W)
    prm[3] = (prm[3] * np.float32(k3_mul)).astype(np.float32)
    prm[6] = (prm[6] * np.float32(k5_mul)).astype(np.float32)
    out, _ = run_cnn(tg, img, n5, prm, precision=tg.TG_FP32_TC)
    ff, _ = run_cnn(tg, img, n5, prm)
    ref = orc.cnn(img, n5, prm)
    assert np.isfinite(out).all()
    e_tc, e_ff = normwise(out, ref), normwise(ff, ref)
    assert e_tc <= 1e-5 and e_ff <= 1e-5, (e_tc, e_ff)


@pytest.mark.parametrize("k3_mul,k5_mul", [(1e4, 1.0), (1.0, 1e4)])
def test_cnn_fp32_tc_huge_weights_stay_finite(tg, orc, k3_mul, k5_mul):
    """Weights x 1e4 (which would overflow fp16 at a fixed scale) stay finite on the 3xFP16
    path. The inputs are ill-conditioned for ANY fp32 evaluation (pre-activations ~1e3: an fp32
    rounding of the 200- or 500-term sum moves a tanh near its zero crossing by ~1e-4), so no
    accuracy bound is claimed here beyond agreeing with the FFMA path to the same order."""
    seed = synth.seed_for_config(3) + 41
    n, H, W, n5 = 2, 92, 100, 60
    img = synth.images_np(seed, n, H, W)
    prm = synth.cnn_params_np(seed, n5, H, W)
    prm[3] = (prm[3] * np.float32(k3_mul)).astype(np.float32)
    prm[6] = (prm[6] * np.float32(k5_mul)).astype(np.float32)
    out, _ = run_cnn(tg, img, n5, prm, precision=tg.TG_FP32_TC)
    ff, _ = run_cnn(tg, img, n5, prm)
    ref = orc.cnn(img, n5, prm)
    assert np.isfinite(out).all()
    print("huge weights normwise: fp32_tc", normwise(out, ref), "fp32", normwise(ff, ref))
    assert normwise(out, ref) <= 10 * max(normwise(ff, ref), 1e-5)


@pytest.mark.parametrize("prec", ["bf16_tc", "fp32_tc"])
def test_cnn_two_host_threads_tensor_core_operands(tg, orc, prec):
    """tg_set_devices([0, 0]): both device threads upload the tensor-core B operands prepared
    ONCE on the calling thread (no race on the plan-level operand cache), every execution."""
    P = {"bf16_tc": tg.TG_BF16_TC, "fp32_tc": tg.TG_FP32_TC}[prec]
    seed = 57
    n, H, W, n5 = 4, 120, 160, 120
    img = synth.images_np(seed, n, H, W)
    prm = synth.cnn_params_np(seed, n5, H, W)
    ref, _ = run_cnn(tg, img, n5, prm, budget=3_000_000, precision=P)
    h5, w5 = synth.cnn_dims(H, W)[4]
    for rep in range(3):
        out = np.zeros((n, 9, h5, w5), np.float32)
        g, _ = tg.cnn_graph(img, n5, prm, out=out)
        g.set(budget=3_000_000, devices=[0, 0], torch_runtime=True, precision=P)
        p = g.plan()
        assert p.stats()["n_chunks"] >= 4
        p.execute()
        p.execute()
        assert np.array_equal(out, ref), rep


@pytest.mark.parametrize("prec", ["fp32", "bf16_tc", "fp32_tc"])
@pytest.mark.parametrize("mode", ["batch", "rows_streamed", "rows_resident", "scalar", "device"])
def test_cnn_slot_layout_covers_every_buffer(tg, orc, prec, mode):
    """The slot layout (the library's design; tests/test_plan_parity.py checks its sizes only by
    properties) holds every buffer the kernels touch: with the arena between guard bands and
    pre-filled with NaN bytes, every precision and chunking leaves the guards intact and matches
    the oracle (an unfilled or overlapping buffer would show up as NaN or a wrong value)."""
    P = {"fp32": tg.TG_FP32, "bf16_tc": tg.TG_BF16_TC, "fp32_tc": tg.TG_FP32_TC}[prec]
    seed = 61
    n, H, W, n5 = (7 if mode == "batch" else 3), 150, 172, 40
    bias = "scalar" if mode == "scalar" else "plane"
    img = synth.images_np(seed, n, H, W)
    prm = synth.cnn_params_np(seed, n5, H, W, bias)
    h5, w5 = synth.cnn_dims(H, W)[4]
    budget = {"batch": 0, "rows_streamed": 1_200_000, "rows_resident": 2_200_000, "scalar": 600_000,
              "device": 0}[mode]
    bm = tg.TG_BIAS_PLANE if bias == "plane" else tg.TG_BIAS_SCALAR
    if mode == "device":
        x = torch.from_numpy(img).cuda()
        out_t = torch.zeros((n, 9, h5, w5), dtype=torch.float32, device="cuda")
        g, _ = tg.cnn_graph(x, n5, prm, out=out_t, bias_mode=bm, device=True)
    else:
        out = np.zeros((n, 9, h5, w5), np.float32)
        g, _ = tg.cnn_graph(img, n5, prm, out=out, bias_mode=bm)
    rt = guard_runtime(tg)
    g.runtime = rt
    tg.tg_set_runtime(g.h, rt.struct)
    g.set(budget=budget, precision=P, max_chunk_px=(H * W * 2 if mode == "batch" else None))
    p = g.plan()
    j = p.json()
    want_bias = {"batch": "resident", "rows_streamed": "streamed", "rows_resident": "resident",
                 "scalar": "scalar", "device": "resident"}[mode]
    assert j["bias"] == want_bias, j["bias"]
    if mode.startswith("rows"):
        assert j["split"] == "rows" and j["n_chunks"] > n
    if mode == "batch":
        assert j["split"] == "batch" and j["B"] > 1 and j["n_chunks"] > 1
    p.execute()
    p.execute()
    got = out_t.cpu().numpy() if mode == "device" else out
    assert rt.guards_intact()
    ref = orc.cnn(img, n5, prm, bias_plane=(bias == "plane"))
    assert np.isfinite(got).all()
    assert normwise(got, ref) <= (2e-2 if prec == "bf16_tc" else 1e-5)


@pytest.mark.parametrize("prec", ["fp32", "bf16_tc", "fp32_tc"])
def test_cnn_graph_replay_and_new_parameters(tg, orc, prec):
    """CUDA-graph replay of a streamed CNN plan (bias rows streamed, several chunks) equals the
    direct execution; after tg_plan_invalidate_params with new weights the graph is recaptured
    and follows them (the captured kernels hold the weights by value)."""
    P = {"fp32": tg.TG_FP32, "bf16_tc": tg.TG_BF16_TC, "fp32_tc": tg.TG_FP32_TC}[prec]
    seed = 77
    n, H, W, n5 = 2, 150, 172, 40
    img = synth.images_np(seed, n, H, W)
    prm = synth.cnn_params_np(seed, n5, H, W)
    h5, w5 = synth.cnn_dims(H, W)[4]
    out = np.zeros((n, 9, h5, w5), np.float32)
    g, _ = tg.cnn_graph(img, n5, prm, out=out)
    g.set(torch_runtime=True, budget=1_200_000, precision=P)
    p = g.plan()
    assert p.json()["n_chunks"] > 2
    p.execute()
    direct = out.copy()
    p.use_graph(True)
    for rep in range(2):
        out[:] = 0
        p.execute()
        assert np.array_equal(out, direct), rep
    for k in (3, 6):                     # new C3 / C5 weights in the caller's parameter buffers
        prm[k] *= np.float32(0.75)
    p.invalidate_params()
    p.execute()
    p.execute()
    ref = orc.cnn(img, n5, prm)
    assert normwise(out, ref) <= (2e-2 if prec == "bf16_tc" else 1e-5)
