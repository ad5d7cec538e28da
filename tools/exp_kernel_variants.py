"""Kernel experiments without experiment hooks in the product sources: copy the package to
_exp/<variant>/ (git-ignored), apply textual patches to one kernel source, build that copy, and time the
CNN units of a workload through it (device-resident, per-unit CUDA events). Prints one JSON line
per variant: {"variant", "unit_ms": {1: U1, 2: U2, 3: U3}, "value_mpx_s"}.

  python tools/exp_kernel_variants.py --workload cnn3 --precision bf16_tc --variants base,no_epi,no_c5
"""
import argparse
import json
import os
import shutil
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = "paper_conf_ipps_sundaramrc09_b200"

VARIANTS_U3_NO_EPI = [
    ("            tc::mbar_wait(&S.t_full[buf], (uint32_t)((k / U3_NB) & 1));\n            tc::fence_after_sync();\n#pragma unroll\n            for (int c = 0; c < NC; ++c) {\n                if (c < nc) {",
     "            tc::mbar_wait(&S.t_full[buf], (uint32_t)((k / U3_NB) & 1));\n            tc::fence_after_sync();\n#pragma unroll\n            for (int c = 0; c < NC; ++c) {\n                if (c < 0) {"),
    ("            if (cur.ok) {\n                float* ob", "            if (false) {\n                float* ob")]


U3_NO_C5 = [("                            tc::mma_bf16(d_base + (uint32_t)(t * 128), ad + (uint64_t)(t * kTileM), bd, idesc,",
             "                            if (r8 < 0) tc::mma_bf16(d_base + (uint32_t)(t * 128), ad + (uint64_t)(t * kTileM), bd, idesc,")]
U3_NO_BIAS = [("            if (16 * c + 16 <= a.n5) {  // a full chunk of real channels (uniform)\n#pragma unroll\n                for (int u = 0; u < 16; ++u, p += bcs) bv[r][u] = __ldg(p);",
               "            if (16 * c + 16 <= a.n5) {  // a full chunk of real channels (uniform)\n#pragma unroll\n                for (int u = 0; u < 16; ++u, p += bcs) bv[r][u] = 0.f;")]
U3_NO_BIAS_Q4 = [("                    const float4 f = (16 * c + 4 * u < a.n5) ? __ldg(p4 + (size_t)u * bcs) : make_float4(0.f, 0.f, 0.f, 0.f);",
                   "                    const float4 f = make_float4(0.f, 0.f, 0.f, 0.f);")]
H3U2_NO_EPI = [("            const bool out_ok = !(lane & 1) && C < a.w4;\n            // the two C3 rows",
                "            const bool out_ok = false; if (k >= 0) continue;\n            // the two C3 rows")]
U3_NO_TANH = [("for (int u = 0; u < 16; ++u) v[u] = tanh_approx(v[u] + bv[0][u]);", "for (int u = 0; u < 16; ++u) v[u] = v[u] + bv[0][u];"),
              ("for (int u = 0; u < 16; ++u) v[u] = tanh_approx(v[u] + bv[1][u]);", "for (int u = 0; u < 16; ++u) v[u] = v[u] + bv[1][u];")]
U3_NO_TMEMLD = [("                    tc::tmem_ld16_async(region + (uint32_t)(16 * c), v);\n                    tc::tmem_wait_ld();",
                 "#pragma unroll\n                    for (int u = 0; u < 16; ++u) v[u] = __int_as_float(region + u) * 1e-30f;")]
U3_NO_TMEMST = [("                    tc::tmem_st8(region + (uint32_t)(8 * c), r);", "                    if (r[0] == 12345u) tc::tmem_st8(region + (uint32_t)(8 * c), r);")]

H3U3_NO_MMA = [
    ("                                    tc::mma_bf16(d, a_hi, bd, idesc, acc0);\n                                    tc::mma_bf16(d, a_hi, bd + b_part, idesc, 1u);\n                                    tc::mma_bf16(d, a_lo, bd, idesc, 1u);",
     "                                    if (acc0 > 7u) tc::mma_bf16(d, a_lo, bd, idesc, 1u);")]
H3U3_NO_EPI = [
    ("#pragma unroll\n            for (int c = 0; c < NCH; ++c) {\n                float v[32];\n                const uint32_t col = (uint32_t)(buf * 256 + t * (kFuse ? 2 * NP : NP) + 32 * c);",
     "#pragma unroll\n            for (int c = 0; c < 0; ++c) {\n                float v[32];\n                const uint32_t col = (uint32_t)(buf * 256 + t * (kFuse ? 2 * NP : NP) + 32 * c);"),
    ("            if (cur.ok) {\n                float* ob = a.out + cur.img * a.out_img_stride", "            if (false) {\n                float* ob = a.out + cur.img * a.out_img_stride")]
H3U3_NO_BCOPY = [
    ("                        tc::mbar_expect_tx(&S.b_full[slot], stage_bytes);\n                        tc::bulk_g2s(S.b[slot], kb + (size_t)(ks / U3H_KST) * stage_bytes, stage_bytes, &S.b_full[slot]);",
     "                        tc::mbar_arrive(&S.b_full[slot]);")]
H3U3_NO_ACOPY = [
    ("                    if (lane == 0) tc::mbar_expect_tx(&S.a_full[slot], (uint32_t)(6 * n * 16));\n                    __syncwarp();\n                    if (n > 0 && lane < 6) {",
     "                    if (lane == 0) tc::mbar_arrive(&S.a_full[slot]);\n                    __syncwarp();\n                    if (false) {")]

U2_NO_COPY = [("            if (lane == 0) tc::mbar_expect_tx(&S.a_full[buf], (uint32_t)(rows * cols * 16));\n            __syncwarp();\n            if (lane < rows) {",
               "            if (lane == 0) tc::mbar_arrive(&S.a_full[buf]);\n            __syncwarp();\n            if (false) {")]
U2_NO_EPI = [("            const bool out_ok = !(lane & 1) && C < a.w4;", "            const bool out_ok = false; if (k >= 0) continue;")]

# variant -> (kernel source, [(old, new), ...]); every `old` must occur in the source
VARIANTS = {
    "base": ("cnn_tc.cu", []),
    # U3 (both tensor-core paths): the C5 bias planes in the plane layout (no channel-quad loads)
    "no_q4": ("../engine.cu", [("    return c.t.kind == Tmpl::Cnn && c.bias == \"resident\" && c.param_off[7] != UINT64_MAX",
                                "    return false && c.t.kind == Tmpl::Cnn && c.bias == \"resident\" && c.param_off[7] != UINT64_MAX")]),
    # U3 bf16: the epilogue only does the barrier hand-offs (no TMEM loads, bias, tanh, stores)
    "u3_no_epi": ("cnn_tc.cu", [
        ("            tc::mbar_wait(&S.t_full[buf], (uint32_t)((k / U3_NB) & 1));\n            tc::fence_after_sync();\n#pragma unroll\n            for (int c = 0; c < NC; ++c) {\n                if (c < nc) {",
         "            tc::mbar_wait(&S.t_full[buf], (uint32_t)((k / U3_NB) & 1));\n            tc::fence_after_sync();\n#pragma unroll\n            for (int c = 0; c < NC; ++c) {\n                if (c < 0) {"),
        ("            if (cur.ok) {\n                float* ob", "            if (false) {\n                float* ob")]),
    # U3 bf16: epilogue hand-offs only AND the C5 MMAs at N = 64 instead of NP (half the B reads
    # and half the math): tells a smem-operand-bound MMA phase from a compute-bound one
    "u3_no_epi_n64": ("cnn_tc.cu", [
        ("            tc::mbar_wait(&S.t_full[buf], (uint32_t)((k / U3_NB) & 1));\n            tc::fence_after_sync();\n#pragma unroll\n            for (int c = 0; c < NC; ++c) {\n                if (c < nc) {",
         "            tc::mbar_wait(&S.t_full[buf], (uint32_t)((k / U3_NB) & 1));\n            tc::fence_after_sync();\n#pragma unroll\n            for (int c = 0; c < NC; ++c) {\n                if (c < 0) {"),
        ("            if (cur.ok) {\n                float* ob", "            if (false) {\n                float* ob"),
        ("        const uint32_t idesc = tc::make_idesc_bf16(kTileM, NP);", "        const uint32_t idesc = tc::make_idesc_bf16(kTileM, 64);")]),
    # U3 bf16: the C5 MMAs at N = 64 with the full epilogue (wrong values; timing only): half the B
    # operand's shared-memory reads -- does the MMAs' port traffic slow the epilogue?
    "u3_n64": ("cnn_tc.cu", [
        ("        const uint32_t idesc = tc::make_idesc_bf16(kTileM, NP);", "        const uint32_t idesc = tc::make_idesc_bf16(kTileM, 64);")]),
    "u3_n64_mma_only": ("cnn_tc.cu", VARIANTS_U3_NO_EPI + [
        ("            if (lane == 0) tc::mbar_expect_tx(&S.a_full[slot], (uint32_t)(3 * n * 16));\n            __syncwarp();\n            if (n > 0 && lane < 3)",
         "            if (lane == 0) tc::mbar_arrive(&S.a_full[slot]);\n            __syncwarp();\n            if (false)"),
        ("        const uint32_t idesc = tc::make_idesc_bf16(kTileM, NP);", "        const uint32_t idesc = tc::make_idesc_bf16(kTileM, 64);")]),
    # U3 bf16: no bias loads (bias 0), the rest of the epilogue as built
    "u3_no_bias": ("cnn_tc.cu", [
        ("            if (16 * c + 16 <= a.n5) {  // a full chunk of real channels (uniform)\n#pragma unroll\n                for (int u = 0; u < 16; ++u, p += bcs) bv[r][u] = __ldg(p);",
         "            if (16 * c + 16 <= a.n5) {  // a full chunk of real channels (uniform)\n#pragma unroll\n                for (int u = 0; u < 16; ++u, p += bcs) bv[r][u] = 0.f;")]),
    # U3 bf16: the MMA warp issues no C5 MMAs (commits still arrive)
    "u3_no_c5": ("cnn_tc.cu", [
        ("                            tc::mma_bf16(d_base + (uint32_t)(t * 128), ad + (uint64_t)(t * kTileM), bd, idesc,",
         "                            if (r8 < 0) tc::mma_bf16(d_base + (uint32_t)(t * 128), ad + (uint64_t)(t * kTileM), bd, idesc,")]),
    # U3 bf16: no C6 MMAs
    "u3_no_c6": ("cnn_tc.cu", [
        ("                        tc::mma_bf16_ts(base + (uint32_t)(t * 128 + U3_C6COL)",
         "                        if (kk < 0) tc::mma_bf16_ts(base + (uint32_t)(t * 128 + U3_C6COL)")]),
    # U3 bf16: no slice copies (the MMAs read whatever the ring holds)
    "u3_no_copy": ("cnn_tc.cu", [
        ("            if (lane == 0) tc::mbar_expect_tx(&S.a_full[slot], (uint32_t)(3 * n * 16));\n            __syncwarp();\n            if (n > 0 && lane < 3)",
         "            if (lane == 0) tc::mbar_arrive(&S.a_full[slot]);\n            __syncwarp();\n            if (false)")]),
    # U3 3xFP16 (TG_FP32_TC): no B-operand streaming (the ring stages arrive without copies)
    "h3u3_no_bcopy": ("cnn_h3.cu", [
        ("                        tc::mbar_expect_tx(&S.b_full[slot], stage_bytes);\n                        tc::bulk_g2s(S.b[slot], kb + (size_t)(ks / U3H_KST) * stage_bytes, stage_bytes, &S.b_full[slot]);",
         "                        tc::mbar_arrive(&S.b_full[slot]);")]),
    # U3 3xFP16: the epilogue only does the hand-offs
    "h3u3_no_epi": ("cnn_h3.cu", [
        ("#pragma unroll\n            for (int c = 0; c < NCH; ++c) {\n                float v[32];\n                const uint32_t col = (uint32_t)(buf * 256 + t * (kFuse ? 2 * NP : NP) + 32 * c);",
         "#pragma unroll\n            for (int c = 0; c < 0; ++c) {\n                float v[32];\n                const uint32_t col = (uint32_t)(buf * 256 + t * (kFuse ? 2 * NP : NP) + 32 * c);"),
        ("            if (cur.ok) {\n                float* ob = a.out + cur.img * a.out_img_stride", "            if (false) {\n                float* ob = a.out + cur.img * a.out_img_stride")]),
    # U3 3xFP16: no MMAs (commits still arrive)
    "h3u3_no_mma": ("cnn_h3.cu", H3U3_NO_MMA),
    # U3 3xFP16: two MMAs per K-step instead of three (hi.hi + hi.lo): the MMA-count sensitivity
    "h3u3_2mma": ("cnn_h3.cu", [
        ("                                    tc::mma_bf16(d, a_hi, bd + b_part, idesc, 1u);\n                                    tc::mma_bf16(d, a_lo, bd, idesc, 1u);",
         "                                    tc::mma_bf16(d, a_hi, bd + b_part, idesc, 1u);")]),
    # U2 bf16 decomposition
    "u2_no_copy": ("cnn_tc.cu", U2_NO_COPY),
    "u2_no_epi": ("cnn_tc.cu", U2_NO_EPI),
    "u2_mma_only": ("cnn_tc.cu", U2_NO_COPY + U2_NO_EPI),
    # U3 3xFP16: the scalar tanh (A/B against the paired tanh_fp32x2 of the tree)
    "h3u3_tanh_scalar": ("cnn_h3.cu", [
        ("""                for (int u = 0; u < 32; u += 2) {
                    const float2 x = __ffma2_rn(make_float2(v[u], v[u + 1]), make_float2(a.w_unscale, a.w_unscale),
                                                make_float2(bv[u], bv[u + 1]));
                    const float2 y = tanh_fp32x2(x);
                    v[u] = y.x;
                    v[u + 1] = y.y;
                }""", """                for (int u = 0; u < 32; ++u) v[u] = tanh_acc(fmaf(v[u], a.w_unscale, bv[u]));""")]),
    # U3 3xFP16 epilogue decomposition (no MMAs; then one epilogue step removed at a time)
    "h3e_no_c6": ("cnn_h3.cu", H3U3_NO_MMA + [
        ("#pragma unroll\n                    for (int o = 0; o < 9; ++o) c6[o] = fmaf(k6w.k6[ch][o], v[u], c6[o]);",
         "                    c6[u % 9] += v[u];")]),
    "h3e_no_bias": ("cnn_h3.cu", H3U3_NO_MMA + [
        ("                for (int u = 0; u < 32; ++u, p += bcs) bv[u] = __ldg(p);\n            } else {",
         "                for (int u = 0; u < 32; ++u, p += bcs) bv[u] = 0.f;\n            } else {")]),
    "h3e_no_tanh": ("cnn_h3.cu", H3U3_NO_MMA + [
        ("for (int u = 0; u < 32; ++u) v[u] = tanh_acc(fmaf(v[u], a.w_unscale, bv[u]));",
         "for (int u = 0; u < 32; ++u) v[u] = fmaf(v[u], a.w_unscale, bv[u]);")]),
    # U3 bf16 with the MMAs: each epilogue step removed in turn (what the combination costs)
    "u3_no_tanh": ("cnn_tc.cu", U3_NO_TANH),
    "u3_no_tmemld": ("cnn_tc.cu", U3_NO_TMEMLD),
    "u3_no_tmemst": ("cnn_tc.cu", U3_NO_TMEMST),
    "u3_no_bias_q4": ("cnn_tc.cu", U3_NO_BIAS_Q4),
    # U3 bf16: the bias ring of two chunk buffers loaded two chunks ahead (as before the end of round 2)
    "u3_bias_ring2": ("cnn_tc.cu", [("        const int ring = (BQ == 1 || nc % 2) ? 1 : 2;", "        const int ring = (nc % 2 == 0) ? 2 : 1;")]),
    # U2 3xFP16 decomposition: epilogue hand-offs only; and also no window copies (MMAs alone)
    "h3u2_no_epi": ("cnn_h3.cu", H3U2_NO_EPI),
    "h3u2_mma_only": ("cnn_h3.cu", H3U2_NO_EPI + [
        ("            if (lane == 0) tc::mbar_expect_tx(&S.a_full[buf], (uint32_t)(2 * rows * cols * 16));\n            __syncwarp();\n            if (lane < 2 * rows) {",
         "            if (lane == 0) tc::mbar_arrive(&S.a_full[buf]);\n            __syncwarp();\n            if (false) {")]),
    # U2 bf16: three epilogue groups (14 warps, 128 registers) and / or 8 TMEM slots
    "u2_nt8": ("cnn_tc.cu", [("constexpr int U2_NT = 4;", "constexpr int U2_NT = 8;")]),
    "h3u2_g2": ("cnn_h3.cu", [("constexpr int U2H_G = 3;", "constexpr int U2H_G = 2;")]),
    "u2_g2": ("cnn_tc.cu", [("constexpr int U2_G = 3;", "constexpr int U2_G = 2;")]),
    "u3_one_tile_bands": ("cnn_tc.cu", [("constexpr int U3_BT = 2;", "constexpr int U3_BT = 1;")]),
    # U3 bf16 epilogue decomposition: no C5 MMAs, then each epilogue step removed in turn
    "u3e": ("cnn_tc.cu", U3_NO_C5),
    "u3e_no_bias": ("cnn_tc.cu", U3_NO_C5 + U3_NO_BIAS),
    "u3e_no_tanh": ("cnn_tc.cu", U3_NO_C5 + U3_NO_TANH),
    "u3e_no_tmemld": ("cnn_tc.cu", U3_NO_C5 + U3_NO_TMEMLD),
    "u3e_no_tmemst": ("cnn_tc.cu", U3_NO_C5 + U3_NO_TMEMST),
    "u3e_no_bias_tanh": ("cnn_tc.cu", U3_NO_C5 + U3_NO_BIAS + U3_NO_TANH),
    "u3e_bare": ("cnn_tc.cu", U3_NO_C5 + U3_NO_BIAS + U3_NO_TANH + U3_NO_TMEMLD + U3_NO_TMEMST),
    "u3_mma_only_no_c6": ("cnn_tc.cu", VARIANTS_U3_NO_EPI + [
        ("            if (lane == 0) tc::mbar_expect_tx(&S.a_full[slot], (uint32_t)(3 * n * 16));\n            __syncwarp();\n            if (n > 0 && lane < 3)",
         "            if (lane == 0) tc::mbar_arrive(&S.a_full[slot]);\n            __syncwarp();\n            if (false)"),
        ("                        tc::mma_bf16_ts(base + (uint32_t)(t * 128 + U3_C6COL)",
         "                        if (kk < 0) tc::mma_bf16_ts(base + (uint32_t)(t * 128 + U3_C6COL)")]),
    # U3 bf16: copies but no epilogue work (the MMA + copy pipeline alone)
    "u3_no_epi_work": ("cnn_tc.cu", VARIANTS_U3_NO_EPI),
    # U3 bf16: neither epilogue work nor slice copies (the MMA issue alone, plus C6)
    "u3_mma_only": ("cnn_tc.cu", VARIANTS_U3_NO_EPI + [
        ("            if (lane == 0) tc::mbar_expect_tx(&S.a_full[slot], (uint32_t)(3 * n * 16));\n            __syncwarp();\n            if (n > 0 && lane < 3)",
         "            if (lane == 0) tc::mbar_arrive(&S.a_full[slot]);\n            __syncwarp();\n            if (false)")]),
    # U3 3xFP16: the epilogue computes as built but never loads TMEM (values from a register)
    "h3u3_no_tmemld": ("cnn_h3.cu", [
        ("                tc::tmem_ld32_async(tmem + lane_base + col, v);\n                if (kFuse) {",
         "#pragma unroll\n                for (int u = 0; u < 32; ++u) v[u] = __int_as_float(col + u) * 1e-30f;\n                if (false) {"),
        ("                } else {\n                    tc::tmem_wait_ld();\n                }\n#pragma unroll\n                for (int u = 0; u < 32; ++u) v[u] = tanh_acc(",
         "                } else {\n                }\n#pragma unroll\n                for (int u = 0; u < 32; ++u) v[u] = tanh_acc(")]),
    # U3 3xFP16: the MMA issue loop alone (no epilogue work, no copies: every wait finds its barrier done)
    "h3u3_mma_only": ("cnn_h3.cu", H3U3_NO_EPI + H3U3_NO_BCOPY + H3U3_NO_ACOPY),
    "h3u3_no_epi_no_bcopy": ("cnn_h3.cu", H3U3_NO_EPI + H3U3_NO_BCOPY),
    # U3 3xFP16: no bias-plane loads (bias 0)
    "h3u3_no_bias": ("cnn_h3.cu", [
        ("                for (int u = 0; u < 32; ++u, p += bcs) bv[u] = __ldg(p);\n            } else {",
         "                for (int u = 0; u < 32; ++u, p += bcs) bv[u] = 0.f;\n            } else {")]),
    # U3 3xFP16: the epilogue without the 9 C6 FMA chains per channel
    "h3u3_no_c6": ("cnn_h3.cu", [
        ("#pragma unroll\n                    for (int o = 0; o < 9; ++o) c6[o] = fmaf(k6w.k6[ch][o], v[u], c6[o]);",
         "                    c6[u % 9] += v[u];")]),
}


def build_variant(name, prebuilt=False):
    if name == "tree":             # the working tree as built in place
        return ROOT
    if name == "head":             # the last commit's sources (same-box A/B against the working tree)
        dst = os.path.join(ROOT, "_exp", name)
        if prebuilt:
            return dst
        shutil.rmtree(dst, ignore_errors=True)
        os.makedirs(dst)
        subprocess.run(f"git -C {ROOT} archive HEAD {PKG} include synth | tar -x -C {dst}", shell=True, check=True)
        r = subprocess.run([sys.executable, os.path.join(dst, PKG, "build.py")], capture_output=True, text=True)
        if r.returncode:
            raise RuntimeError(r.stderr[-3000:])
        shutil.rmtree(os.path.join(dst, PKG, "_build"), ignore_errors=True)
        return dst
    spec = VARIANTS[name]
    files = spec if isinstance(spec, list) else [spec]   # [(kernel source, patches), ...]
    dst = os.path.join(ROOT, "_exp", name)   # git-ignored; travels to the GPU box with the snapshot
    if prebuilt:
        return dst
    if os.path.exists(dst):
        shutil.rmtree(dst)
    os.makedirs(dst)
    shutil.copytree(os.path.join(ROOT, PKG), os.path.join(dst, PKG),
                    ignore=shutil.ignore_patterns("_build*", "libtg.so*", "__pycache__"))
    shutil.copytree(os.path.join(ROOT, "include"), os.path.join(dst, "include"))
    shutil.copytree(os.path.join(ROOT, "synth"), os.path.join(dst, "synth"))
    for src_file, patches in files:
        path = os.path.join(dst, PKG, "csrc", "kernels", src_file)
        s = open(path).read()
        for old, new in patches:
            assert old in s, (name, old[:80])
            s = s.replace(old, new)
        open(path, "w").write(s)
    r = subprocess.run([sys.executable, os.path.join(dst, PKG, "build.py")], capture_output=True, text=True)
    if r.returncode:
        raise RuntimeError(r.stderr[-3000:])
    shutil.rmtree(os.path.join(dst, PKG, "_build"), ignore_errors=True)   # keep the snapshot small
    return dst


TIMER = r'''
import json, sys
sys.path.insert(0, sys.argv[1])
import torch, synth
from paper_conf_ipps_sundaramrc09_b200 import tg
wl, prec, steps = sys.argv[2], sys.argv[3], int(sys.argv[4])
n, H, W = 64, 480, 640
n5 = 20 if wl == "cnn3s" else 120
if wl == "cnn4":
    n, H, W = 1, 4800, 6400
seed = synth.seed_for_config(3)
torch.cuda.set_device(0)
x = synth.images_torch(seed, n, H, W, "cuda:0")
h5, w5 = synth.cnn_dims(H, W)[4]
y = torch.empty((n, 9, h5, w5), dtype=torch.float32, device="cuda:0")
scalar = wl == "cnn3b"   # scalar C-layer biases (TG_BIAS_SCALAR)
prm = synth.cnn_params_np(seed, n5, H, W, "scalar" if scalar else "plane")
g, _ = tg.cnn_graph(x, n5, prm, out=y, device=True, bias_mode=tg.TG_BIAS_SCALAR if scalar else tg.TG_BIAS_PLANE)
g.set(torch_runtime=True, precision={"fp32": 0, "bf16_tc": 1, "fp32_tc": 2}[prec])
p = g.plan()
for _ in range(3):
    p.execute()
p.profiling(True, copies=False)
cs = p.compute_stream(0)
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record(cs)
for _ in range(steps):
    p.execute(blocking=False)
e1.record(cs)
torch.cuda.synchronize()
t = p.timing()
ms = e0.elapsed_time(e1) / steps
print(json.dumps({"unit_ms": {u: t["kernel_ms"][u] / steps for u in (1, 2, 3)}, "step_ms": ms,
                  "value_mpx_s": n * H * W / ms / 1e3, "checksum": float(y.double().abs().sum())}))
'''


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="cnn3")
    ap.add_argument("--precision", default="bf16_tc")
    ap.add_argument("--variants", default="base")
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--build-only", action="store_true", help="build the variants here (no GPU needed)")
    ap.add_argument("--prebuilt", action="store_true", help="run variants built earlier with --build-only")
    args = ap.parse_args()
    if args.build_only:
        for v in args.variants.split(","):
            build_variant(v)
            print("built", v, flush=True)
        return
    for v in args.variants.split(","):
        try:
            d = build_variant(v, args.prebuilt)
            r = subprocess.run([sys.executable, "-c", TIMER, d, args.workload, args.precision, str(args.steps)],
                               capture_output=True, text=True, timeout=600)
            out = json.loads(r.stdout.strip().splitlines()[-1]) if r.returncode == 0 else {"error": r.stderr[-800:]}
        except Exception as e:  # noqa: BLE001
            out = {"error": str(e)[-800:]}
        print(json.dumps({"variant": v, "workload": args.workload, "precision": args.precision, **out}), flush=True)


if __name__ == "__main__":
    main()
