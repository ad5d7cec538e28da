"""The code generator (tg_plan_codegen: the execution plan becomes "a hybrid
CPU/GPU program ... compiled together with a larger application"):
  * CPU: the generated C source for split TG_PER_OP / TG_BASELINE plans compiles against
    include/tg.h and the CUDA runtime headers, holds one tg_oplib_run call per planned operator
    piece and one copy per planned transfer; TG_FUSED plans are refused;
  * GPU: the generated program, compiled with gcc and linked against the library, reproduces
    the library's own execution of the plan bit for bit and the CPU oracle within 1e-5."""
import ctypes
import os
import subprocess

import numpy as np
import pytest

import synth
from split_graphs import cnn_spec, edge_spec, lib_graph, mixed_spec

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CUDA_INC = "/usr/local/cuda/include"


def plan_of(spec, frac, mode_name="TG_PER_OP", torch_runtime=False):
    from paper_conf_ipps_sundaramrc09_b200 import tg
    out = np.full(spec.shapes[spec.output], np.nan, np.float32)
    budget = int(spec.total_bytes() * frac) // 256 * 256
    g = lib_graph(spec, out, budget=budget, torch_runtime=torch_runtime)
    return g, g.plan(getattr(tg, mode_name)), out


def specs():
    K1, K2 = synth.random_edge_filters_np(7)
    H, W, n5 = 77, 41, 4
    return {"edge": (edge_spec(301, 64, K1, K2, n=2, rng=3), 0.2),
            "cnn": (cnn_spec(1, H, W, n5, synth.cnn_params_np(11, n5, H, W)), 0.25),
            "mixed": (mixed_spec(83, 30, 7), 0.15)}


@pytest.mark.parametrize("name", ["edge", "cnn", "mixed"])
@pytest.mark.parametrize("mode_name", ["TG_PER_OP", "TG_BASELINE"])
def test_codegen_source(tmp_path, name, mode_name):
    spec, frac = specs()[name]
    if mode_name == "TG_BASELINE":
        frac = 0          # the baseline runs operators whole: uncapped
    g, p, _ = plan_of(spec, frac, mode_name)
    src = p.codegen()
    j = p.json()
    assert src.count("tg_oplib_run(&op") == len(j["ops"])
    assert src.count("tgg_rows(arena") + src.count("cudaMemcpyAsync(") == len(j["trace"]) - len(j["ops"])
    assert f"#define TG_GEN_ARENA_BYTES {j['arena_bytes']}ull" in src
    f = tmp_path / "gen.c"
    f.write_text(src)
    if not os.path.isdir(CUDA_INC):
        pytest.skip("no CUDA headers")
    subprocess.check_call(["gcc", "-std=c11", "-Wall", "-Werror", "-fsyntax-only", "-I", os.path.join(ROOT, "include"),
                           "-I", CUDA_INC, str(f)])


def test_codegen_refuses_fused():
    from paper_conf_ipps_sundaramrc09_b200 import tg
    img = np.zeros((1, 1, 64, 64), np.float32)
    K1, K2 = synth.random_edge_filters_np(1)
    g, _ = tg.edge_graph(img, K1, out=np.zeros_like(img))
    with pytest.raises(tg.TGError) as e:
        g.plan(tg.TG_FUSED).codegen()
    assert e.value.code == tg.TG_E_UNSUPPORTED


@pytest.mark.gpu
@pytest.mark.parametrize("name,mode_name", [("edge", "TG_PER_OP"), ("cnn", "TG_PER_OP"), ("mixed", "TG_PER_OP"),
                                            ("cnn", "TG_BASELINE"), ("mixed", "TG_BASELINE")])
def test_generated_program_runs(tmp_path, orc, name, mode_name):
    from gpu_util import need_gpu, normwise, torch
    need_gpu()
    from paper_conf_ipps_sundaramrc09_b200 import tg
    torch.cuda.set_device(0)
    spec, frac = specs()[name]
    if mode_name == "TG_BASELINE":
        frac = 0                                     # the baseline runs operators whole
    g, p, out = plan_of(spec, frac, mode_name, torch_runtime=True)
    p.execute()                                      # the library's own executor
    if mode_name == "TG_PER_OP":
        assert max(p.json()["k"].values()) > 1
    src = tmp_path / "gen.c"
    src.write_text(p.codegen())
    so = tmp_path / "libgen.so"
    subprocess.check_call(["gcc", "-std=c11", "-O1", "-shared", "-fPIC", "-o", str(so), str(src),
                           "-I", os.path.join(ROOT, "include"), "-I", CUDA_INC, tg.LIB_PATH,
                           "-L/usr/local/cuda/lib64", "-lcudart", f"-Wl,-rpath,{os.path.dirname(tg.LIB_PATH)}"])
    lib = ctypes.CDLL(str(so))
    lib.tg_generated_execute.restype = ctypes.c_int
    lib.tg_generated_execute.argtypes = [ctypes.POINTER(ctypes.c_void_p), ctypes.c_void_p, ctypes.c_void_p]
    gen_out = np.full_like(out, np.nan)
    host = (ctypes.c_void_p * len(spec.shapes))()
    for d, a in spec.data.items():
        host[d] = a.ctypes.data
    host[spec.output] = gen_out.ctypes.data
    arena = torch.empty(p.json()["arena_bytes"], dtype=torch.uint8, device="cuda")
    torch.cuda.synchronize()
    assert lib.tg_generated_execute(host, arena.data_ptr(), None) == 0
    assert np.array_equal(gen_out, out)
    if name == "edge":
        K1, K2 = spec.data[1][0, 0], spec.data[2][0, 0]
        want = np.stack([orc.edge(spec.data[0][i, 0], K1, K2) for i in range(2)])[:, None]
        assert normwise(gen_out[:, 0], want[:, 0]) <= 1e-5
