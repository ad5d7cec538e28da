"""The C-ABI library loads on a CPU-only box, exports every function include/tg.h declares,
and its host-side calls (graph building, planning, error reporting) work without a GPU."""
import ctypes
import os
import re

import numpy as np
import pytest

from conftest import ROOT


def header_functions():
    src = open(os.path.join(ROOT, "include", "tg.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    names = re.findall(r"^\s*(?:const\s+)?[\w]+\s*\*?\s*(tg_\w+)\s*\(", src, flags=re.M)
    return sorted(set(names))


def test_library_exports_every_header_symbol():
    from paper_conf_ipps_sundaramrc09_b200 import tg
    lib = ctypes.CDLL(tg.LIB_PATH)
    names = header_functions()
    assert len(names) >= 30
    for n in names:
        assert hasattr(lib, n), n
    assert set(names) == set(tg.EXPORTED)
    assert tg.tg_version().startswith("tg ")


def test_errors_are_reported():
    from paper_conf_ipps_sundaramrc09_b200 import tg
    g = tg.Graph()
    x = g.input(np.zeros((1, 1, 8, 8), np.float32))
    with pytest.raises(tg.TGError) as e:
        tg.tg_conv2d(g.h, x, 99, -1, tg.TG_SAME)
    assert e.value.code == tg.TG_E_ARG and "unknown DS id" in str(e.value)
    k = g.param(np.zeros((1, 2, 3, 3), np.float32))
    with pytest.raises(tg.TGError) as e:
        g.conv2d(x, k, -1, tg.TG_SAME)
    assert e.value.code == tg.TG_E_SHAPE
    with pytest.raises(tg.TGError) as e:
        tg.tg_set_shard(g.h, 2, 2)
    assert e.value.code == tg.TG_E_ARG
    with pytest.raises(tg.TGError) as e:   # no output bound
        g.plan()
    assert e.value.code == tg.TG_E_STATE


def test_cnn_n5_range_is_checked():
    """tg_cnn takes 1 <= n5 <= 128 (include/tg.h; the tensor-core U3 holds n5 padded to 16 maps in
    one 128-column accumulator): outside that range the graph call fails with TG_E_ARG."""
    from paper_conf_ipps_sundaramrc09_b200 import tg
    for n5 in (0, 129):
        g = tg.Graph()
        x = g.input(np.zeros((1, 1, 64, 64), np.float32))
        prm = [g.param(np.zeros((1, 1, 1, 1), np.float32)) for _ in range(10)]
        with pytest.raises(tg.TGError) as e:
            g.cnn(x, n5, prm)
        assert e.value.code == tg.TG_E_ARG and "n5" in str(e.value)


def test_unsupported_graph_and_infeasible_budget():
    from paper_conf_ipps_sundaramrc09_b200 import tg
    img = np.zeros((1, 1, 64, 64), np.float32)
    g = tg.Graph()
    x = g.input(img)
    y = tg.tg_tanh(g.h, x)
    g.output(y, np.zeros_like(img))
    with pytest.raises(tg.TGError) as e:
        g.plan()
    assert e.value.code == tg.TG_E_UNSUPPORTED
    K = np.ones((16, 16), np.float32)
    g, _ = tg.edge_graph(img, K, out=np.zeros_like(img))
    g.set(budget=4096)
    with pytest.raises(tg.TGError) as e:
        g.plan()
    assert e.value.code == tg.TG_E_INFEASIBLE


def test_shapes_and_templates_build():
    from paper_conf_ipps_sundaramrc09_b200 import tg
    import synth
    H, W = 480, 640
    img = np.zeros((2, 1, H, W), np.float32)
    prm = synth.cnn_params_np(1, 120, H, W)
    g, y = tg.cnn_graph(img, 120, prm)
    assert g.shape(y) == (2, 9, 113, 153)
    g2, e = tg.edge_graph(img[:1], np.ones((16, 16), np.float32))
    assert g2.shape(e) == (1, 1, H, W)


def test_plan_stats_match_table1_counts():
    """Stats of a planned template reproduce Table 1 and the operator/DS
    counts of PAPER.md:637 through the library's own accounting."""
    from paper_conf_ipps_sundaramrc09_b200 import tg
    import synth
    img = np.zeros((1, 1, 1000, 1000), np.float32)
    g, _ = tg.edge_graph(img, np.ones((16, 16), np.float32), out=np.zeros_like(img))
    s = g.plan().stats()
    assert s["io_lower_bound_bytes"] == 2000512 * 4 and s["total_temp_bytes"] == 6000512 * 4
    assert s["n_ops_fig7"] == 5 and s["n_ds_fig7"] == 8
    for n5, total, io, ops, ds in [(20, 59308709, 4870082, 1600, 2434), (120, 163093609, 6649882, 7500, 11334)]:
        img = np.zeros((1, 1, 480, 640), np.float32)
        prm = synth.cnn_params_np(1, n5, 480, 640)
        out = np.zeros((1, 9, 113, 153), np.float32)
        g, _ = tg.cnn_graph(img, n5, prm, out=out)
        s = g.plan().stats()
        assert (s["total_temp_bytes"], s["io_lower_bound_bytes"]) == (total * 4, io * 4)
        assert (s["n_ops_fig7"], s["n_ds_fig7"]) == (ops, ds)


def test_degenerate_shapes_rejected():
    """Empty inputs are a shape error at graph construction (no plan, no launch); a CNN image
    smaller than the receptive field (32 x 32 input -> 1 x 1 output) cannot be
    built: its C5/C6 planes would be empty."""
    from paper_conf_ipps_sundaramrc09_b200 import tg
    import synth
    for shape in [(0, 1, 8, 8), (1, 1, 0, 8), (1, 1, 8, 0)]:
        g = tg.Graph()
        with pytest.raises(tg.TGError) as e:
            g.input(np.zeros(shape, np.float32))
        assert e.value.code == tg.TG_E_SHAPE
    prm = synth.cnn_params_np(1, 20, 32, 32)
    g, y = tg.cnn_graph(np.zeros((1, 1, 32, 32), np.float32), 20, prm)
    assert g.shape(y) == (1, 9, 1, 1)
    g = tg.Graph()
    x = g.input(np.zeros((1, 1, 4, 4), np.float32))
    k = g.param(np.zeros((8, 1, 5, 5), np.float32))
    with pytest.raises(tg.TGError) as e:   # VALID 5x5 on a 4x4 image: empty output
        g.conv2d(x, k, -1, tg.TG_VALID)
    assert e.value.code == tg.TG_E_SHAPE


def test_oplib_descriptor_abi_and_validation(tmp_path):
    """tg_oplib_op has the same layout in C and in the binding (sizeof and field offsets from a
    program compiled against include/tg.h), and malformed descriptors are refused with TG_E_ARG
    before anything reaches the device (so this runs without a GPU)."""
    import subprocess
    from paper_conf_ipps_sundaramrc09_b200 import tg
    src = tmp_path / "abi.c"
    src.write_text('#include <stdio.h>\n#include <stddef.h>\n#include "tg.h"\nint main(void) {\n'
                   '  printf("%zu %zu %zu %zu %zu %zu\\n", sizeof(tg_oplib_op), offsetof(tg_oplib_op, in_dims),\n'
                   '         offsetof(tg_oplib_op, y), offsetof(tg_oplib_op, r0), offsetof(tg_oplib_op, a),\n'
                   '         sizeof(tg_oplib_view));\n  return 0;\n}\n')
    exe = tmp_path / "abi"
    subprocess.check_call(["gcc", "-std=c11", "-I", os.path.join(ROOT, "include"), "-o", str(exe), str(src)])
    got = [int(v) for v in subprocess.check_output([str(exe)], text=True).split()]
    T = tg.tg_oplib_op
    assert got == [ctypes.sizeof(T), T.in_dims.offset, T.y.offset, T.r0.offset, T.a.offset,
                   ctypes.sizeof(tg.tg_oplib_view)]
    op = tg.tg_oplib_op()
    with pytest.raises(tg.TGError) as e:          # no inputs
        tg.tg_oplib_run(op)
    assert e.value.code == tg.TG_E_ARG
    op.nin, op.kind, op.y = 1, 7, 256            # unknown kind (the view is checked first: give one)
    op.y_dims[:] = [1, 1, 4, 4]
    op.r0, op.r1 = 0, 4
    op.in_[0].nseg = 1
    op.in_[0].seg[0].p, op.in_[0].seg[0].r0, op.in_[0].seg[0].r1 = 512, 0, 4
    with pytest.raises(tg.TGError) as e:
        tg.tg_oplib_run(op)
    assert e.value.code == tg.TG_E_ARG and "kind" in str(e.value)
    op.kind, op.nin = tg.TG_OPLIB_CONV, 2        # kernel not in one whole piece
    op.in_dims[1][:] = [1, 1, 3, 3]
    op.in_[1].nseg = 2
    with pytest.raises(tg.TGError) as e:
        tg.tg_oplib_run(op)
    assert e.value.code == tg.TG_E_ARG
    op.kind, op.nin, op.r1 = tg.TG_OPLIB_ELEM, 1, 9   # rows beyond the output
    with pytest.raises(tg.TGError) as e:
        tg.tg_oplib_run(op)
    assert e.value.code == tg.TG_E_ARG


def test_device_io_needs_one_device():
    """Device-resident inputs/outputs live on one GPU: a plan over two distinct devices would
    make every device thread dereference them (TG_E_UNSUPPORTED at planning)."""
    from paper_conf_ipps_sundaramrc09_b200 import tg
    g = tg.Graph()
    x = tg.tg_input_device(g.h, 2, 1, 64, 64, 0x1000)
    k = g.param(np.ones((1, 1, 16, 16), np.float32))
    tg.tg_output_device(g.h, g.find_edges(x, k), 0x2000)
    g.set(devices=[0, 1])
    with pytest.raises(tg.TGError) as e:
        g.plan()
    assert e.value.code == tg.TG_E_UNSUPPORTED and "one-device" in str(e.value)
    g.set(devices=[0, 0])          # the same device twice is one device's memory
    g.plan()
