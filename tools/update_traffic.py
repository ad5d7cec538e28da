"""Refresh profiles/traffic.json from the ncu full captures of a round (run here, on CPU):
(dram__bytes_read.sum + dram__bytes_write.sum) of one launch / output pixels of that launch.

  python tools/update_traffic.py gpurun_out/k1_full.ncu-rep gpurun_out/cnn_bf16_full.ncu-rep \
      gpurun_out/cnn_fp32_full.ncu-rep gpurun_out/cnn_fp32tc_full.ncu-rep

The captures are tools/prof_k1.py 15 (15 x 10000x10000 edge images) and tools/prof_cnn.py 120
[bf16] (cnn3: 64 x 480x640, n5 = 120). U1 and U2 do not depend on n5, so their figures serve
cnn3s too; the single-image cnn4 is not captured (its bias planes are not shared, so per-pixel
traffic differs) and has no entry.
"""
import csv
import io
import json
import os
import subprocess
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synth  # noqa: E402

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
NAMES = {"edge": "edge_fused_kernel (K1)", "u1": "cnn_u1_kernel (U1: C1 T S2 T)",
         "u2": "cnn_u2_kernel (U2: C3 T S4 T)", "u3": "cnn_u3_kernel (U3: C5 T C6)"}


PIPES = {"tensor_pipe_pct": "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
         "fma_pipe_pct": "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
         "issue_active_pct": "smsp__issue_active.avg.pct_of_peak_sustained_active"}


def launches(rep):
    out = subprocess.check_output(["ncu", "-i", rep, "--page", "raw", "--csv"], text=True)
    rows = list(csv.reader(io.StringIO(out)))
    hdr = rows[0]
    for r in rows[2:]:
        name = r[hdr.index("Kernel Name")]
        unit = rows[1][hdr.index("dram__bytes_read.sum")]
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}[unit]
        b = (float(r[hdr.index("dram__bytes_read.sum")]) + float(r[hdr.index("dram__bytes_write.sum")])) * scale
        pipes = {k: float(r[hdr.index(m)]) for k, m in PIPES.items() if m in hdr}
        yield name, b, pipes


def main(reps):
    dims = synth.cnn_dims(480, 640)
    opx = {"u1": 64 * dims[1][0] * dims[1][1], "u2": 64 * dims[3][0] * dims[3][1], "u3": 64 * dims[4][0] * dims[4][1]}
    out = {"_source": "ncu --set full --clock-control none captures (tools/prof_k1.py 15, tools/prof_cnn.py 120 "
                      "[bf16|fp32tc]); (dram__bytes_read.sum + dram__bytes_write.sum) of one launch / output "
                      "pixels of that launch, and the tensor / FMA pipe and issue utilisation of that launch; "
                      "written by tools/update_traffic.py"}
    for rep in reps:
        prec = "bf16_tc" if "bf16" in rep else "fp32_tc" if "fp32tc" in rep else "fp32"
        for name, b, pipes in launches(rep):
            if "edge" in name:
                out[f"edge:fp32:{NAMES['edge']}"] = {"dram_bytes_per_out_px": b / (15 * 10000 * 10000),
                                                     "note": "8 B/px algorithmic (4 in + 4 out)", **pipes}
                continue
            u = "u1" if "u1" in name else "u2" if "u2" in name else "u3" if "u3" in name else None
            if u is None:
                continue
            per = b / opx[u]
            out[f"cnn3:{prec}:{NAMES[u]}"] = {"dram_bytes_per_out_px": per, **pipes}
            if u != "u3":
                out[f"cnn3s:{prec}:{NAMES[u]}"] = {"dram_bytes_per_out_px": per, **pipes}
    json.dump(out, open(os.path.join(ROOT, "profiles", "traffic.json"), "w"), indent=1)
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main(sys.argv[1:])
