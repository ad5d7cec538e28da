"""Markdown summary of a default bench line (README.md): one row per BASELINE config
line, then the uncapped e2e values, configs[0]'s microseconds, the digest and the CPU oracle.

  python tools/bench_table.py profiles/r02/bench_default.json
"""
import json
import sys

DESC = {
    "edge": "edge 15×10000², 768 MiB",
    "edge256": "edge 1×256²",
    "cnn4": "large CNN 6400×4800, 1.5 GiB",
    "cnn26": "large CNN 26×480×640, 1.5 GiB",
    "cnn3": "large CNN 64×480×640",
    "cnn3s": "small CNN 64×480×640",
    "cnn3b": "large CNN 64×480×640, bias scalar",
}
SHORT = {"edge_fused_kernel (K1)": "K1", "cnn_u1_kernel (U1: C1 T S2 T)": "U1",
         "cnn_u2_kernel (U2: C3 T S4 T)": "U2", "cnn_u3_kernel (U3: C5 T C6)": "U3"}


def rows(j):
    head = dict(j)
    head["template"] = "edge"
    head["precision"] = j["config"]["precision"]
    head["baseline_config"] = j["config"]["baseline_config"]
    yield head
    yield from j.get("per_template", [])


def main(path):
    j = [json.loads(l) for l in open(path) if l.strip().startswith("{")][0]
    out = ["| workload, precision | cfg | value Mpx/s | e2e Mpx/s | streamed roofline | bytes / bound | "
           "dominant kernel, frac | vs oracle |", "|---|---|---|---|---|---|---|---|"]
    unc = []
    for t in rows(j):
        e = t["e2e"]
        sr = e.get("streamed_roofline")
        frac, bound = (sr["frac"], sr["bound"]) if sr else (e["streamed_roofline_frac"], e["streamed_roofline_bound"])
        r = t["roofline"]
        v = t["verified"]
        verr = f"{v['max_normwise_err']:.1e}" if v else "n/a (N > 1)"
        cfg = t["baseline_config"].replace("configs", "")
        out.append(f"| {DESC[t['template']]}, {t['precision']} | {cfg} | {t['value']:,.0f} | {e['value']:,.0f} | "
                   f"{frac:.2f} ({bound}) | {e['bytes_vs_lower_bound']:.4f} | "
                   f"{SHORT.get(r['kernel'], r['kernel'])} {r['frac']:.2f} ({r['bound']}) | {verr} |")
        if e.get("uncapped"):
            unc.append(f"{DESC[t['template']].split(',')[0]} {t['precision']} {e['uncapped']['value']:,.0f}")
    link = j["measured_peaks"]["host_link_gbs"]
    out.append("")
    out.append("Link rates measured in the run: H2D %.1f, D2H %.1f, both at once %.1f GB/s per direction; FP32 peak "
               "%.1f TFLOP/s (measured), bf16 %s TFLOP/s, HBM %s GB/s (MEASURED_PEAKS.json)." % (
                   link["h2d"], link["d2h"], link["bidir_each"], j["measured_peaks"]["fp32_tflops"],
                   next((t["roofline"]["peak"] for t in rows(j) if t["roofline"]["unit"] == "TFLOP/s"
                         and t["roofline"]["peak"] > 500), "n/a"),
                   next((t["roofline"]["peak"] for t in rows(j) if t["roofline"]["unit"] == "GB/s"), "n/a")))
    out.append("Uncapped e2e (Mpx/s): " + "; ".join(unc) + ".")
    small = next((t for t in rows(j) if t["template"] == "edge256"), None)
    if small:
        out.append(f"configs[0] (256²): {small['us_per_step_device']:.1f} µs per device step (graph replay), "
                   f"{small['us_per_step_e2e']:.1f} µs end to end.")
    c = j["checksum"]
    cb = j.get("cpu_baseline")  # rank 0 at N = 1 only
    first = f" (first share {c['digest_first_share']})" if "digest_first_share" in c else ""
    oracle = f"; CPU oracle ({cb['cores']} host cores): {cb['value']:.1f} Mpx/s ({cb['sample']})" if cb else ""
    out.append(f"N = {j['n_gpus']}: output digest {c['digest_all']}{first}{oracle}; clocks {j['clocks'].get('sm_mhz')} "
               f"MHz, reasons {j['clocks'].get('reasons')}.")
    print("\n".join(out))


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else "profiles/r02/bench_default.json")
